// epilogue.cuh — the fused per-quad epilogue shared by every contraction kernel (step a6/a7 of
// SURVEY.md §8(a)):
//   (1) assemble the 81 "generalized" counts of a quad w<x<y<z for one phenotype: index
//       27α+9β+3γ+δ with α..δ in {0 = AA, 1 = Aa, 2 = '*' (any genotype)}:
//         no '*'     -> the 16 counts of the 4-way contraction
//         one '*'    -> 3-way tables T3 of the other three SNPs
//         two '*'    -> 2-way tables T2
//         three '*'  -> 1-way tables T1
//         four '*'   -> n_p
//   (2) recover every cell with an aa genotype axis by axis, v_aa = v_* - v_AA - v_Aa
//       ("subtracting the counts for genotypes {..Y0..} and {..Y1..} from the counts
//       for the third-order genotype", applied recursively, L130-131) — after axis t the digit 2 on
//       axis t means aa; 4 axes x 27 slices x 2 subtractions = 216 per phenotype;
//   (3) K2 in double in canonical cell order (reading #4):
//       t_c = (L[r_c0 + r_c1 + 1] - L[r_c0]) - L[r_c1], K2 += t_c, c = 0..80, L[n] = lgamma(n+1);
//   (4) keep the best quads: (K2, packed index) keys offered to a per-CTA sorted top-k list in shared
//       memory (per-thread -> shared memory -> global reduction), ties by index.
#pragma once
#include "epi4_internal.cuh"

namespace epi4 {

// lower-order values of one quad (w<x<y<z) for both phenotypes
struct LowOrder {
    uint32_t t3[2][4][8];   // [p][wxy, wxz, wyz, xyz][4a+2b+c]
    uint32_t t2[2][6][4];   // [p][wx, wy, wz, xy, xz, yz][2a+b]
    uint32_t t1[2][4][2];   // [p][w, x, y, z][a]
};

__device__ __forceinline__ void load8(const uint32_t* p, uint32_t (&v)[8]) {
    uint4 a = __ldg(reinterpret_cast<const uint4*>(p));
    uint4 b = __ldg(reinterpret_cast<const uint4*>(p) + 1);
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w; v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
}
__device__ __forceinline__ void load4(const uint32_t* p, uint32_t (&v)[4]) {
    uint4 a = __ldg(reinterpret_cast<const uint4*>(p));
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
}
__device__ __forceinline__ void load_t3(const DevData& d, int i, int j, int k, int slot, LowOrder& lo) {
    const uint32_t* p = d.T3 + rank3(i, j, k) * 16;
    load8(p, lo.t3[0][slot]);
    load8(p + 8, lo.t3[1][slot]);
}
__device__ __forceinline__ void load_t2(const DevData& d, int i, int j, int slot, LowOrder& lo) {
    const uint32_t* p = d.T2 + rank2(i, j) * 8;
    load4(p, lo.t2[0][slot]);
    load4(p + 4, lo.t2[1][slot]);
}
__device__ __forceinline__ void load_t1(const DevData& d, int i, int slot, LowOrder& lo) {
    const uint32_t* p = d.T1 + (int64_t)i * 4;
    uint4 a = __ldg(reinterpret_cast<const uint4*>(p));
    lo.t1[0][slot][0] = a.x; lo.t1[0][slot][1] = a.y; lo.t1[1][slot][0] = a.z; lo.t1[1][slot][1] = a.w;
}
__device__ __forceinline__ void load_low(const DevData& d, int w, int x, int y, int z, LowOrder& lo) {
    load_t3(d, w, x, y, 0, lo);
    load_t3(d, w, x, z, 1, lo);
    load_t3(d, w, y, z, 2, lo);
    load_t3(d, x, y, z, 3, lo);
    load_t2(d, w, x, 0, lo);
    load_t2(d, w, y, 1, lo);
    load_t2(d, w, z, 2, lo);
    load_t2(d, x, y, 3, lo);
    load_t2(d, x, z, 4, lo);
    load_t2(d, y, z, 5, lo);
    load_t1(d, w, 0, lo);
    load_t1(d, x, 1, lo);
    load_t1(d, y, 2, lo);
    load_t1(d, z, 3, lo);
}

// (1) generalized counts of phenotype p; c16[8a+4b+2c+d] = 4-way counts with a..d in {0,1}
template <int P>
__device__ __forceinline__ void fill_generalized(int (&g)[81], const uint32_t (&c16)[16], const LowOrder& lo,
                                                 uint32_t np) {
#pragma unroll
    for (int c = 0; c < 81; ++c) {
        const int a = c / 27, b = (c / 9) % 3, e = (c / 3) % 3, f = c % 3;
        const int ns = (a == 2) + (b == 2) + (e == 2) + (f == 2);
        uint32_t v;
        if (ns == 0) {
            v = c16[a * 8 + b * 4 + e * 2 + f];
        } else if (ns == 1) {
            if (f == 2) v = lo.t3[P][0][a * 4 + b * 2 + e];        // (w,x,y)
            else if (e == 2) v = lo.t3[P][1][a * 4 + b * 2 + f];   // (w,x,z)
            else if (b == 2) v = lo.t3[P][2][a * 4 + e * 2 + f];   // (w,y,z)
            else v = lo.t3[P][3][b * 4 + e * 2 + f];               // (x,y,z)
        } else if (ns == 2) {
            if (e == 2 && f == 2) v = lo.t2[P][0][a * 2 + b];      // (w,x)
            else if (b == 2 && f == 2) v = lo.t2[P][1][a * 2 + e]; // (w,y)
            else if (b == 2 && e == 2) v = lo.t2[P][2][a * 2 + f]; // (w,z)
            else if (a == 2 && f == 2) v = lo.t2[P][3][b * 2 + e]; // (x,y)
            else if (a == 2 && e == 2) v = lo.t2[P][4][b * 2 + f]; // (x,z)
            else v = lo.t2[P][5][e * 2 + f];                       // (y,z)
        } else if (ns == 3) {
            if (a != 2) v = lo.t1[P][0][a];
            else if (b != 2) v = lo.t1[P][1][b];
            else if (e != 2) v = lo.t1[P][2][e];
            else v = lo.t1[P][3][f];
        } else {
            v = np;
        }
        g[c] = (int)v;
    }
}

// (2) aa recovery, axis by axis (216 subtractions)
__device__ __forceinline__ void mobius(int (&g)[81]) {
#pragma unroll
    for (int ax = 0; ax < 4; ++ax) {
        const int s = ax == 0 ? 27 : ax == 1 ? 9 : ax == 2 ? 3 : 1;
#pragma unroll
        for (int c = 0; c < 81; ++c)
            if (((c / s) % 3) == 2) g[c] = g[c] - g[c - s] - g[c - 2 * s];
    }
}

// (3) K2 in canonical order; explicit round-to-nearest adds so nothing can be reassociated
__device__ __forceinline__ double k2_score(const int (&g0)[81], const int (&g1)[81], const double* __restrict__ L) {
    double k2 = 0.0;
#pragma unroll
    for (int c = 0; c < 81; ++c) {
        const int r0 = g0[c], r1 = g1[c];
        const double t = __dsub_rn(__dsub_rn(__ldg(L + (r0 + r1 + 1)), __ldg(L + r0)), __ldg(L + r1));
        k2 = __dadd_rn(k2, t);
    }
    return k2;
}

// full epilogue for one quad given its 2 x 16 contraction counts; optionally dumps the 162 counts
__device__ __forceinline__ double score_quad(const DevData& d, int w, int x, int y, int z,
                                             const uint32_t (&c0)[16], const uint32_t (&c1)[16],
                                             uint32_t* dump_row) {
    LowOrder lo;
    load_low(d, w, x, y, z, lo);
    int g0[81], g1[81];
    fill_generalized<0>(g0, c0, lo, d.np[0]);
    fill_generalized<1>(g1, c1, lo, d.np[1]);
    mobius(g0);
    mobius(g1);
    if (dump_row) {
#pragma unroll
        for (int c = 0; c < 81; ++c) {
            dump_row[c] = (uint32_t)g0[c];
            dump_row[81 + c] = (uint32_t)g1[c];
        }
    }
    return k2_score(g0, g1, d.lgam);
}

// ---------------------------------------------------------------------------------------------
// (4) per-CTA top-k list in shared memory, updated by whole warps under a CTA spin lock.
struct TopKSmem {
    double* k2;          // [cap], sorted ascending by (k2, idx)
    uint64_t* idx;
    int* cnt;
    int* lock;
    double* thr;         // k2 of the last entry when full, +inf otherwise (monotone non-increasing)
    int cap;
};

__device__ __forceinline__ bool key_less(double ka, uint64_t ia, double kb, uint64_t ib) {
    return ka < kb || (ka == kb && ia < ib);
}

// warp-cooperative insertion of one key (all 32 lanes, lock held)
__device__ __forceinline__ void warp_insert(TopKSmem& tk, double kk, uint64_t ii) {
    const int lane = threadIdx.x & 31;
    const int cnt = *reinterpret_cast<volatile int*>(tk.cnt);
    if (cnt == tk.cap && !key_less(kk, ii, tk.k2[cnt - 1], tk.idx[cnt - 1])) return;
    int pos = 0;
    for (int base = 0; base < cnt; base += 32) {
        const int e = base + lane;
        const bool lt = e < cnt && key_less(tk.k2[e], tk.idx[e], kk, ii);
        pos += __popc(__ballot_sync(0xffffffffu, lt));
    }
    const int ncnt = cnt < tk.cap ? cnt + 1 : cnt;
    for (int e = ncnt - 1; e > pos; e -= 32) {
        const int dst = e - lane;
        double vk = 0.0;
        uint64_t vi = 0;
        const bool act = dst > pos;
        if (act) { vk = tk.k2[dst - 1]; vi = tk.idx[dst - 1]; }
        __syncwarp();
        if (act) { tk.k2[dst] = vk; tk.idx[dst] = vi; }
        __syncwarp();
    }
    if (lane == 0) {
        tk.k2[pos] = kk;
        tk.idx[pos] = ii;
        *tk.cnt = ncnt;
        if (ncnt == tk.cap) *reinterpret_cast<volatile double*>(tk.thr) = tk.k2[ncnt - 1];
    }
    __syncwarp();
}

// Offer one key per lane (has = false lanes offer nothing).  Must be called by all 32 lanes.
__device__ __forceinline__ void warp_offer(TopKSmem& tk, bool has, double key, uint64_t idx) {
    const double thr = *reinterpret_cast<volatile double*>(tk.thr);
    unsigned m = __ballot_sync(0xffffffffu, has && key <= thr);
    if (!m) return;
    const int lane = threadIdx.x & 31;
    if (lane == 0) {
        while (atomicCAS(tk.lock, 0, 1) != 0) __nanosleep(20);
        __threadfence_block();
    }
    __syncwarp();
    while (m) {
        const int src = __ffs(m) - 1;
        m &= m - 1;
        const double kk = __shfl_sync(0xffffffffu, key, src);
        const uint64_t ii = __shfl_sync(0xffffffffu, idx, src);
        warp_insert(tk, kk, ii);
    }
    __threadfence_block();
    __syncwarp();
    if (lane == 0) atomicExch(tk.lock, 0);
}

// carve the top-k state from dynamic shared memory (8-byte aligned base)
__device__ __forceinline__ TopKSmem topk_carve(unsigned char* base, int cap) {
    TopKSmem tk;
    tk.k2 = reinterpret_cast<double*>(base);
    tk.idx = reinterpret_cast<uint64_t*>(base + sizeof(double) * cap);
    tk.thr = reinterpret_cast<double*>(base + 16 * cap);
    tk.cnt = reinterpret_cast<int*>(base + 16 * cap + 8);
    tk.lock = reinterpret_cast<int*>(base + 16 * cap + 12);
    tk.cap = cap;
    return tk;
}
__host__ __device__ constexpr size_t topk_smem_bytes(int cap) { return 16 * (size_t)cap + 16; }

// load this CTA's list from its global slot (call with all threads, followed by a barrier)
__device__ __forceinline__ void topk_load(TopKSmem& tk, const SearchParams& sp, int slot, int tid, int nthr) {
    const int cnt = sp.list_cnt[slot];
    for (int e = tid; e < cnt; e += nthr) {
        tk.k2[e] = sp.list_k2[(int64_t)slot * sp.topk + e];
        tk.idx[e] = sp.list_idx[(int64_t)slot * sp.topk + e];
    }
    if (tid == 0) {
        *tk.cnt = cnt;
        *tk.lock = 0;
        *tk.thr = (cnt == tk.cap) ? sp.list_k2[(int64_t)slot * sp.topk + cnt - 1] : __longlong_as_double(0x7ff0000000000000LL);
    }
}
__device__ __forceinline__ void topk_store(TopKSmem& tk, const SearchParams& sp, int slot, int tid, int nthr) {
    const int cnt = *tk.cnt;
    for (int e = tid; e < cnt; e += nthr) {
        sp.list_k2[(int64_t)slot * sp.topk + e] = tk.k2[e];
        sp.list_idx[(int64_t)slot * sp.topk + e] = tk.idx[e];
    }
    if (tid == 0) sp.list_cnt[slot] = cnt;
}

}  // namespace epi4
