// epilogue.cuh — the fused per-quad epilogue shared by every contraction kernel (step a6/a7 of
// SURVEY.md §8(a)):
//   (1) assemble the 81 "generalized" counts of a quad w<x<y<z for one phenotype (in three slabs of 27
//       along the first SNP, see quad_eval): index
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

// ---- lower-order table access (both phenotypes of an entry are adjacent) ----------------------------
// T3 entry of (i<j<k): 16 uint32 = [p][4a+2b+c];  T2 entry of (i<j): 8 uint32 = [p][2a+b];  T1[snp]: [p][a].
__device__ __forceinline__ uint4 t3_half(const DevData& d, int i, int j, int k, int p, int a) {
    // the 4 cells with first genotype a of phenotype p
    return __ldg(reinterpret_cast<const uint4*>(d.T3 + rank3(i, j, k) * 16 + p * 8 + a * 4));
}
__device__ __forceinline__ uint2 t2_row(const DevData& d, int i, int j, int p, int a) {
    return __ldg(reinterpret_cast<const uint2*>(d.T2 + rank2(i, j) * 8 + p * 4 + a * 2));
}
__device__ __forceinline__ uint4 t2_all(const DevData& d, int i, int j, int p) {
    return __ldg(reinterpret_cast<const uint4*>(d.T2 + rank2(i, j) * 8 + p * 4));
}
__device__ __forceinline__ uint2 t1_all(const DevData& d, int i, int p) {
    return __ldg(reinterpret_cast<const uint2*>(d.T1 + (int64_t)i * 4 + p * 2));
}
__device__ __forceinline__ uint32_t u4(const uint4& v, int k) { return k == 0 ? v.x : k == 1 ? v.y : k == 2 ? v.z : v.w; }
__device__ __forceinline__ uint32_t u2(const uint2& v, int k) { return k == 0 ? v.x : v.y; }

// Slab decomposition along the first SNP (w) of the quad.  For α in {0, 1, '*'} the slab
// S_α[β][γ][δ] = G[α][β][γ][δ] holds 27 generalized counts (digits in {0, 1, 2 = '*'}):
//   slab '*' (w marginalised): T3(x,y,z), T2 of (x,y),(x,z),(y,z), T1 of x,y,z and n_p;
//   slab α in {0,1}:           the 4-way counts c16[α...], T3 of (w,x,y),(w,x,z),(w,y,z), T2 of (w,.),
//                              T1(w) — all restricted to genotype α of w.
// Möbius on the remaining three axes gives the cells r[α][...] for α = 0, 1; and, because the
// recovery is linear, r[2][...] = M3(S_*) - M3(S_0) - M3(S_1)  (PAPER.md:L126 applied on axis w).
// Cells therefore come out a-major, i.e. in canonical order c = 27a + 9b + 3c + d.
template <int P>
__device__ __forceinline__ void fill_slab_star(int (&g)[27], const DevData& d, int x, int y, int z) {
    const uint4 txyz0 = t3_half(d, x, y, z, P, 0), txyz1 = t3_half(d, x, y, z, P, 1);
    const uint4 pxy = t2_all(d, x, y, P), pxz = t2_all(d, x, z, P), pyz = t2_all(d, y, z, P);
    const uint2 sx = t1_all(d, x, P), sy = t1_all(d, y, P), sz = t1_all(d, z, P);
#pragma unroll
    for (int c = 0; c < 27; ++c) {
        const int b = c / 9, e = (c / 3) % 3, f = c % 3;
        const int ns = (b == 2) + (e == 2) + (f == 2);
        uint32_t v;
        if (ns == 0) v = b ? u4(txyz1, e * 2 + f) : u4(txyz0, e * 2 + f);
        else if (ns == 1) {
            if (f == 2) v = u4(pxy, b * 2 + e);
            else if (e == 2) v = u4(pxz, b * 2 + f);
            else v = u4(pyz, e * 2 + f);
        } else if (ns == 2) {
            if (b != 2) v = u2(sx, b);
            else if (e != 2) v = u2(sy, e);
            else v = u2(sz, f);
        } else {
            v = d.np[P];
        }
        g[c] = (int)v;
    }
}
template <int P, int A>
__device__ __forceinline__ void fill_slab_w(int (&g)[27], const uint32_t (&c16)[16], const DevData& d, int w, int x,
                                            int y, int z) {
    const uint4 twxy = t3_half(d, w, x, y, P, A), twxz = t3_half(d, w, x, z, P, A), twyz = t3_half(d, w, y, z, P, A);
    const uint2 pwx = t2_row(d, w, x, P, A), pwy = t2_row(d, w, y, P, A), pwz = t2_row(d, w, z, P, A);
    const uint2 sw = t1_all(d, w, P);
#pragma unroll
    for (int c = 0; c < 27; ++c) {
        const int b = c / 9, e = (c / 3) % 3, f = c % 3;
        const int ns = (b == 2) + (e == 2) + (f == 2);
        uint32_t v;
        if (ns == 0) v = c16[A * 8 + b * 4 + e * 2 + f];
        else if (ns == 1) {
            if (f == 2) v = u4(twxy, b * 2 + e);
            else if (e == 2) v = u4(twxz, b * 2 + f);
            else v = u4(twyz, e * 2 + f);
        } else if (ns == 2) {
            if (b != 2) v = u2(pwx, b);
            else if (e != 2) v = u2(pwy, e);
            else v = u2(pwz, f);
        } else {
            v = u2(sw, A);
        }
        g[c] = (int)v;
    }
}

// Slab α = aa of w, before recovery: S_*[c] - S_0[c] - S_1[c] (the generalized counts restricted to w = aa).
// Because the recovery is linear, M3 of it is r[2][...] (PAPER.md:L126 applied on axis w); computing it from
// the raw tables (instead of keeping M3(S_*), M3(S_0), M3(S_1) alive) holds one slab per phenotype at a time.
template <int P>
__device__ __forceinline__ void fill_slab_aa(int (&g)[27], const uint32_t (&c16)[16], const DevData& d, int w, int x,
                                             int y, int z) {
    const uint4 txyz0 = t3_half(d, x, y, z, P, 0), txyz1 = t3_half(d, x, y, z, P, 1);
    const uint4 pxy = t2_all(d, x, y, P), pxz = t2_all(d, x, z, P), pyz = t2_all(d, y, z, P);
    const uint2 sx = t1_all(d, x, P), sy = t1_all(d, y, P), sz = t1_all(d, z, P);
    const uint4 twxy0 = t3_half(d, w, x, y, P, 0), twxy1 = t3_half(d, w, x, y, P, 1);
    const uint4 twxz0 = t3_half(d, w, x, z, P, 0), twxz1 = t3_half(d, w, x, z, P, 1);
    const uint4 twyz0 = t3_half(d, w, y, z, P, 0), twyz1 = t3_half(d, w, y, z, P, 1);
    const uint4 pwx = t2_all(d, w, x, P), pwy = t2_all(d, w, y, P), pwz = t2_all(d, w, z, P);
    const uint2 sw = t1_all(d, w, P);
#pragma unroll
    for (int c = 0; c < 27; ++c) {
        const int b = c / 9, e = (c / 3) % 3, f = c % 3;
        const int ns = (b == 2) + (e == 2) + (f == 2);
        uint32_t v;
        if (ns == 0) {
            v = (b ? u4(txyz1, e * 2 + f) : u4(txyz0, e * 2 + f)) - c16[b * 4 + e * 2 + f] - c16[8 + b * 4 + e * 2 + f];
        } else if (ns == 1) {
            if (f == 2) v = u4(pxy, b * 2 + e) - u4(twxy0, b * 2 + e) - u4(twxy1, b * 2 + e);
            else if (e == 2) v = u4(pxz, b * 2 + f) - u4(twxz0, b * 2 + f) - u4(twxz1, b * 2 + f);
            else v = u4(pyz, e * 2 + f) - u4(twyz0, e * 2 + f) - u4(twyz1, e * 2 + f);
        } else if (ns == 2) {
            if (b != 2) v = u2(sx, b) - u4(pwx, b) - u4(pwx, 2 + b);
            else if (e != 2) v = u2(sy, e) - u4(pwy, e) - u4(pwy, 2 + e);
            else v = u2(sz, f) - u4(pwz, f) - u4(pwz, 2 + f);
        } else {
            v = d.np[P] - sw.x - sw.y;
        }
        g[c] = (int)v;
    }
}

// aa recovery on the three axes of a slab (strides 9, 3, 1): 3 x 9 x 2 = 54 subtractions
__device__ __forceinline__ void mobius3(int (&g)[27]) {
#pragma unroll
    for (int ax = 0; ax < 3; ++ax) {
        const int s = ax == 0 ? 9 : ax == 1 ? 3 : 1;
#pragma unroll
        for (int c = 0; c < 27; ++c)
            if (((c / s) % 3) == 2) g[c] = g[c] - g[c - s] - g[c - 2 * s];
    }
}

// ---- the fp32 K2 filter (reading #16) -----------------------------------------------------
// Stirling (ln k! = ln Gamma(k+1), z = k+1): ln k! = (k + 1/2) ln(k+1) - k + C0 + mu(k+1), C0 = ln(2 pi)/2 - 1,
// 0 < mu(z) < 1/(12 z).  In a cell the "-k" parts cancel to -1 ((n+1) - r0 - r1), so with
//     T_c = (n + 3/2) lg2(n + 2) - (r0 + 1/2) lg2(r0 + 1) - (r1 + 1/2) lg2(r1 + 1)      (fp32, MUFU lg2)
// the cell term is t_c = ln2 T_c - 1 - C0 + [mu(n+2) - mu(r0+1) - mu(r1+1)], and over the 81 cells
// K2 - (ln2 sum T_c - 81 - 81 C0) lies in (-13.5, 3.375).  With the fp32 rounding bound E(M) computed on the
// host (api.cu: filter_offset), K2 > ln2 A - 81 - 81 C0 - 13.5 - E for the computed A = sum T_c, so a quad is
// scored exactly (double, lgamma table) only if ln2 A + flt_off <= the CTA's current k-th best K2: the top-k
// is exactly the oracle's.  Per cell: 2 LOP3 + 7 FADD/FMUL + 2 FFMA + 3 MUFU, no table, no conversions
// (a count r < 2^22 becomes the float 2^23 + r by an OR of the exponent bits; r + 1 and r + 1/2 then follow
// by one exact FADD each).
__device__ __forceinline__ float lg2_approx(float x) {
    float y;
    asm("lg2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
__device__ __forceinline__ float cell_T(int r0, int r1) {
    const float m0 = __int_as_float(r0 | 0x4B000000), m1 = __int_as_float(r1 | 0x4B000000);   // 2^23 + r
    const float f0 = m0 + (1.0f - 8388608.0f), f1 = m1 + (1.0f - 8388608.0f);              // r + 1
    const float h0 = m0 + (0.5f - 8388608.0f), h1 = m1 + (0.5f - 8388608.0f);              // r + 1/2
    const float fn = f0 + f1, hn = fn - 0.5f;                                               // n + 2, n + 3/2
    float t = hn * lg2_approx(fn);
    t = fmaf(-h0, lg2_approx(f0), t);
    return fmaf(-h1, lg2_approx(f1), t);
}

// Per-quad evaluation in canonical cell order, one slab (27 cells x 2 phenotypes) at a time:
// alpha = AA (cells 0..26), Aa (27..53), aa (54..80).  MODE 0: the fp32 filter value A = sum T_c (above);
// MODE 1: exact K2 in double, t_c = (L[r+1] - L[r0]) - L[r1], K2 += t_c, c = 0..80 (
// reading #4); MODE 2: exact K2 and the 2 x 81 cells written to dump (controls first).
template <int MODE>
__device__ __forceinline__ void quad_eval(const DevData& d, int w, int x, int y, int z, const uint32_t (&c0)[16],
                                          const uint32_t (&c1)[16], float& flt, double& k2, uint32_t* dump) {
    float fa = 0.0f, fb = 0.0f;
    double kk = 0.0;
    auto consume = [&](const int (&T0)[27], const int (&T1)[27], int base) {
#pragma unroll
        for (int c = 0; c < 27; ++c) {
            const int r0 = T0[c], r1 = T1[c];
            if (MODE == 0) {
                const float t = cell_T(r0, r1);
                if (c & 1) fb += t; else fa += t;
            } else {
                const double t = __dsub_rn(__dsub_rn(__ldg(d.lgam + (r0 + r1 + 1)), __ldg(d.lgam + r0)), __ldg(d.lgam + r1));
                kk = __dadd_rn(kk, t);
                if (MODE == 2) {
                    dump[base + c] = (uint32_t)r0;
                    dump[81 + base + c] = (uint32_t)r1;
                }
            }
        }
    };
#pragma unroll
    for (int a = 0; a < 3; ++a) {
        int T0[27], T1[27];
        if (a == 0) { fill_slab_w<0, 0>(T0, c0, d, w, x, y, z); fill_slab_w<1, 0>(T1, c1, d, w, x, y, z); }
        else if (a == 1) { fill_slab_w<0, 1>(T0, c0, d, w, x, y, z); fill_slab_w<1, 1>(T1, c1, d, w, x, y, z); }
        else { fill_slab_aa<0>(T0, c0, d, w, x, y, z); fill_slab_aa<1>(T1, c1, d, w, x, y, z); }
        mobius3(T0);
        mobius3(T1);
        consume(T0, T1, 27 * a);
    }
    flt = fa + fb;
    k2 = kk;
}

// exact K2 of one quad (double, canonical order); optionally dumps its 162 cells.  Not inlined: in the
// tensor-core epilogue it runs only for filter candidates, so its registers must not add to the hot loop's.
static __device__ __noinline__ double score_quad(const DevData& d, int w, int x, int y, int z,
                                          const uint32_t (&c0)[16], const uint32_t (&c1)[16],
                                          uint32_t* dump_row) {
    float flt;
    double k2;
    if (dump_row) quad_eval<2>(d, w, x, y, z, c0, c1, flt, k2, dump_row);
    else quad_eval<1>(d, w, x, y, z, c0, c1, flt, k2, nullptr);
    return k2;
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
