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
//       axis t means aa; 108 three-input subtractions on packed (control | case) words cover both
//       phenotypes at once (section "packed counts" below);
//   (3) K2 in double in canonical cell order (reading #4):
//       t_c = (L[r_c0 + r_c1 + 1] - L[r_c0]) - L[r_c1], K2 += t_c, c = 0..80, L[n] = lgamma(n+1);
//   (4) keep the best quads: (K2, packed index) keys offered to a per-CTA sorted top-k list in shared
//       memory (per-thread -> shared memory -> global reduction), ties by index.
#pragma once
#include "epi4_internal.cuh"

namespace epi4 {

// ---- packed counts -----------------------------------------------------------------------------------
// Every count the epilogue handles is a PACKED pair v = c0 | c1 << pks (controls in the low pks bits, cases
// above).  The aa recovery of PAPER.md:L126 is a chain of subtractions v_aa = v_* - v_AA - v_Aa in which every
// operand and every result is the number of samples of one phenotype in a genotype subset, i.e. a non-negative
// count per field: no borrow ever crosses the field boundary, so one subtraction recovers both phenotypes
// exactly (half the instructions of two separate recoveries, and half the table bytes).  The packed word P is
// uint32_t with pks = bits(n0) when bits(n0) + bits(n1) <= 32 (every BASELINE.json config), else ("wide",
// DevData.wide) uint64_t with pks = 32: the same code on 64-bit words (sample counts up to 2^23 per class).
//
// Lower-order tables (api.cu / k_prep.cu, colex ranks):  T3[rank3(i,j,k)][4a+2b+c], T2[rank2(i,j)][2a+b],
// T1[snp][a], all packed P words; npk = n0 | n1 << pks.
template <typename P>
struct Q4 { P v[4]; };
template <typename P>
struct Q2 { P v[2]; };
// 4 / 2 consecutive P words at P-index e of a table
template <typename P>
__device__ __forceinline__ Q4<P> ldq4(const uint32_t* base, int64_t e) {
    Q4<P> q;
    if constexpr (sizeof(P) == 4) {
        const uint4 t = __ldg(reinterpret_cast<const uint4*>(base + e));
        q.v[0] = t.x; q.v[1] = t.y; q.v[2] = t.z; q.v[3] = t.w;
    } else {
        const ulonglong2 a = __ldg(reinterpret_cast<const ulonglong2*>(base + 2 * e));
        const ulonglong2 b = __ldg(reinterpret_cast<const ulonglong2*>(base + 2 * e) + 1);
        q.v[0] = a.x; q.v[1] = a.y; q.v[2] = b.x; q.v[3] = b.y;
    }
    return q;
}
template <typename P>
__device__ __forceinline__ Q2<P> ldq2(const uint32_t* base, int64_t e) {
    Q2<P> q;
    if constexpr (sizeof(P) == 4) {
        const uint2 t = __ldg(reinterpret_cast<const uint2*>(base + e));
        q.v[0] = t.x; q.v[1] = t.y;
    } else {
        const ulonglong2 a = __ldg(reinterpret_cast<const ulonglong2*>(base + 2 * e));
        q.v[0] = a.x; q.v[1] = a.y;
    }
    return q;
}
template <typename P>
__device__ __forceinline__ Q4<P> t3_half(const DevData& d, int64_t r3, int a) { return ldq4<P>(d.T3, r3 * 8 + a * 4); }
template <typename P>
__device__ __forceinline__ Q4<P> t3x_half(const DevData& d, int64_t r3, int a) { return ldq4<P>(d.T3x, r3 * 8 + a * 4); }
template <typename P>
__device__ __forceinline__ Q4<P> t2_all(const DevData& d, int64_t r2) { return ldq4<P>(d.T2, r2 * 4); }
template <typename P>
__device__ __forceinline__ Q2<P> t1_all(const DevData& d, int i) { return ldq2<P>(d.T1, (int64_t)i * 2); }
template <typename P>
__device__ __forceinline__ P npk_of(const DevData& d) {
    return sizeof(P) == 4 ? (P)d.npk : (P)d.np[0] | ((P)d.np[1] << 32);
}

// colex ranks of the lower-order tables a quad w < x < y < z reads
struct QuadRanks {
    int64_t wxy, wxz, wyz, xyz;   // T3
    int64_t wx, wy, wz, xy, xz, yz;   // T2
};
// T3 entries: resident (colex rank3) or windowed (slab entries, epi4_internal.cuh DevData); xyz is read from T3x
__device__ __forceinline__ QuadRanks quad_ranks(const DevData& d, int w, int x, int y, int z) {
    QuadRanks q;
    const int64_t c2x = c2(x), c2y = c2(y), c2z = c2(z);
    if (d.t3_win) {
        const int64_t pn = c2(d.n), bw = (int64_t)(w - d.t3_w0) * pn;
        q.wxy = bw + c2y + x;
        q.wxz = bw + c2z + x;
        q.wyz = bw + c2z + y;
        q.xyz = (int64_t)(x - d.t3_x0) * pn + c2z + y;
    } else {
        const int64_t c3y = c3(y), c3z = c3(z);
        q.wxy = c3y + c2x + w;
        q.wxz = c3z + c2x + w;
        q.wyz = c3z + c2y + w;
        q.xyz = c3z + c2y + x;
    }
    q.wx = c2x + w;
    q.wy = c2y + w;
    q.wz = c2z + w;
    q.xy = c2y + x;
    q.xz = c2z + x;
    q.yz = c2z + y;
    return q;
}

// Generalized counts of one slab along the first SNP w: for w-genotype A in {AA, Aa}
// or '*' (any), S[9b + 3e + f] with digits b (x), e (y), f (z) in {0 = AA, 1 = Aa, 2 = '*'}:
//   no '*'    -> the 4-way contraction counts c16[8A + 4b + 2e + f]
//   one '*'   -> 3-way tables of the other three SNPs
//   two '*'   -> 2-way tables
//   three '*' -> 1-way table / n_p
template <int A, typename P>
__device__ __forceinline__ void fill_slab_w(P (&S)[27], const P (&c16)[16], const Q4<P>& twxy, const Q4<P>& twxz,
                                            const Q4<P>& twyz, const Q4<P>& pwx, const Q4<P>& pwy, const Q4<P>& pwz,
                                            const Q2<P>& sw) {
#pragma unroll
    for (int c = 0; c < 27; ++c) {
        const int b = c / 9, e = (c / 3) % 3, f = c % 3;
        const int ns = (b == 2) + (e == 2) + (f == 2);
        P v;
        if (ns == 0) v = c16[A * 8 + b * 4 + e * 2 + f];
        else if (ns == 1) {
            if (f == 2) v = twxy.v[b * 2 + e];
            else if (e == 2) v = twxz.v[b * 2 + f];
            else v = twyz.v[e * 2 + f];
        } else if (ns == 2) {
            if (b != 2) v = pwx.v[A * 2 + b];
            else if (e != 2) v = pwy.v[A * 2 + e];
            else v = pwz.v[A * 2 + f];
        } else {
            v = sw.v[A];
        }
        S[c] = v;
    }
}
// slab w = '*': the (x, y, z) marginal tables
template <typename P>
__device__ __forceinline__ void fill_slab_star(P (&S)[27], const Q4<P>& txyz0, const Q4<P>& txyz1, const Q4<P>& pxy,
                                               const Q4<P>& pxz, const Q4<P>& pyz, const Q2<P>& sx, const Q2<P>& sy,
                                               const Q2<P>& sz, P npk) {
#pragma unroll
    for (int c = 0; c < 27; ++c) {
        const int b = c / 9, e = (c / 3) % 3, f = c % 3;
        const int ns = (b == 2) + (e == 2) + (f == 2);
        P v;
        if (ns == 0) v = b ? txyz1.v[e * 2 + f] : txyz0.v[e * 2 + f];
        else if (ns == 1) {
            if (f == 2) v = pxy.v[b * 2 + e];
            else if (e == 2) v = pxz.v[b * 2 + f];
            else v = pyz.v[e * 2 + f];
        } else if (ns == 2) {
            if (b != 2) v = sx.v[b];
            else if (e != 2) v = sy.v[e];
            else v = sz.v[f];
        } else {
            v = npk;
        }
        S[c] = v;
    }
}

// aa recovery on the three axes of a slab (strides 9, 3, 1): 27 three-input subtractions on packed words
template <typename P>
__device__ __forceinline__ void mobius3(P (&g)[27]) {
#pragma unroll
    for (int ax = 0; ax < 3; ++ax) {
        const int s = ax == 0 ? 9 : ax == 1 ? 3 : 1;
#pragma unroll
        for (int c = 0; c < 27; ++c)
            if (((c / s) % 3) == 2) g[c] = g[c] - g[c - s] - g[c - 2 * s];
    }
}

// the two counts of a packed word, as 32-bit integers (r0 controls, r1 cases)
template <typename P>
__device__ __forceinline__ uint32_t cnt0(P v, uint32_t pks, uint32_t pkm) {
    return sizeof(P) == 4 ? (uint32_t)v & pkm : (uint32_t)v;
}
template <typename P>
__device__ __forceinline__ uint32_t cnt1(P v, uint32_t pks) {
    return sizeof(P) == 4 ? (uint32_t)(v >> pks) : (uint32_t)(v >> 32);
}
// 2^23 + r0, 2^23 + r1 as floats (exact for counts < 2^23); with 16-bit fields one byte permute each
template <bool PK16, typename P>
__device__ __forceinline__ void cnt_f(P v, uint32_t pks, uint32_t pkm, float& m0, float& m1) {
    if constexpr (sizeof(P) == 4 && PK16) {
        m0 = __uint_as_float(__byte_perm((uint32_t)v, 0x4B000000u, 0x7410));
        m1 = __uint_as_float(__byte_perm((uint32_t)v, 0x4B000000u, 0x7432));
    } else {
        m0 = __uint_as_float(cnt0(v, pks, pkm) | 0x4B000000u);
        m1 = __uint_as_float(cnt1(v, pks) | 0x4B000000u);
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
// is exactly the oracle's.  Per cell: 3 ALU (unpack; 2 with pks = 16), 6 FADD + 3 FFMA into a running sum, 3 MUFU
// (with EPI4_FILTER_F2 the paired form cell_T_acc2 below: two running sums in the lanes of an fp32 pair);
// no table and no conversion instruction (a count r < 2^23 becomes the float 2^23 + r by setting the exponent
// bits).
__device__ __forceinline__ float lg2_approx(float x) {
    float y;
    asm("lg2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
template <bool PK16, typename P>
__device__ __forceinline__ void cell_T_acc(P v, uint32_t pks, uint32_t pkm, float& acc) {
    float m0, m1;
    cnt_f<PK16>(v, pks, pkm, m0, m1);
    const float f0 = m0 - 8388607.0f, f1 = m1 - 8388607.0f;     // r + 1
    const float h0 = m0 - 8388607.5f, h1 = m1 - 8388607.5f;     // r + 1/2
    const float fn = f0 + f1, hn = h0 + f1;                     // n + 2, n + 3/2
    acc = fmaf(hn, lg2_approx(fn), acc);   // the cell's three terms go straight into the running sum
    acc = fmaf(-h0, lg2_approx(f0), acc);  // (rounding bound: api.cu filter_offset)
    acc = fmaf(-h1, lg2_approx(f1), acc);
}

#ifndef EPI4_FILTER_F2
#define EPI4_FILTER_F2 0    // 1: the paired FFMA2 filter below (fewer instructions, measured 1.5 % slower at C2, profiles/r02l_topk.log)
#endif
// The same cell terms for two cells at once with sm_100's packed fp32 pairs (FADD2 / FFMA2: two IEEE
// round-to-nearest operations per instruction, lane-wise identical to the scalar ones): cell a goes to lane 0 and
// cell b to lane 1 of the running pair acc2, each lane adding its cell's three terms in the scalar order above,
// so the rounding bound (api.cu filter_offset: every rounding <= u times a partial sum of cell terms) is unchanged.
// Per two cells: 4 PRMT, 6 FADD2, 6 MUFU, 3 FFMA2 (19 instructions instead of 28).
__device__ __forceinline__ uint64_t f2_pack(float lo, float hi) {
    uint64_t r;
    asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(lo), "f"(hi));
    return r;
}
__device__ __forceinline__ void f2_unpack(uint64_t v, float& lo, float& hi) {
    asm("mov.b64 {%0, %1}, %2;" : "=f"(lo), "=f"(hi) : "l"(v));
}
__device__ __forceinline__ uint64_t f2_add(uint64_t a, uint64_t b) {
    uint64_t r;
    asm("add.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
__device__ __forceinline__ uint64_t f2_sub(uint64_t a, uint64_t b) {
    uint64_t r;
    asm("sub.rn.f32x2 %0, %1, %2;" : "=l"(r) : "l"(a), "l"(b));
    return r;
}
__device__ __forceinline__ uint64_t f2_fma(uint64_t a, uint64_t b, uint64_t c) {
    uint64_t r;
    asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(r) : "l"(a), "l"(b), "l"(c));
    return r;
}
__device__ __forceinline__ uint64_t f2_lg2(uint64_t v) {
    float lo, hi;
    f2_unpack(v, lo, hi);
    return f2_pack(lg2_approx(lo), lg2_approx(hi));
}
template <bool PK16, typename P>
__device__ __forceinline__ void cell_T_acc2(P va, P vb, uint32_t pks, uint32_t pkm, uint64_t& acc2) {
    float a0, a1, b0, b1;
    cnt_f<PK16>(va, pks, pkm, a0, a1);
    cnt_f<PK16>(vb, pks, pkm, b0, b1);
    const uint64_t m0 = f2_pack(a0, b0), m1 = f2_pack(a1, b1);            // 2^23 + r0, 2^23 + r1 of both cells
    const uint64_t c1 = f2_pack(8388607.0f, 8388607.0f), ch = f2_pack(8388607.5f, 8388607.5f);
    const uint64_t f0 = f2_sub(m0, c1), f1 = f2_sub(m1, c1);             // r + 1
    const uint64_t nh0 = f2_sub(ch, m0), nh1 = f2_sub(ch, m1);           // -(r + 1/2), exact
    const uint64_t fn = f2_add(f0, f1);                                   // n + 2
    const uint64_t hn = f2_sub(f1, nh0);                                  // n + 3/2 = (r0 + 1/2) + (r1 + 1)
    acc2 = f2_fma(hn, f2_lg2(fn), acc2);
    acc2 = f2_fma(nh0, f2_lg2(f0), acc2);
    acc2 = f2_fma(nh1, f2_lg2(f1), acc2);
}

// ---- the fp32 chi-square filter (EPI4_OBJ_CHI2) ---------------------------------------------------------
// X^2 + M = sum_{c} u_c with u_c = (r0^2 (M/n0) + r1^2 (M/n1)) / r_c (cells with r_c = 0 give 0: the
// numerator is 0 and the divisor is clamped to 1).  In fp32 every count is exact (< 2^23, exponent-bit
// conversion as in cell_T_acc), each u_c carries at most ~8 roundings (alpha/beta, 2 products, FMA, rcp.approx,
// product; each <= 2^-23 relative), and the three running sums of positive terms add <= 29 more, so the
// computed sum U satisfies |U - (X^2 + M)| <= 40 * 2^-23 (X^2 + M) < 2^-17 (X^2 + M).  The kernel scores a
// quad exactly only if -(U (1 + 2^-12) - M) <= the current k-th best key: 2^-12 is 32x the bound.
__device__ __forceinline__ float rcp_approx(float x) {
    float y;
    asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
    return y;
}
template <bool PK16, typename P>
__device__ __forceinline__ void cell_chi_acc(P v, uint32_t pks, uint32_t pkm, float ca, float cb, float& acc) {
    float m0, m1;
    cnt_f<PK16>(v, pks, pkm, m0, m1);
    const float f0 = m0 - 8388608.0f, f1 = m1 - 8388608.0f;     // r0, r1 (exact)
    const float num = fmaf(f0 * ca, f0, (f1 * cb) * f1);
    acc = fmaf(num, rcp_approx(fmaxf(f0 + f1, 1.0f)), acc);
}

// ---- the fp32 mutual-information filter (EPI4_OBJ_MI) ----------------------------------------------------
// M*I = ln2 V + mi_const with V = sum_c [X2(r0) + X2(r1) - X2(r_c)], X2(k) = k lg2 k (X2(0) = 0: lg2 of
// max(k, 1)).  Each cell value is formed first (two FMAs onto -r_c lg2 r_c; |value| <= r_c bits), then added
// to a running sum, so |V_computed - V| <= mi_E (api.cu: lg2.approx, the cell roundings, the additions).
// The kernel scores a quad exactly only if -(ln2 (V + mi_E) + mi_const) <= the current k-th best key.
template <bool PK16, typename P>
__device__ __forceinline__ void cell_mi_acc(P v, uint32_t pks, uint32_t pkm, float& acc) {
    float m0, m1;
    cnt_f<PK16>(v, pks, pkm, m0, m1);
    const float f0 = m0 - 8388608.0f, f1 = m1 - 8388608.0f, fn = f0 + f1;   // r0, r1, r_c (exact)
    const float cell = fmaf(f0, lg2_approx(fmaxf(f0, 1.0f)), fmaf(f1, lg2_approx(fmaxf(f1, 1.0f)),
                                                                  -fn * lg2_approx(fmaxf(fn, 1.0f))));
    acc += cell;
}

// Per-quad evaluation from the 16 packed contraction counts c16[8a + 4b + 2c + d] of quad (w, x, y, z).
// Slabs along w: R2 := M3(S_*) (the recovered (x, y, z) table); for A = AA, Aa: r_A = M3(S_A) is consumed
// and subtracted from R2, which ends as r_aa = M3(S_*) - M3(S_AA) - M3(S_Aa) (linearity of the recovery,
// PAPER.md:L126 applied on axis w).  Cells are consumed slab by slab in canonical order c = 27a + 9b + 3c + d.
// MODE 0: the fp32 filter value A = sum T_c (above); MODE 5: the fp32 chi-square sum U ~ X^2 + M (above);
// MODE 6: the fp32 MI sum V (above); MODE 1: exact K2 in double, t_c = (L[r_c0 + r_c1 + 1] -
// L[r_c0]) - L[r_c1], K2 += t_c, c = 0..80 (reading #4); MODE 2: exact K2 and the
// 2 x 81 cells written to dump (controls first).
template <int MODE, bool PK16 = false, typename P = uint32_t>
__device__ __forceinline__ void quad_eval(const DevData& d, const QuadRanks& q, int w, int x, int y, int z,
                                          const P (&c16)[16], float& flt, double& k2, uint32_t* dump) {
    const uint32_t pks = (uint32_t)d.pk_shift, pkm = sizeof(P) == 4 ? (1u << pks) - 1u : 0xFFFFFFFFu;
    // all table reads up front (one round of load latency per quad)
    const Q4<P> txyz0 = t3x_half<P>(d, q.xyz, 0), txyz1 = t3x_half<P>(d, q.xyz, 1);
    const Q4<P> pxy = t2_all<P>(d, q.xy), pxz = t2_all<P>(d, q.xz), pyz = t2_all<P>(d, q.yz);
    const Q2<P> sx = t1_all<P>(d, x), sy = t1_all<P>(d, y), sz = t1_all<P>(d, z);
    const Q4<P> twxy0 = t3_half<P>(d, q.wxy, 0), twxz0 = t3_half<P>(d, q.wxz, 0), twyz0 = t3_half<P>(d, q.wyz, 0);
    const Q4<P> twxy1 = t3_half<P>(d, q.wxy, 1), twxz1 = t3_half<P>(d, q.wxz, 1), twyz1 = t3_half<P>(d, q.wyz, 1);
    const Q4<P> pwx = t2_all<P>(d, q.wx), pwy = t2_all<P>(d, q.wy), pwz = t2_all<P>(d, q.wz);
    const Q2<P> sw = t1_all<P>(d, w);
    float fa = 0.0f, fb = 0.0f, fc = 0.0f;
    uint64_t acc2 = 0;   // MODE 0: two running sums (+0.0f, +0.0f) in the lanes of an fp32 pair
    double kk = 0.0;
    auto consume = [&](const P (&S)[27], int base) {
        if constexpr (MODE == 0 && EPI4_FILTER_F2) {   // cells 2j, 2j+1 of the slab as a pair, cell 26 into lane 0
#pragma unroll
            for (int c = 0; c + 1 < 27; c += 2) cell_T_acc2<PK16>(S[c], S[c + 1], pks, pkm, acc2);
            float lo, hi;
            f2_unpack(acc2, lo, hi);
            cell_T_acc<PK16>(S[26], pks, pkm, lo);
            acc2 = f2_pack(lo, hi);
        } else {
#pragma unroll
        for (int c = 0; c < 27; ++c) {
            if (MODE == 0) {
                cell_T_acc<PK16>(S[c], pks, pkm, c % 3 == 0 ? fa : c % 3 == 1 ? fb : fc);
            } else if (MODE == 6) {
                cell_mi_acc<PK16>(S[c], pks, pkm, c % 3 == 0 ? fa : c % 3 == 1 ? fb : fc);
            } else if (MODE == 5) {
                cell_chi_acc<PK16>(S[c], pks, pkm, d.chi_a, d.chi_b, c % 3 == 0 ? fa : c % 3 == 1 ? fb : fc);
            } else if (MODE == 4) {
                // Pearson chi-square (EPI4_OBJ_CHI2): S += (r0^2 n1 + r1^2 n0) / r_c over cells with r_c > 0,
                // exact uint64 numerator, one correctly rounded division (oracle_chi2's order)
                const uint32_t r0 = cnt0(S[c], pks, pkm), r1 = cnt1(S[c], pks), rc = r0 + r1;
                if (rc) {
                    const unsigned long long num = (unsigned long long)r0 * r0 * d.np[1] +
                                                   (unsigned long long)r1 * r1 * d.np[0];
                    kk = __dadd_rn(kk, __ddiv_rn(__ull2double_rn(num), __uint2double_rn(rc)));
                }
            } else if (MODE == 3) {
                // mutual information (EPI4_OBJ_MI): (X(r0) + X(r1)) - X(r0 + r1), X(k) = k ln k
                const uint32_t r0 = cnt0(S[c], pks, pkm), r1 = cnt1(S[c], pks);
                kk = __dadd_rn(kk, __dsub_rn(__dadd_rn(__ldg(d.xlx + r0), __ldg(d.xlx + r1)), __ldg(d.xlx + (r0 + r1))));
            } else {
                const uint32_t r0 = cnt0(S[c], pks, pkm), r1 = cnt1(S[c], pks);
                const double t = __dsub_rn(__dsub_rn(__ldg(d.lgam + (r0 + r1 + 1)), __ldg(d.lgam + r0)), __ldg(d.lgam + r1));
                kk = __dadd_rn(kk, t);
                if (MODE == 2) {
                    dump[base + c] = r0;
                    dump[81 + base + c] = r1;
                }
            }
        }
        }
    };
    P R2[27];
    fill_slab_star<P>(R2, txyz0, txyz1, pxy, pxz, pyz, sx, sy, sz, npk_of<P>(d));
    mobius3(R2);
    {
        P S[27];
        fill_slab_w<0, P>(S, c16, twxy0, twxz0, twyz0, pwx, pwy, pwz, sw);
        mobius3(S);
        consume(S, 0);
#pragma unroll
        for (int c = 0; c < 27; ++c) R2[c] -= S[c];
    }
    {
        P S[27];
        fill_slab_w<1, P>(S, c16, twxy1, twxz1, twyz1, pwx, pwy, pwz, sw);
        mobius3(S);
        consume(S, 27);
#pragma unroll
        for (int c = 0; c < 27; ++c) R2[c] -= S[c];
    }
    consume(R2, 54);
    if (MODE == 0 && EPI4_FILTER_F2) {
        float lo, hi;
        f2_unpack(acc2, lo, hi);
        flt = lo + hi;
    } else {
        flt = fa + fb + fc;
    }
    if (MODE == 4) {   // chi-square: X^2 = M S / (n0 n1) - M (0 with an empty phenotype); key = -X^2
        const double n0 = __uint2double_rn(d.np[0]), n1 = __uint2double_rn(d.np[1]), M = __dadd_rn(n0, n1);
        k2 = (d.np[0] == 0 || d.np[1] == 0) ? 0.0 : -__dsub_rn(__ddiv_rn(__dmul_rn(M, kk), __dmul_rn(n0, n1)), M);
    } else {
        k2 = MODE == 3 ? -__dadd_rn(kk, d.mi_const) : kk;   // MI: key = -M*I (largest MI first)
    }
}

// exact K2 of one quad (double, canonical order) from its packed contraction counts; optionally dumps its 162
// cells.  Not inlined: in the tensor-core epilogue it runs only for filter candidates, so its registers must
// not add to the hot loop's.
template <typename P = uint32_t>
static __device__ __noinline__ double score_quad(const DevData& d, int w, int x, int y, int z, const P (&c16)[16],
                                                 uint32_t* dump_row) {
    float flt;
    double k2;
    const QuadRanks q = quad_ranks(d, w, x, y, z);
    if (dump_row) quad_eval<2, false, P>(d, q, w, x, y, z, c16, flt, k2, dump_row);
    else if (d.objective == EPI4_OBJ_MI) quad_eval<3, false, P>(d, q, w, x, y, z, c16, flt, k2, nullptr);
    else if (d.objective == EPI4_OBJ_CHI2) quad_eval<4, false, P>(d, q, w, x, y, z, c16, flt, k2, nullptr);
    else quad_eval<1, false, P>(d, q, w, x, y, z, c16, flt, k2, nullptr);
    return k2;
}
// Call-site wrapper for the hot loops: the counts are copied into an array local to the (rare) branch that
// calls the noinline scorer, so the loop's own c16 never has its address taken and stays in registers (passing
// c16 itself made the compiler store all 16 counts to the stack on every quad: 1.5 G STL per C2 slice, ncu).
template <typename P = uint32_t>
static __device__ __forceinline__ double score_quad_rare(const DevData& d, int w, int x, int y, int z,
                                                         const P (&c16)[16], uint32_t* dump_row) {
    P t[16];
#pragma unroll
    for (int k = 0; k < 16; ++k) t[k] = c16[k];
    return score_quad<P>(d, w, x, y, z, t, dump_row);
}
// Verification sample (epi4_set_sample): is quad `idx` sampled?  Then record it: packed index, exact key of the
// context's objective and its 2 x 81 counts, from the counts the search kernel itself produced.  Returns the
// exact key through `key` (the quad is then offered to the top-k with it).  Slots beyond samp_cap are counted only.
__device__ __forceinline__ bool sample_hit(const SearchParams& sp, uint64_t idx) {
    return sp.samp_cap && (mix64(idx ^ sp.samp_seed) & sp.samp_mask) == 0;
}
template <typename P = uint32_t>
static __device__ __noinline__ double sample_record(const SearchParams& sp, int w, int x, int y, int z,
                                                    const P (&c16)[16]) {
    const unsigned long long slot = atomicAdd(sp.samp_n, 1ull);
    uint32_t scratch[162];
    uint32_t* row = slot < (unsigned long long)sp.samp_cap ? sp.samp_counts + slot * 162 : scratch;
    double key = score_quad<P>(sp.d, w, x, y, z, c16, row);            // K2 + counts
    if (sp.d.objective != EPI4_OBJ_K2) key = score_quad<P>(sp.d, w, x, y, z, c16, nullptr);
    if (slot < (unsigned long long)sp.samp_cap) {
        sp.samp_idx[slot] = pack_quad(w, x, y, z);
        sp.samp_key[slot] = key;
    }
    return key;
}
template <typename P = uint32_t>
static __device__ __forceinline__ double sample_record_rare(const SearchParams& sp, int w, int x, int y, int z,
                                                            const P (&c16)[16]) {
    P t[16];
#pragma unroll
    for (int k = 0; k < 16; ++k) t[k] = c16[k];
    return sample_record<P>(sp, w, x, y, z, t);
}

// Third-order search: exact K2 of triple w < x < y from its 8 packed non-aa counts
// c8[4a + 2b + c] (the 3-way-table mode's d = AA columns), the same recovery one order lower: generalized
// cells S[9a + 3b + c] (digit 2 = '*') from c8, T2, T1 and n, aa recovered on the three axes,
// K2 = sum_c ((L[r_c + 1] - L[r_c0]) - L[r_c1]) in canonical order c = 9a + 3b + c (reading #4); with
// EPI4_OBJ_MI / EPI4_OBJ_CHI2 the key is -M*I / -X^2 of the 2 x 27 table, as in quad_eval MODE 3 / 4.
template <typename P = uint32_t>
static __device__ __noinline__ double score_triple(const DevData& d, int w, int x, int y, const P (&c8)[8]) {
    const uint32_t pks = (uint32_t)d.pk_shift, pkm = sizeof(P) == 4 ? (1u << pks) - 1u : 0xFFFFFFFFu;
    const Q4<P> pwx = t2_all<P>(d, c2(x) + w), pwy = t2_all<P>(d, c2(y) + w), pxy = t2_all<P>(d, c2(y) + x);
    const Q2<P> sw = t1_all<P>(d, w), sx = t1_all<P>(d, x), sy = t1_all<P>(d, y);
    P S[27];
#pragma unroll
    for (int c = 0; c < 27; ++c) {
        const int a = c / 9, b = (c / 3) % 3, e = c % 3;
        const int ns = (a == 2) + (b == 2) + (e == 2);
        P v;
        if (ns == 0) v = c8[4 * a + 2 * b + e];
        else if (ns == 1) {
            if (a == 2) v = pxy.v[2 * b + e];
            else if (b == 2) v = pwy.v[2 * a + e];
            else v = pwx.v[2 * a + b];
        } else if (ns == 2) {
            if (a != 2) v = sw.v[a];
            else if (b != 2) v = sx.v[b];
            else v = sy.v[e];
        } else {
            v = npk_of<P>(d);
        }
        S[c] = v;
    }
    mobius3(S);
    double kk = 0.0;
    if (d.objective == EPI4_OBJ_MI) {   // -M*I over the 27 cells (oracle mi_27's order)
#pragma unroll
        for (int c = 0; c < 27; ++c) {
            const uint32_t r0 = cnt0(S[c], pks, pkm), r1 = cnt1(S[c], pks);
            kk = __dadd_rn(kk, __dsub_rn(__dadd_rn(__ldg(d.xlx + r0), __ldg(d.xlx + r1)), __ldg(d.xlx + (r0 + r1))));
        }
        return -__dadd_rn(kk, d.mi_const);
    }
    if (d.objective == EPI4_OBJ_CHI2) {   // -X^2 over the 27 cells (oracle chi2_27's order)
        if (d.np[0] == 0 || d.np[1] == 0) return 0.0;
#pragma unroll
        for (int c = 0; c < 27; ++c) {
            const uint32_t r0 = cnt0(S[c], pks, pkm), r1 = cnt1(S[c], pks), rc = r0 + r1;
            if (rc) {
                const unsigned long long num = (unsigned long long)r0 * r0 * d.np[1] +
                                               (unsigned long long)r1 * r1 * d.np[0];
                kk = __dadd_rn(kk, __ddiv_rn(__ull2double_rn(num), __uint2double_rn(rc)));
            }
        }
        const double n0 = __uint2double_rn(d.np[0]), n1 = __uint2double_rn(d.np[1]), M = __dadd_rn(n0, n1);
        return -__dsub_rn(__ddiv_rn(__dmul_rn(M, kk), __dmul_rn(n0, n1)), M);
    }
#pragma unroll
    for (int c = 0; c < 27; ++c) {
        const uint32_t r0 = cnt0(S[c], pks, pkm), r1 = cnt1(S[c], pks);
        kk = __dadd_rn(kk, __dsub_rn(__dsub_rn(__ldg(d.lgam + (r0 + r1 + 1)), __ldg(d.lgam + r0)), __ldg(d.lgam + r1)));
    }
    return kk;
}

// pack separate control / case counts (CUDA-core kernels)
template <typename P = uint32_t>
__device__ __forceinline__ void pack16(const DevData& d, const uint32_t (&c0)[16], const uint32_t (&c1)[16],
                                       P (&c16)[16]) {
#pragma unroll
    for (int k = 0; k < 16; ++k) c16[k] = (P)c0[k] | ((P)c1[k] << d.pk_shift);
}

// ---------------------------------------------------------------------------------------------
// (4) per-CTA top-k list in shared memory, updated by whole warps under a CTA spin lock.
struct TopKSmem {
    double* k2;          // [cap], sorted ascending by (k2, idx)
    uint64_t* idx;
    int* cnt;
    int* lock;
    double* thr;         // k2 of the last entry when full, +inf otherwise (monotone non-increasing)
    double* stage_k;     // [8][WL_MAX] staging of the per-warp register lists (wl_merge_store)
    uint64_t* stage_i;
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

// (4b) race-free alternative for top_k <= 32 (the tensor-core kernel's default): every warp keeps its own sorted
// list in registers, lane j holding the j-th smallest (K2, index) key of the warp (empty = +inf / ~0); no state
// is shared between warps, so no lock.  At the end of the kernel the warps stage their lists in shared memory,
// meet at a named barrier, and one warp merges them into the CTA's list (wl_merge_store).
constexpr int WL_MAX = 32;
#ifndef EPI4_WARP_LISTS
#define EPI4_WARP_LISTS 0   // 1: per-warp register lists for top_k <= 32 (race-free; measured 1-2 % slower, profiles/r02l_topk.log)
#endif
__host__ __device__ constexpr bool use_warp_lists(int topk) { return EPI4_WARP_LISTS && topk <= WL_MAX; }
struct WarpList {
    double k;
    uint64_t i;
};
__device__ __forceinline__ void wl_init(WarpList& L) {
    L.k = __longlong_as_double(0x7ff0000000000000LL);
    L.i = ~0ull;
}
// the key of entry cap - 1 (+inf while the list has fewer than cap entries); uniform across the warp
__device__ __forceinline__ double wl_thr(const WarpList& L, int cap) { return __shfl_sync(0xffffffffu, L.k, cap - 1); }
// insert one key (all 32 lanes, uniform kk / ii); entries past cap are kept sorted but never read
__device__ __forceinline__ void wl_insert(WarpList& L, int cap, double kk, uint64_t ii) {
    const int lane = threadIdx.x & 31;
    const int pos = __popc(__ballot_sync(0xffffffffu, key_less(L.k, L.i, kk, ii)));
    if (pos >= cap) return;
    const double uk = __shfl_up_sync(0xffffffffu, L.k, 1);
    const uint64_t ui = __shfl_up_sync(0xffffffffu, L.i, 1);
    if (lane > pos) { L.k = uk; L.i = ui; }
    else if (lane == pos) { L.k = kk; L.i = ii; }
}
// offer one key per lane (has = false lanes offer nothing); thr is updated to the list's new threshold
__device__ __forceinline__ void wl_offer(WarpList& L, int cap, double& thr, bool has, double key, uint64_t idx) {
    unsigned m = __ballot_sync(0xffffffffu, has && key <= thr);
    if (!m) return;
    while (m) {
        const int src = __ffs(m) - 1;
        m &= m - 1;
        wl_insert(L, cap, __shfl_sync(0xffffffffu, key, src), __shfl_sync(0xffffffffu, idx, src));
    }
    thr = wl_thr(L, cap);
}
// the CTA's list of a previous launch (global slot `slot`) into warp list L (call with one warp)
__device__ __forceinline__ void wl_load(WarpList& L, const SearchParams& sp, int slot) {
    const int lane = threadIdx.x & 31, cnt = sp.list_cnt[slot];
    wl_init(L);
    if (lane < cnt) {
        L.k = sp.list_k2[(int64_t)slot * sp.topk + lane];
        L.i = sp.list_idx[(int64_t)slot * sp.topk + lane];
    }
}
// nw warps (ids ew = 0..nw-1, named barrier `bar` over their 32 nw threads) fold their lists into the CTA's global
// slot: staging area stage[nw][32] in shared memory, then warp 0 merges (every staged key through wl_insert)
__device__ __forceinline__ void wl_merge_store(const WarpList& L, int cap, int ew, int nw, int bar, double* stage_k,
                                               uint64_t* stage_i, const SearchParams& sp, int slot) {
    const int lane = threadIdx.x & 31;
    stage_k[ew * WL_MAX + lane] = L.k;
    stage_i[ew * WL_MAX + lane] = L.i;
    asm volatile("bar.sync %0, %1;" ::"r"(bar), "r"(32 * nw) : "memory");
    if (ew != 0) return;
    WarpList R;
    wl_init(R);
    for (int w = 0; w < nw; ++w)
        for (int j = 0; j < cap; ++j) {
            const double kk = stage_k[w * WL_MAX + j];
            if (!(kk < __longlong_as_double(0x7ff0000000000000LL))) break;   // the rest of this list is empty
            wl_insert(R, cap, kk, stage_i[w * WL_MAX + j]);
        }
    const bool full = lane < cap && R.k < __longlong_as_double(0x7ff0000000000000LL);
    if (full) {
        sp.list_k2[(int64_t)slot * sp.topk + lane] = R.k;
        sp.list_idx[(int64_t)slot * sp.topk + lane] = R.i;
    }
    const int cnt = __popc(__ballot_sync(0xffffffffu, full));
    if (lane == 0) sp.list_cnt[slot] = cnt;
}

// carve the top-k state from dynamic shared memory (8-byte aligned base)
__device__ __forceinline__ TopKSmem topk_carve(unsigned char* base, int cap) {
    TopKSmem tk;
    tk.k2 = reinterpret_cast<double*>(base);
    tk.idx = reinterpret_cast<uint64_t*>(base + sizeof(double) * cap);
    tk.thr = reinterpret_cast<double*>(base + 16 * cap);
    tk.cnt = reinterpret_cast<int*>(base + 16 * cap + 8);
    tk.lock = reinterpret_cast<int*>(base + 16 * cap + 12);
    tk.stage_k = reinterpret_cast<double*>(base + 16 * cap + 16);
    tk.stage_i = reinterpret_cast<uint64_t*>(base + 16 * cap + 16 + 8 * 32 * sizeof(double));
    tk.cap = cap;
    return tk;
}
__host__ __device__ constexpr size_t topk_smem_bytes(int cap) { return 16 * (size_t)cap + 16 + 8 * 32 * 16; }

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
