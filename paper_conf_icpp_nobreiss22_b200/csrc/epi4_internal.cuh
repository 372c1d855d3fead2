// epi4_internal.cuh — internal declarations shared by the libepi4 translation units.
//
// Device data layout in HBM:
//   planes[p]  : uint32, chunked K-major: [chunk kc][snp (padded, see npad)][g = 0 AA, 1 Aa][4 words]
//                one chunk = 128 samples of phenotype p; pad bits are 0 (PAPER.md:L66-68 encoding,
//                re-tiled so that consecutive SNPs are contiguous per chunk).
//   expl[p]    : the same planes as E2M1 {0, 1.0} nibbles (256 samples = 128 bytes per row and fp4 chunk),
//                blocked [chunk pair][128-row block][chunk & 1][row r = 2 snp + g][128 bytes] (expl_off) with the
//                UMMA 128-byte swizzle applied in HBM (16-byte piece c of row r stored at piece c ^ (r & 7)), so
//                one linear 32 KiB bulk copy lands two chunks of a 128-row A tile in the canonical K-major SW128
//                shared-memory layout; the chunk count is padded to even with zero chunks.
//   lower-order tables, every entry a PACKED pair c0 | c1 << pk_shift (controls low, cases high; epilogue.cuh):
//   T1[snp][2]          popc(P_a(snp))                              (PAPER.md:L85 indivPop)
//   T2[rank2][4]        popc(P_a(i) & P_b(j)), i<j, cell 2a+b       (PAPER.md:L86 pairwPop)
//   T3[rank3][8]        popc(P_a(i) & P_b(j) & P_c(k)), i<j<k, cell 4a+2b+c
//   lgam[n] = lgamma(n+1) for n in [0, M+1], double, built on the host
// colex ranks: rank2(i,j) = C(j,2)+i, rank3(i,j,k) = C(k,3)+C(j,2)+i, rank4 = C(l,4)+C(k,3)+C(j,2)+i.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/epi4.h"

#define EPI4_B 32             // SNP block size accepted in epi4_opts (32-SNP blocks)
#define EPI4_WR 64            // w-range of one CTA / rows of its A operand: 64 SNPs x {AA, Aa}
#define EPI4_WP 128           // w-range of a work unit (a CTA pair: two 64-SNP halves)
#define EPI4_YR 16            // y-range of a CUDA-core (LOP3) tile: 16 consecutive SNPs after x
// tensor-core tile geometries (k_quad_tc.cuh Geom128 / Geom224): y-range of a tile (8 columns per y) and fp4
// chunks per pipeline step (overridable for diagnostics builds only)
#ifndef EPI4_YR_N128
#define EPI4_YR_N128 16
#endif
#ifndef EPI4_CH_N128
#define EPI4_CH_N128 2
#endif
#ifndef EPI4_YR_N224
#define EPI4_YR_N224 28
#endif
#ifndef EPI4_CH_N224
#define EPI4_CH_N224 1
#endif
#define EPI4_YR_MAX 32        // SNP rows a tile may read past its y0 (planes are zero-padded that far)
#define EPI4_CHUNK_WORDS 4    // 128 samples per chunk
#define EPI4_CHUNK_SAMPLES 128

// device-side status bits (atomicOr'ed by kernels, read by the host after a phase)
#define EPI4_ST_BAD_GENO   1u
#define EPI4_ST_BAD_PHEN   2u
#define EPI4_ST_PAD_BITS   4u
#define EPI4_ST_AA_AND_Aa  8u
#define EPI4_ST_TOPK_OVF  16u

namespace epi4 {

// fp4 chunks (256 samples) per tensor-core pipeline step of a geometry, and the steps of a phenotype
__host__ __device__ __forceinline__ int32_t tc_chunks(int32_t yr) { return yr == EPI4_YR_N224 ? EPI4_CH_N224 : EPI4_CH_N128; }
__host__ __device__ __forceinline__ int32_t tc_steps(int32_t nchunks4, int32_t yr) {
    return (nchunks4 + tc_chunks(yr) - 1) / tc_chunks(yr);
}

__host__ __device__ __forceinline__ int64_t c2(int64_t n) { return n * (n - 1) / 2; }
__host__ __device__ __forceinline__ int64_t c3(int64_t n) { return n * (n - 1) * (n - 2) / 6; }
__host__ __device__ __forceinline__ int64_t c4(int64_t n) { return n * (n - 1) * (n - 2) * (n - 3) / 24; }
__host__ __device__ __forceinline__ int64_t rank2(int i, int j) { return c2(j) + i; }
__host__ __device__ __forceinline__ int64_t rank3(int i, int j, int k) { return c3(k) + c2(j) + i; }
__host__ __device__ __forceinline__ int64_t rank4(int i, int j, int k, int l) {
    return c4(l) + c3(k) + c2(j) + i;
}
__host__ __device__ __forceinline__ uint64_t pack_quad(int i, int j, int k, int l) {
    return ((uint64_t)(uint16_t)i << 48) | ((uint64_t)(uint16_t)j << 32) | ((uint64_t)(uint16_t)k << 16) |
           (uint64_t)(uint16_t)l;
}

// Everything a kernel needs to read the dataset and the lower-order tables.
struct DevData {
    const uint32_t* planes[2];   // chunked planes per phenotype
    int32_t nchunks[2];          // 128-sample chunks per phenotype
    int32_t nchunks4[2];         // 256-sample fp4 chunks per phenotype (rows of expl)
    int32_t nrb;                 // 128-row blocks of expl per chunk (= npad / 64)
    int32_t pk_shift;            // (control, case) counts packed as c0 | c1 << pk_shift everywhere (bits(n0))
    int32_t wide;                // 1: packed words are 64-bit (pk_shift = 32) because bits(n0) + bits(n1) > 32
    int32_t n;                   // SNPs
    int32_t npad;                // SNP rows per chunk: ceil((n + 16) / 64) * 64 (zero rows beyond n)
    uint32_t np[2];              // n0, n1
    uint32_t npk;                // n0 | n1 << pk_shift
    const uint32_t* T1;
    const uint32_t* T2;
    const uint32_t* T3;          // resident: all triples, colex rank; windowed: the slab FIRST(R) (below)
    // Windowed T3 (t3_win = 1): every triple a quad w < x < y < z reads starts with w (wxy, wxz,
    // wyz) or with x (xyz).  T3 holds FIRST(R) = {(w, j, k): w in the 128-SNP w-range R = [t3_w0, t3_w0 + 128)} at
    // entry (w - t3_w0) * C(n,2) + rank2(j, k); T3x holds FIRST(X) for the x-range X = [t3_x0, t3_x0 + 128) the
    // same way (T3x == T3 when X == R).
    const uint32_t* T3x;
    int32_t t3_win, t3_w0, t3_x0;
    const double* lgam;          // M + 2 entries
    const double* xlx;           // X(k) = k ln k, M + 2 entries (EPI4_OBJ_MI)
    double mi_const;             // X(M) - X(n0) - X(n1)
    int32_t objective;           // EPI4_OBJ_*
    const uint8_t* expl[2];      // E2M1 {0, 1.0} nibble planes (tcgen05 operands; layout: expl_off below)
    double flt_off;              // fp32 K2 filter: exact-score a quad iff ln2 A + flt_off <= threshold (epilogue.cuh)
    float chi_a, chi_b;          // fp32 chi-square filter: M / n0, M / n1 (epilogue.cuh, cell_chi_acc)
    double chi_M;                // M
    double mi_E;                 // fp32 MI filter: rounding bound (bits) on V = sum_c [X2(r0) + X2(r1) - X2(r_c)]
};

// byte offset of (fp4 chunk C, row r = 2 snp + g) in expl: blocked [chunk pair][128-row block][C & 1][row][128 B]
// so that the 2 chunks x 128 rows of one A tile are one contiguous 32 KiB bulk copy (a 16 KiB copy is processed
// at ~42 B/clk/SM, a 32 KiB copy at ~75: tools/probe_tma3.cu)
__host__ __device__ __forceinline__ int64_t expl_off(int64_t C, int64_t r, int32_t nrb) {
    return ((((C >> 1) * nrb + (r >> 7)) * 2 + (C & 1)) * 128 + (r & 127)) * 128;
}

// offset (in uint32 words) of (chunk kc, snp, g, word w) in a chunked plane array
__host__ __device__ __forceinline__ int64_t plane_off(int64_t kc, int32_t npad, int32_t snp, int g, int w) {
    return ((kc * npad + snp) * 2 + g) * EPI4_CHUNK_WORDS + w;
}

// A work unit (wp, x): the quads (w, x, y, z) with w in the 128-SNP range [128 wp, 128 wp + 128), w < x,
// second SNP x, and any x < y < z < n.  Its tiles are (y0, z): y in [y0, y0 + yr) with y0 = x + 1 + yr k,
// and z in (y0, n); a tile holds 128 x yr (w, y) combinations (yr = EPI4_YR_N128 / EPI4_YR_N224 tensor core, EPI4_YR CUDA core), split into
// the two 64-SNP halves of the w-range (the two CTAs of a tensor-core cluster, or two tiles of the CUDA-core
// kernel).
struct Unit {
    int32_t wr, x;   // wr = 128-SNP w-range index
};

__host__ __device__ __forceinline__ int64_t unit_tiles(int32_t n, int32_t x, int32_t yr = EPI4_YR) {
    int64_t t = 0;
    for (int32_t y0 = x + 1; y0 <= n - 2; y0 += yr) t += n - y0 - 1;
    return t;
}

// decode tile t of unit (x) -> (y0, z), y-range yr
__device__ __forceinline__ void unit_tile_decode(int32_t n, int32_t x, int64_t t, int32_t& y0, int32_t& z,
                                                 int32_t yr = EPI4_YR) {
    for (y0 = x + 1; y0 <= n - 2; y0 += yr) {
        const int64_t cnt = n - y0 - 1;
        if (t < cnt) {
            z = y0 + 1 + (int32_t)t;
            return;
        }
        t -= cnt;
    }
    z = n;  // unreachable for valid t
}

// find the unit of a flat tile index by binary search on the inclusive prefix of tile counts
__device__ __forceinline__ int64_t find_unit(const int64_t* prefix, int64_t nunits, int64_t tile) {
    int64_t lo = 0, hi = nunits - 1;
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if (prefix[mid] > tile) hi = mid; else lo = mid + 1;
    }
    return lo;
}

// Per-search launch parameters common to the contraction kernels.
struct SearchParams {
    DevData d;
    int32_t yr;                // tensor-core pipe: y-range of a tile = the geometry (EPI4_YR_N128 / EPI4_YR_N224)
    const Unit* units;
    const int64_t* prefix;     // inclusive prefix of tiles per unit
    const uint64_t* tile_info; // (tensor-core pipe) decoded tiles: wp | x << 16 | y0 << 32 | z << 48 (k_tile_table)
    uint32_t* t3_out;          // non-NULL: 3-way-table mode of k_quad_tc (z = the all-ones SNP n, writes T3)
    int32_t t3_slab_w0;        // 3-way-table mode: < 0 resident colex layout, else the slab FIRST([w0, w0+128))
    int32_t search3;           // third-order search mode (z = the all-ones SNP n, epi4_search3)
    int64_t nunits;
    int64_t ntiles;
    unsigned long long* tile_counter;   // dynamic scheduler
    int32_t topk;              // list capacity used (<= EPI4_MAX_TOPK)
    double* list_k2;           // per-CTA lists [grid][topk]
    uint64_t* list_idx;
    int32_t* list_cnt;         // [grid]
    uint32_t* dump;            // optional 162 counts per quad indexed by rank4 (NULL = off)
    unsigned int* status;
    unsigned long long* quads_done;   // useful quads evaluated (atomicAdd once per CTA)
    unsigned long long* prof;  // [16] diagnostics: [0] exact K2 evaluations, [1..] per-role cycle counters
    int32_t use_filter;        // fp32 filter before the exact double score: 1 = Stirling K2 filter, 2 = chi-square
                               // upper bound (EPI4_OBJ_CHI2), 3 = MI upper bound (EPI4_OBJ_MI) (epilogue.cuh);
                               // 0 = every quad scored exactly

    int32_t debug;             // diagnostics only (results invalid): 1 skip producers, 2 skip scoring, 4 skip MMA,
                               // 128 no A copies (16: exact K2 for every quad, 64: trace)
    // verification sample (epi4_set_sample): quads with (mix64(index ^ samp_seed) & samp_mask) == 0 are recorded
    // with their exact key and 162 counts (the search kernel's own contraction + recovery); samp_cap = 0: off
    int64_t samp_cap;
    uint64_t samp_seed, samp_mask;
    unsigned long long* samp_n;
    uint64_t* samp_idx;
    double* samp_key;
    uint32_t* samp_counts;
};

// splitmix64 finalizer: the verification-sample hash (epi4.h epi4_set_sample)
__host__ __device__ __forceinline__ uint64_t mix64(uint64_t x) {
    x ^= x >> 30;
    x *= 0xBF58476D1CE4E5B9ull;
    x ^= x >> 27;
    x *= 0x94D049BB133111EBull;
    x ^= x >> 31;
    return x;
}

}  // namespace epi4

// kernel launchers (each .cu provides its own)
namespace epi4 {
cudaError_t launch_split_phen(const uint8_t* phen, int64_t m, int32_t* idx0, int32_t* idx1, int32_t* counts,
                              unsigned int* status, cudaStream_t s, int64_t* launches);
cudaError_t launch_pack(const uint8_t* geno, int32_t n, int64_t m, const int32_t* idx, int64_t np, int32_t npad,
                        int32_t nchunks, uint32_t* planes, unsigned int* status, cudaStream_t s, int64_t* launches);
cudaError_t launch_retile(const uint32_t* rows, int32_t n, int64_t np, int32_t npad, int32_t nchunks,
                          uint32_t* planes, unsigned int* status, cudaStream_t s, int64_t* launches);
cudaError_t launch_untile(const uint32_t* planes, int32_t n, int64_t np, int32_t npad, int32_t nchunks,
                          uint32_t* rows, cudaStream_t s, int64_t* launches);
cudaError_t launch_expand(const uint32_t* planes, int32_t npad, int32_t nchunks, uint8_t* expl, cudaStream_t s,
                          int64_t* launches);
cudaError_t launch_ones_plane(uint32_t* planes, int32_t n, int32_t npad, int32_t nchunks, int64_t np, cudaStream_t s,
                              int64_t* launches);
cudaError_t launch_pop(const DevData& d, uint32_t* T1, uint32_t* T2, uint32_t* T3, int64_t t3_lo, int64_t t3_hi,
                       cudaStream_t s, int64_t* launches);
cudaError_t launch_quad_lop3(const SearchParams& sp, int32_t grid, cudaStream_t s, int64_t* launches);
cudaError_t launch_quad_tc(const SearchParams& sp, int32_t grid, cudaStream_t s, int64_t* launches);
cudaError_t launch_tile_table(const SearchParams& sp, int64_t t0, int64_t t1, uint64_t* out, cudaStream_t s,
                              int64_t* launches);
int32_t quad_split(int32_t pipe);   // tiles per unit tile (CUDA-core kernel: the two 64-SNP halves)
cudaError_t launch_merge(const SearchParams& sp, int32_t nlists, double* out_k2, uint64_t* out_idx,
                         int32_t* out_n, cudaStream_t s, int64_t* launches);
cudaError_t launch_tables(const DevData& d, const uint64_t* quads, int64_t n, uint32_t* out, unsigned int* status,
                          cudaStream_t s, int64_t* launches);
}  // namespace epi4
