// epi4_internal.cuh — internal declarations shared by the libepi4 translation units.
//
// Device data layout in HBM:
//   planes[p]  : uint32, chunked K-major: [chunk kc][snp (padded to 32)][g = 0 AA, 1 Aa][4 words]
//                one chunk = 128 samples of phenotype p; pad bits are 0 (PAPER.md:L66-68 encoding,
//                re-tiled so that the 32 SNPs of a block are 1 KiB contiguous per chunk).
//   T1[snp][p][2]          popc(P_a(snp))                              (PAPER.md:L85 indivPop)
//   T2[rank2][p][4]        popc(P_a(i) & P_b(j)), i<j, cell 2a+b       (PAPER.md:L86 pairwPop)
//   T3[rank3][p][8]        popc(P_a(i) & P_b(j) & P_c(k)), i<j<k, cell 4a+2b+c
//   lgam[n] = lgamma(n+1) for n in [0, M+1], double, built on the host
// colex ranks: rank2(i,j) = C(j,2)+i, rank3(i,j,k) = C(k,3)+C(j,2)+i, rank4 = C(l,4)+C(k,3)+C(j,2)+i.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/epi4.h"

#define EPI4_B 32             // SNP block size (32-SNP blocks)
#define EPI4_CHUNK_WORDS 4    // 128 samples per chunk
#define EPI4_CHUNK_SAMPLES 128

// device-side status bits (atomicOr'ed by kernels, read by the host after a phase)
#define EPI4_ST_BAD_GENO   1u
#define EPI4_ST_BAD_PHEN   2u
#define EPI4_ST_PAD_BITS   4u
#define EPI4_ST_AA_AND_Aa  8u
#define EPI4_ST_TOPK_OVF  16u

namespace epi4 {

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
    int32_t nchunks[2];          // chunks per phenotype
    int32_t n;                   // SNPs
    int32_t npad;                // SNPs padded to a multiple of 32 (row count of a chunk / 2)
    uint32_t np[2];              // n0, n1
    const uint32_t* T1;
    const uint32_t* T2;
    const uint32_t* T3;
    const double* lgam;          // M + 2 entries
    const uint8_t* expl[2];      // {0,1}-byte expanded planes [chunk][snp][g][128 samples] (tcgen05 operands)
};

// offset (in uint32 words) of (chunk kc, snp, g, word w) in a chunked plane array
__host__ __device__ __forceinline__ int64_t plane_off(int64_t kc, int32_t npad, int32_t snp, int g, int w) {
    return ((kc * npad + snp) * 2 + g) * EPI4_CHUNK_WORDS + w;
}

// A work unit (wb, x): quads with w in block wb (w < x), second SNP x, any y < z after x.
struct Unit {
    int32_t wb, x;
};

// number of tiles of unit (wb,x) when a tile covers ZT consecutive z values:
// tiles iterate y-blocks yb >= (x+1)/32 and z in [max(x+2, 32*yb+1), n)
__host__ __device__ __forceinline__ int64_t unit_tiles(int32_t n, int32_t x, int32_t zt) {
    int64_t t = 0;
    int32_t nb = (n + EPI4_B - 1) / EPI4_B;
    for (int32_t yb = (x + 1) / EPI4_B; yb < nb; ++yb) {
        int32_t zlo = max(x + 2, yb * EPI4_B + 1);
        if (zlo < n) t += (n - zlo + zt - 1) / zt;
    }
    return t;
}

// decode tile t of unit (x) -> (yb, z0)
__device__ __forceinline__ void unit_tile_decode(int32_t n, int32_t x, int32_t zt, int64_t t, int32_t& yb,
                                                 int32_t& z0) {
    int32_t nb = (n + EPI4_B - 1) / EPI4_B;
    for (yb = (x + 1) / EPI4_B; yb < nb; ++yb) {
        int32_t zlo = max(x + 2, yb * EPI4_B + 1);
        int64_t cnt = (zlo < n) ? (n - zlo + zt - 1) / zt : 0;
        if (t < cnt) {
            z0 = zlo + (int32_t)t * zt;
            return;
        }
        t -= cnt;
    }
    z0 = n;  // unreachable for valid t
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
    const Unit* units;
    const int64_t* prefix;     // inclusive prefix of tiles per unit
    int64_t nunits;
    int64_t ntiles;
    int32_t zt;                // z values per tile
    unsigned long long* tile_counter;   // dynamic scheduler
    int32_t topk;              // list capacity used (<= EPI4_MAX_TOPK)
    double* list_k2;           // per-CTA lists [grid][topk]
    uint64_t* list_idx;
    int32_t* list_cnt;         // [grid]
    uint32_t* dump;            // optional 162 counts per quad indexed by rank4 (NULL = off)
    unsigned int* status;
    unsigned long long* quads_done;   // useful quads evaluated (atomicAdd once per CTA)
};

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
cudaError_t launch_pop(const DevData& d, uint32_t* T1, uint32_t* T2, uint32_t* T3, cudaStream_t s,
                       int64_t* launches);
cudaError_t launch_quad_lop3(const SearchParams& sp, int32_t grid, cudaStream_t s, int64_t* launches);
cudaError_t launch_quad_i8tc(const SearchParams& sp, int32_t grid, cudaStream_t s, int64_t* launches);
int32_t quad_zt(int32_t pipe);
cudaError_t launch_merge(const SearchParams& sp, int32_t nlists, double* out_k2, uint64_t* out_idx,
                         int32_t* out_n, cudaStream_t s, int64_t* launches);
cudaError_t launch_tables(const DevData& d, const uint64_t* quads, int64_t n, uint32_t* out, unsigned int* status,
                          cudaStream_t s, int64_t* launches);
}  // namespace epi4
