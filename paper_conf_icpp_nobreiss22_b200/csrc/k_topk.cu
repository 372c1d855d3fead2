// k_topk.cu — final reduction of the per-CTA top-k lists (the findGloballyBestSol step,
// per-thread -> shared memory -> global), and the epi4_tables verification
// kernel (16 cells by AND+POPC, 65 by the epilogue's lower-order recovery).
#include "epilogue.cuh"

namespace epi4 {

__device__ __forceinline__ bool kl(double ka, uint64_t ia, double kb, uint64_t ib) {
    return ka < kb || (ka == kb && ia < ib);
}

// one CTA: running best list of `cap` keys in smem; each per-CTA list is merged by a bitonic sort of
// the 2*cap (padded to a power of two) candidates.  Lists that cannot improve the best are skipped.
__global__ void __launch_bounds__(1024) k_merge(const double* __restrict__ lk2, const uint64_t* __restrict__ lidx,
                                               const int32_t* __restrict__ lcnt, int32_t nlists, int32_t cap,
                                               double* out_k2, uint64_t* out_idx, int32_t* out_n) {
    extern __shared__ __align__(16) unsigned char smem[];
    int S = 1;
    while (S < 2 * cap) S <<= 1;
    double* k = reinterpret_cast<double*>(smem);
    uint64_t* ix = reinterpret_cast<uint64_t*>(smem + sizeof(double) * S);
    __shared__ int s_have, s_skip;
    const int tid = threadIdx.x;
    const double INF = __longlong_as_double(0x7ff0000000000000LL);
    for (int e = tid; e < S; e += blockDim.x) { k[e] = INF; ix[e] = ~0ull; }
    if (tid == 0) s_have = 0;
    __syncthreads();
    for (int l = 0; l < nlists; ++l) {
        const int cnt = lcnt[l];
        if (tid == 0) {
            // skip if the list's best key is not better than our worst (when full)
            s_skip = (cnt == 0) || (s_have == cap && !kl(lk2[(int64_t)l * cap], lidx[(int64_t)l * cap], k[cap - 1], ix[cap - 1]));
        }
        __syncthreads();
        if (s_skip) { __syncthreads(); continue; }
        for (int e = tid; e < S - cap; e += blockDim.x) {
            if (e < cnt) { k[cap + e] = lk2[(int64_t)l * cap + e]; ix[cap + e] = lidx[(int64_t)l * cap + e]; }
            else { k[cap + e] = INF; ix[cap + e] = ~0ull; }
        }
        __syncthreads();
        for (int size = 2; size <= S; size <<= 1) {
            for (int stride = size >> 1; stride > 0; stride >>= 1) {
                for (int e = tid; e < S; e += blockDim.x) {
                    const int p = e ^ stride;
                    if (p > e) {
                        const bool up = (e & size) == 0;
                        const bool sw = up ? kl(k[p], ix[p], k[e], ix[e]) : kl(k[e], ix[e], k[p], ix[p]);
                        if (sw) {
                            const double tk = k[e]; k[e] = k[p]; k[p] = tk;
                            const uint64_t ti = ix[e]; ix[e] = ix[p]; ix[p] = ti;
                        }
                    }
                }
                __syncthreads();
            }
        }
        if (tid == 0) s_have = min(cap, s_have + cnt);
        __syncthreads();
    }
    for (int e = tid; e < cap; e += blockDim.x) { out_k2[e] = k[e]; out_idx[e] = ix[e]; }
    if (tid == 0) *out_n = s_have;
}

cudaError_t launch_merge(const SearchParams& sp, int32_t nlists, double* out_k2, uint64_t* out_idx,
                         int32_t* out_n, cudaStream_t s, int64_t* launches) {
    int S = 1;
    while (S < 2 * sp.topk) S <<= 1;
    const size_t smem = 16 * (size_t)S;
    cudaError_t e = cudaFuncSetAttribute(k_merge, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    k_merge<<<1, 1024, smem, s>>>(sp.list_k2, sp.list_idx, sp.list_cnt, nlists, sp.topk, out_k2, out_idx, out_n);
    if (launches) ++*launches;
    return cudaGetLastError();
}

// ---- tables of arbitrary quads ---------------------------------------------------------------------
__global__ void __launch_bounds__(128) k_tables(DevData d, const uint64_t* __restrict__ quads, int64_t nq,
                                                uint32_t* __restrict__ out, unsigned int* status) {
    const int64_t q = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (q >= nq) return;
    const uint64_t pk = quads[q];
    int v[4] = {(int)((pk >> 48) & 0xFFFF), (int)((pk >> 32) & 0xFFFF), (int)((pk >> 16) & 0xFFFF),
                (int)(pk & 0xFFFF)};
    int pos[4] = {0, 1, 2, 3};   // pos[t] = slot of given SNP t after sorting
    // sort (w<x<y<z) keeping the permutation
    int s[4] = {v[0], v[1], v[2], v[3]}, o[4] = {0, 1, 2, 3};
    for (int a = 0; a < 4; ++a)
        for (int b = 0; b < 3 - a; ++b)
            if (s[b] > s[b + 1]) {
                int t = s[b]; s[b] = s[b + 1]; s[b + 1] = t;
                t = o[b]; o[b] = o[b + 1]; o[b + 1] = t;
            }
    for (int a = 0; a < 4; ++a) pos[o[a]] = a;
    uint32_t* dst = out + q * 162;
    if (s[0] == s[1] || s[1] == s[2] || s[2] == s[3] || s[3] >= d.n) {
        atomicOr(status, 32u);
        for (int c = 0; c < 162; ++c) dst[c] = 0;
        return;
    }
    uint32_t c4[2][16];
    for (int p = 0; p < 2; ++p) {
        for (int c = 0; c < 16; ++c) c4[p][c] = 0;
        for (int kc = 0; kc < d.nchunks[p]; ++kc) {
            uint32_t pl[4][2][4];
            for (int t = 0; t < 4; ++t)
                for (int g = 0; g < 2; ++g) {
                    const uint4 u = __ldg(reinterpret_cast<const uint4*>(d.planes[p] + plane_off(kc, d.npad, s[t], g, 0)));
                    pl[t][g][0] = u.x; pl[t][g][1] = u.y; pl[t][g][2] = u.z; pl[t][g][3] = u.w;
                }
            for (int wd = 0; wd < 4; ++wd)
                for (int c = 0; c < 16; ++c)
                    c4[p][c] += __popc(pl[0][(c >> 3) & 1][wd] & pl[1][(c >> 2) & 1][wd] & pl[2][(c >> 1) & 1][wd] &
                                       pl[3][c & 1][wd]);
        }
    }
    uint32_t g[162];
    {
        uint32_t c0[16], c1[16];
        for (int c = 0; c < 16; ++c) { c0[c] = c4[0][c]; c1[c] = c4[1][c]; }
        uint32_t tmp[162];
        if (d.wide) {
            uint64_t c16[16];
            pack16<uint64_t>(d, c0, c1, c16);
            (void)score_quad<uint64_t>(d, s[0], s[1], s[2], s[3], c16, tmp);
        } else {
            uint32_t c16[16];
            pack16<uint32_t>(d, c0, c1, c16);
            (void)score_quad<uint32_t>(d, s[0], s[1], s[2], s[3], c16, tmp);
        }
        for (int c = 0; c < 162; ++c) g[c] = tmp[c];
    }
    // sorted cell (digits for s[0..3]) -> cell in the given order: digit of given SNP t = digit[pos[t]]
    const int pw[4] = {27, 9, 3, 1};
    for (int c = 0; c < 81; ++c) {
        const int dg[4] = {c / 27, (c / 9) % 3, (c / 3) % 3, c % 3};
        int co = 0;
        for (int t = 0; t < 4; ++t) co += pw[t] * dg[pos[t]];
        dst[co] = g[c];
        dst[81 + co] = g[81 + c];
    }
}

cudaError_t launch_tables(const DevData& d, const uint64_t* quads, int64_t n, uint32_t* out, unsigned int* status,
                          cudaStream_t s, int64_t* launches) {
    if (n <= 0) return cudaSuccess;
    k_tables<<<(unsigned)((n + 127) / 128), 128, 0, s>>>(d, quads, n, out, status);
    if (launches) ++*launches;
    return cudaGetLastError();
}

}  // namespace epi4
