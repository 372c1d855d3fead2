// k_prep.cu — data preparation kernels (steps a1 and a2 of SURVEY.md §8(a)):
//   split_phen : list the sample indices of each phenotype ("genotypic data is split
//                into cases and controls ... stored in a contiguous memory region")
//   pack       : byte genotypes -> 2 bit planes per SNP per phenotype, AA and Aa; aa not stored
//                (§3.1), written in the chunked device layout (epi4_internal.cuh)
//   retile     : row-major host planes (the ABI format) -> chunked layout, validating pad bits and
//                AA & Aa == 0;  untile: the reverse (epi4_get_bits)
//   pop        : T1 (indivPop), T2 (pairwPop, L86, L112-114) and the 3-way tables T3
//                (8 non-aa cells per triple, the tensorOp_3way proto-tables of) by AND+POPC.
#include "epi4_internal.cuh"

namespace epi4 {

// ---- split by phenotype ------------------------------------------------------------------------
__global__ void __launch_bounds__(1024) k_split_phen(const uint8_t* __restrict__ phen, int64_t m,
                                                     int32_t* __restrict__ idx0, int32_t* __restrict__ idx1,
                                                     int32_t* counts, unsigned int* status) {
    __shared__ int s_w1[32];
    __shared__ int s_base1, s_base0;
    const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
    if (tid == 0) { s_base0 = 0; s_base1 = 0; }
    __syncthreads();
    for (int64_t off = 0; off < m; off += 1024) {
        const int64_t s = off + tid;
        int v = 0, valid = s < m;
        if (valid) {
            v = phen[s];
            if (v > 1) { atomicOr(status, EPI4_ST_BAD_PHEN); v = 1; }
        }
        const unsigned b1 = __ballot_sync(0xffffffffu, valid && v == 1);
        if (lane == 0) s_w1[wid] = __popc(b1);
        __syncthreads();
        int pre1 = 0, tot1 = 0;
        for (int k = 0; k < 32; ++k) {
            if (k < wid) pre1 += s_w1[k];
            tot1 += s_w1[k];
        }
        // the valid threads of this round are a prefix of the block, so tid = rank among valid
        const int r1 = pre1 + __popc(b1 & ((1u << lane) - 1));
        const int r0 = tid - r1;
        const int base0 = s_base0, base1 = s_base1;
        if (valid) {
            if (v == 1) idx1[base1 + r1] = (int32_t)s; else idx0[base0 + r0] = (int32_t)s;
        }
        __syncthreads();
        if (tid == 0) {
            const int nvalid = (m - off) < 1024 ? (int)(m - off) : 1024;
            s_base1 = base1 + tot1;
            s_base0 = base0 + (nvalid - tot1);
        }
        __syncthreads();
    }
    if (tid == 0) { counts[0] = s_base0; counts[1] = s_base1; }
}

cudaError_t launch_split_phen(const uint8_t* phen, int64_t m, int32_t* idx0, int32_t* idx1, int32_t* counts,
                              unsigned int* status, cudaStream_t s, int64_t* launches) {
    k_split_phen<<<1, 1024, 0, s>>>(phen, m, idx0, idx1, counts, status);
    if (launches) ++*launches;
    return cudaGetLastError();
}

// ---- pack: one thread = one 32-sample word of (snp, chunk, word) -> AA and Aa words ---------------
__global__ void __launch_bounds__(256) k_pack(const uint8_t* __restrict__ geno, int32_t n, int64_t m,
                                              const int32_t* __restrict__ idx, int64_t np, int32_t npad,
                                              int32_t nchunks, uint32_t* __restrict__ planes,
                                              unsigned int* status) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t total = (int64_t)n * nchunks * EPI4_CHUNK_WORDS;
    if (t >= total) return;
    const int w = (int)(t % EPI4_CHUNK_WORDS);
    const int32_t snp = (int32_t)((t / EPI4_CHUNK_WORDS) % n);
    const int64_t kc = t / ((int64_t)EPI4_CHUNK_WORDS * n);
    const uint8_t* row = geno + (int64_t)snp * m;
    const int64_t s0 = kc * EPI4_CHUNK_SAMPLES + (int64_t)w * 32;
    uint32_t aa = 0, het = 0;
    bool bad = false;
#pragma unroll 8
    for (int b = 0; b < 32; ++b) {
        const int64_t k = s0 + b;
        if (k < np) {
            const uint8_t g = row[idx[k]];
            bad |= g > 2;
            aa |= (uint32_t)(g == 0) << b;
            het |= (uint32_t)(g == 1) << b;
        }
    }
    if (bad) atomicOr(status, EPI4_ST_BAD_GENO);
    planes[plane_off(kc, npad, snp, 0, w)] = aa;
    planes[plane_off(kc, npad, snp, 1, w)] = het;
}

cudaError_t launch_pack(const uint8_t* geno, int32_t n, int64_t m, const int32_t* idx, int64_t np, int32_t npad,
                        int32_t nchunks, uint32_t* planes, unsigned int* status, cudaStream_t s, int64_t* launches) {
    const int64_t total = (int64_t)n * nchunks * EPI4_CHUNK_WORDS;
    const int64_t blocks = (total + 255) / 256;
    if (blocks > 0) {
        k_pack<<<(unsigned)blocks, 256, 0, s>>>(geno, n, m, idx, np, npad, nchunks, planes, status);
        if (launches) ++*launches;
    }
    return cudaGetLastError();
}

// ---- retile / untile: row-major [2n][wp] <-> chunked ----------------------------------------------
__global__ void __launch_bounds__(256) k_retile(const uint32_t* __restrict__ rows, int32_t n, int64_t np,
                                                int32_t npad, int32_t nchunks, uint32_t* __restrict__ planes,
                                                unsigned int* status) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const int64_t total = (int64_t)n * nchunks * EPI4_CHUNK_WORDS;
    if (t >= total) return;
    const int w = (int)(t % EPI4_CHUNK_WORDS);
    const int32_t snp = (int32_t)((t / EPI4_CHUNK_WORDS) % n);
    const int64_t kc = t / ((int64_t)EPI4_CHUNK_WORDS * n);
    const int64_t wp = (np + 31) / 32;
    const int64_t word = kc * EPI4_CHUNK_WORDS + w;
    uint32_t aa = 0, het = 0;
    if (word < wp) {
        aa = rows[(2 * (int64_t)snp + 0) * wp + word];
        het = rows[(2 * (int64_t)snp + 1) * wp + word];
        if (word == wp - 1 && (np & 31)) {
            const uint32_t pad = ~((1u << (np & 31)) - 1u);
            if ((aa | het) & pad) atomicOr(status, EPI4_ST_PAD_BITS);
        }
        if (aa & het) atomicOr(status, EPI4_ST_AA_AND_Aa);
    }
    planes[plane_off(kc, npad, snp, 0, w)] = aa;
    planes[plane_off(kc, npad, snp, 1, w)] = het;
}

cudaError_t launch_retile(const uint32_t* rows, int32_t n, int64_t np, int32_t npad, int32_t nchunks,
                          uint32_t* planes, unsigned int* status, cudaStream_t s, int64_t* launches) {
    const int64_t total = (int64_t)n * nchunks * EPI4_CHUNK_WORDS;
    const int64_t blocks = (total + 255) / 256;
    if (blocks > 0) {
        k_retile<<<(unsigned)blocks, 256, 0, s>>>(rows, n, np, npad, nchunks, planes, status);
        if (launches) ++*launches;
    }
    return cudaGetLastError();
}

__global__ void __launch_bounds__(256) k_untile(const uint32_t* __restrict__ planes, int32_t n, int64_t np,
                                                int32_t npad, int32_t nchunks, uint32_t* __restrict__ rows) {
    const int64_t wp = (np + 31) / 32;
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= 2 * (int64_t)n * wp) return;
    const int64_t word = t % wp;
    const int64_t r = t / wp;
    const int32_t snp = (int32_t)(r >> 1);
    const int g = (int)(r & 1);
    rows[t] = planes[plane_off(word / EPI4_CHUNK_WORDS, npad, snp, g, (int)(word % EPI4_CHUNK_WORDS))];
}

cudaError_t launch_untile(const uint32_t* planes, int32_t n, int64_t np, int32_t npad, int32_t nchunks,
                          uint32_t* rows, cudaStream_t s, int64_t* launches) {
    (void)nchunks;
    const int64_t total = 2 * (int64_t)n * ((np + 31) / 32);
    const int64_t blocks = (total + 255) / 256;
    if (blocks > 0) {
        k_untile<<<(unsigned)blocks, 256, 0, s>>>(planes, n, np, npad, nchunks, rows);
        if (launches) ++*launches;
    }
    return cudaGetLastError();
}

// ---- E2M1 expansion of the planes (operands of the tensor-core pipe) ------------------------------
// Tensor-core operand planes: E2M1 nibbles (1.0 = 0x2 for a set bit, 0 otherwise), two samples per byte
// (sample 2j in the low nibble of byte j), 256 samples = one 128-byte K-major row per fp4 chunk C (the 128-sample
// plane chunks 2C and 2C+1; a missing odd chunk reads as zeros).  Layout [C][row r = 2 snp + g][128 B] with
// the UMMA 128-byte swizzle applied: 16-byte piece cc of row r stored at piece cc ^ (r & 7).
__global__ void __launch_bounds__(256) k_expand(const uint32_t* __restrict__ planes, int32_t npad, int32_t nchunks,
                                                int64_t total16, uint8_t* __restrict__ expl) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= total16) return;
    const int cc = (int)(t & 7);                 // 16-byte piece (32 samples) of the 256-sample row
    const int64_t rowid = t >> 3;                // (C, r)
    const int64_t rows = (int64_t)npad * 2;
    const int64_t C = rowid / rows, r = rowid - C * rows;
    const int64_t c128 = 2 * C + (cc >> 2);
    const uint32_t word = c128 < nchunks ? planes[(c128 * rows + r) * EPI4_CHUNK_WORDS + (cc & 3)] : 0u;
    uint32_t o[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) {
        uint32_t v = 0;
#pragma unroll
        for (int b = 0; b < 4; ++b) {
            v |= ((word >> (8 * k + 2 * b)) & 1u) << (8 * b + 1);
            v |= ((word >> (8 * k + 2 * b + 1)) & 1u) << (8 * b + 5);
        }
        o[k] = v;
    }
    const int sw = cc ^ (int)(r & 7);
    reinterpret_cast<uint4*>(expl + expl_off(C, r, npad / 64))[sw] = make_uint4(o[0], o[1], o[2], o[3]);
}

cudaError_t launch_expand(const uint32_t* planes, int32_t npad, int32_t nchunks, uint8_t* expl, cudaStream_t s,
                          int64_t* launches) {
    const int64_t nc4 = ((nchunks + 1) / 2 + 1) / 2 * 2;   // fp4 chunks, padded to even (zero chunk)
    const int64_t total16 = nc4 * npad * 2 * 8;
    if (total16 > 0) {
        k_expand<<<(unsigned)((total16 + 255) / 256), 256, 0, s>>>(planes, npad, nchunks, total16, expl);
        if (launches) ++*launches;
    }
    return cudaGetLastError();
}

// The all-ones SNP: padding row n (AA plane = every real sample, Aa = 0), the virtual z of k_quad_tc's 3-way-table
// mode (its columns x_b & y_c & z_AA are then x_b & y_c: T3(w, x, y) on the tensor cores
// "tensorOp_3way").  Row n exists (npad >= n + 16) and lies outside every real quad.
__global__ void k_ones_plane(uint32_t* __restrict__ planes, int32_t n, int32_t npad, int32_t nchunks, int64_t np) {
    const int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;   // (chunk, word)
    if (t >= (int64_t)nchunks * EPI4_CHUNK_WORDS) return;
    const int64_t kc = t / EPI4_CHUNK_WORDS;
    const int w = (int)(t % EPI4_CHUNK_WORDS);
    const int64_t s0 = kc * EPI4_CHUNK_SAMPLES + 32 * w;
    const uint32_t ones = s0 + 32 <= np ? 0xFFFFFFFFu : (s0 >= np ? 0u : ((1u << (np - s0)) - 1u));
    planes[plane_off(kc, npad, n, 0, w)] = ones;
    planes[plane_off(kc, npad, n, 1, w)] = 0u;
}
cudaError_t launch_ones_plane(uint32_t* planes, int32_t n, int32_t npad, int32_t nchunks, int64_t np, cudaStream_t s,
                              int64_t* launches) {
    const int64_t tot = (int64_t)nchunks * EPI4_CHUNK_WORDS;
    if (tot <= 0) return cudaSuccess;
    k_ones_plane<<<(unsigned)((tot + 255) / 256), 256, 0, s>>>(planes, n, npad, nchunks, np);
    if (launches) ++*launches;
    return cudaGetLastError();
}

// ---- lower-order tables ---------------------------------------------------------------------------
// packed (control, case) word of the tables: c0 | c1 << pk_shift, 32 or (wide) 64 bits
template <typename P>
__device__ __forceinline__ P pkw(const DevData& d, uint32_t c0, uint32_t c1) { return (P)c0 | ((P)c1 << d.pk_shift); }

template <typename P>
__global__ void __launch_bounds__(256) k_pop1(DevData d, uint32_t* __restrict__ T1) {
    const int snp = blockIdx.x * blockDim.x + threadIdx.x;
    if (snp >= d.n) return;
    uint32_t c[2][2] = {{0, 0}, {0, 0}};
    for (int p = 0; p < 2; ++p)
        for (int kc = 0; kc < d.nchunks[p]; ++kc)
#pragma unroll
            for (int g = 0; g < 2; ++g) {
                const uint4 v = __ldg(reinterpret_cast<const uint4*>(d.planes[p] + plane_off(kc, d.npad, snp, g, 0)));
                c[p][g] += __popc(v.x) + __popc(v.y) + __popc(v.z) + __popc(v.w);
            }
    P* o = reinterpret_cast<P*>(T1) + (int64_t)snp * 2;
    o[0] = pkw<P>(d, c[0][0], c[1][0]);
    o[1] = pkw<P>(d, c[0][1], c[1][1]);
}

__device__ __forceinline__ void decode2(int64_t r, int& i, int& j) {
    int jj = (int)floor((1.0 + sqrt(1.0 + 8.0 * (double)r)) * 0.5);
    while (c2(jj) > r) --jj;
    while (c2(jj + 1) <= r) ++jj;
    j = jj;
    i = (int)(r - c2(jj));
}
__device__ __forceinline__ void decode3(int64_t r, int& i, int& j, int& k) {
    int kk = (int)floor(cbrt(6.0 * (double)r)) + 1;
    while (c3(kk) > r) --kk;
    while (c3(kk + 1) <= r) ++kk;
    k = kk;
    decode2(r - c3(kk), i, j);
}

__device__ __forceinline__ void ld_planes(const DevData& d, int p, int kc, int snp, uint32_t (&v)[2][4]) {
    const uint4 a = __ldg(reinterpret_cast<const uint4*>(d.planes[p] + plane_off(kc, d.npad, snp, 0, 0)));
    const uint4 b = __ldg(reinterpret_cast<const uint4*>(d.planes[p] + plane_off(kc, d.npad, snp, 1, 0)));
    v[0][0] = a.x; v[0][1] = a.y; v[0][2] = a.z; v[0][3] = a.w;
    v[1][0] = b.x; v[1][1] = b.y; v[1][2] = b.z; v[1][3] = b.w;
}

template <typename P>
__global__ void __launch_bounds__(256) k_pop2(DevData d, uint32_t* __restrict__ T2, int64_t npairs) {
    const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= npairs) return;
    int i, j;
    decode2(r, i, j);
    uint32_t out[2][4];
    for (int p = 0; p < 2; ++p) {
        uint32_t c[4] = {0, 0, 0, 0};
        for (int kc = 0; kc < d.nchunks[p]; ++kc) {
            uint32_t a[2][4], b[2][4];
            ld_planes(d, p, kc, i, a);
            ld_planes(d, p, kc, j, b);
#pragma unroll
            for (int w = 0; w < 4; ++w)
#pragma unroll
                for (int x = 0; x < 2; ++x)
#pragma unroll
                    for (int y = 0; y < 2; ++y) c[x * 2 + y] += __popc(a[x][w] & b[y][w]);
        }
#pragma unroll
        for (int q = 0; q < 4; ++q) out[p][q] = c[q];
    }
    P* o = reinterpret_cast<P*>(T2) + r * 4;
#pragma unroll
    for (int q = 0; q < 4; ++q) o[q] = pkw<P>(d, out[0][q], out[1][q]);
}

template <typename P>
__global__ void __launch_bounds__(256) k_pop3(DevData d, uint32_t* __restrict__ T3, int64_t lo, int64_t hi) {
    const int64_t r = lo + (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (r >= hi) return;
    int i, j, k;
    decode3(r, i, j, k);
    uint32_t out[2][8];
    for (int p = 0; p < 2; ++p) {
        uint32_t c[8] = {0, 0, 0, 0, 0, 0, 0, 0};
        for (int kc = 0; kc < d.nchunks[p]; ++kc) {
            uint32_t a[2][4], b[2][4], e[2][4];
            ld_planes(d, p, kc, i, a);
            ld_planes(d, p, kc, j, b);
            ld_planes(d, p, kc, k, e);
            // POPC-bound: the 4 words of a cell are summed with one carry-save step, x0 + x1 + x2 + x3 =
            // popc(s ^ x3) + 2 (popc(maj(x0, x1, x2)) + popc(s & x3)) with s = x0 ^ x1 ^ x2: 3 POPC, not 4
#pragma unroll
            for (int x = 0; x < 2; ++x)
#pragma unroll
                for (int y = 0; y < 2; ++y)
#pragma unroll
                    for (int z = 0; z < 2; ++z) {
                        uint32_t v[4];
#pragma unroll
                        for (int w = 0; w < 4; ++w) v[w] = a[x][w] & b[y][w] & e[z][w];
                        const uint32_t s3 = v[0] ^ v[1] ^ v[2];
                        const uint32_t cy = (v[0] & v[1]) | (v[2] & (v[0] ^ v[1]));
                        c[x * 4 + y * 2 + z] += __popc(s3 ^ v[3]) + 2 * (__popc(cy) + __popc(s3 & v[3]));
                    }
        }
#pragma unroll
        for (int q = 0; q < 8; ++q) out[p][q] = c[q];
    }
    P* o = reinterpret_cast<P*>(T3) + r * 8;
#pragma unroll
    for (int q = 0; q < 8; ++q) o[q] = pkw<P>(d, out[0][q], out[1][q]);
}

cudaError_t launch_pop(const DevData& d, uint32_t* T1, uint32_t* T2, uint32_t* T3, int64_t t3_lo, int64_t t3_hi,
                       cudaStream_t s, int64_t* launches) {
    if (d.wide) k_pop1<uint64_t><<<(d.n + 255) / 256, 256, 0, s>>>(d, T1);
    else k_pop1<uint32_t><<<(d.n + 255) / 256, 256, 0, s>>>(d, T1);
    if (launches) ++*launches;
    const int64_t np2 = c2(d.n);
    if (d.wide) k_pop2<uint64_t><<<(unsigned)((np2 + 255) / 256), 256, 0, s>>>(d, T2, np2);
    else k_pop2<uint32_t><<<(unsigned)((np2 + 255) / 256), 256, 0, s>>>(d, T2, np2);
    if (launches) ++*launches;
    if (t3_hi > t3_lo) {   // the triples [t3_lo, t3_hi) of the colex order (all of them unless sharded)
        if (d.wide) k_pop3<uint64_t><<<(unsigned)((t3_hi - t3_lo + 255) / 256), 256, 0, s>>>(d, T3, t3_lo, t3_hi);
        else k_pop3<uint32_t><<<(unsigned)((t3_hi - t3_lo + 255) / 256), 256, 0, s>>>(d, T3, t3_lo, t3_hi);
        if (launches) ++*launches;
    }
    return cudaGetLastError();
}

}  // namespace epi4
