// k_quad_tc.cu — the hot kernel: 4-way contraction on the 5th-generation tensor cores
// (tcgen05.mma kind::i8, {0,1} operands, s32 accumulators in TMEM) with the fused epilogue.
//
// What it computes: for a tile (w-block wb, x, y-block yb, z) the
// 128 x 128 matrix C_p[(w,x,a,b)][(y,z,c,d)] = sum over samples s of phenotype p of
// P_a(w)[s] P_b(x)[s] P_c(y)[s] P_d(z)[s]   — the 16 non-aa genotype counts of the 32 x 32 quads
// (w, x, y, z), for controls and for cases (tensorOp_4way, "a matrix with 16
// values per each quad").  Rows are pair products of the w-block with x and columns pair products of
// the y-block with z (the paper's `combine`), built on chip.
//
// Why i8: sm_100a has no native binary (b1) tensor op — ptxas emulates
// mma.sync ...b1.and.popc with legacy IMMA — so the AND+POPC of the paper becomes an
// integer MAC on {0,1} bytes: AND(a,b) = a*b and POPC = the K-sum, exact in s32.
//
// Warp roles (CTA = 8 warps, 1 CTA per SM, persistent, static tile stride):
//   warp 0      : TMEM allocation (512 columns) + one elected thread issuing tcgen05.mma
//   warps 1..3  : producers — per 128-sample chunk, AND the pre-expanded {0,1} byte planes of the single
//                 SNPs into the A (pair rows) and B (pair columns) tiles, stored K-major with the 128-byte
//                 swizzle (UMMA canonical SW128 layout), then fence.proxy.async + mbarrier arrive
//   warps 4..7  : epilogue — tcgen05.ld the control and case accumulators, 4x4 lane transposes so that
//                 one thread holds one quad's 2 x 16 counts, then the shared epilogue (aa recovery,
//                 K2 in double, top-k; epilogue.cuh)
// Pipelines: smem ring of STAGES x (A 16 KiB + B 16 KiB) (full/empty mbarriers); TMEM double buffer
// (2 x [128 ctrl | 128 case] columns) between MMA and epilogue (tmem_full/tmem_empty mbarriers).
#include "epilogue.cuh"

namespace epi4 {

namespace tc {
constexpr int M = 128, N = 128;          // UMMA shape (cta_group::1), K = 32 bytes per instruction
constexpr int KCH = EPI4_CHUNK_SAMPLES;  // 128 samples (bytes) per pipeline stage
constexpr int STAGES = 4;
constexpr int A_BYTES = M * KCH, B_BYTES = N * KCH, STAGE_BYTES = A_BYTES + B_BYTES;
constexpr int PROD_WARPS = 3, EPI_WARPS = 4;
constexpr int THREADS = 32 * (1 + PROD_WARPS + EPI_WARPS);
constexpr int TMEM_COLS = 512;
// instruction descriptor: D s32 (bits 4-5 = 2), A/B u8 (0), K-major, N>>3 at bit 17, M>>4 at bit 24
constexpr uint32_t IDESC = (2u << 4) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}  // namespace tc

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
    asm volatile("{\n\t.reg .b64 st;\n\tmbarrier.arrive.shared::cta.b64 st, [%0];\n\t}" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}
// Bounded wait: a pipeline bug traps (kernel error) after ~20 s instead of hanging the GPU.
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    if (mbar_try_wait(bar, parity)) return;
    const long long t0 = clock64();
    while (!mbar_try_wait(bar, parity)) {
        if (clock64() - t0 > 40000000000LL) __trap();
    }
}
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

// UMMA shared-memory descriptor, K-major, 128-byte swizzle: 8-row groups 1024 B apart (SBO), version 1.
__device__ __forceinline__ uint64_t sw128_desc(uint32_t saddr) {
    uint64_t d = (uint64_t)((saddr & 0x3FFFFu) >> 4);
    d |= (uint64_t)1 << 16;                 // LBO (unused for swizzled K-major)
    d |= (uint64_t)(1024 >> 4) << 32;       // SBO
    d |= (uint64_t)1 << 46;                 // descriptor version (sm_100)
    d |= (uint64_t)2 << 61;                 // SWIZZLE_128B
    return d;
}

__device__ __forceinline__ void mma_i8(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t acc) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %3, 0;\n\t"
        "tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %4, p;\n\t}" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(acc), "r"(tc::IDESC));
}
__device__ __forceinline__ void mma_commit(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
                 : "memory");
}

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t (&v)[16]) {
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
        : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
          "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
        : "r"(taddr));
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

// byte offset of (row r, 16-byte chunk c) inside a K-major SW128 tile of 128-byte rows
__device__ __forceinline__ uint32_t sw128_off(int r, int c) {
    return (uint32_t)((r >> 3) * 1024 + (r & 7) * 128 + ((c ^ (r & 7)) << 4));
}

__device__ __forceinline__ uint4 and4(uint4 a, uint4 b) { return make_uint4(a.x & b.x, a.y & b.y, a.z & b.z, a.w & b.w); }

// 4x4 transpose inside each group of 4 lanes.  In: lane t (t = lane & 3) holds v[4*jj + cd] = its row
// (ab = t) for quads jj = 0..3.  Out: lane t holds w[4*ab + cd] of quad jj = t.
__device__ __forceinline__ void quad_transpose(const uint32_t (&v)[16], uint32_t (&w)[16]) {
    const int t = threadIdx.x & 3;
    uint32_t r[4][4];   // r[k][cd]: value received in round k (k = 0: own diagonal)
#pragma unroll
    for (int cd = 0; cd < 4; ++cd) {
        r[0][cd] = t == 0 ? v[cd] : t == 1 ? v[4 + cd] : t == 2 ? v[8 + cd] : v[12 + cd];
#pragma unroll
        for (int k = 1; k < 4; ++k) {
            const int jj = t ^ k;   // send my row's value for quad jj to lane jj
            const uint32_t s = jj == 0 ? v[cd] : jj == 1 ? v[4 + cd] : jj == 2 ? v[8 + cd] : v[12 + cd];
            r[k][cd] = __shfl_xor_sync(0xffffffffu, s, k);
        }
    }
    // w[ab][cd] came in round k = ab ^ t
#pragma unroll
    for (int ab = 0; ab < 4; ++ab)
#pragma unroll
        for (int cd = 0; cd < 4; ++cd) {
            const int k = ab ^ t;
            w[ab * 4 + cd] = k == 0 ? r[0][cd] : k == 1 ? r[1][cd] : k == 2 ? r[2][cd] : r[3][cd];
        }
}

struct TileInfo {
    int32_t wb, x, yb, z;
};
__device__ __forceinline__ TileInfo decode_tile(const SearchParams& sp, int64_t tile) {
    const int64_t u = find_unit(sp.prefix, sp.nunits, tile);
    const int64_t t = tile - (u ? sp.prefix[u - 1] : 0);
    TileInfo ti;
    ti.wb = sp.units[u].wb;
    ti.x = sp.units[u].x;
    unit_tile_decode(sp.d.n, ti.x, 1, t, ti.yb, ti.z);
    return ti;
}

__global__ void __launch_bounds__(tc::THREADS, 1) k_quad_i8tc(SearchParams sp) {
    extern __shared__ unsigned char smem_raw[];
    __shared__ __align__(8) uint64_t full_bar[tc::STAGES], empty_bar[tc::STAGES];
    __shared__ __align__(8) uint64_t tfull_bar[2], tempty_bar[2];
    __shared__ uint32_t s_tmem;
    // 1024-aligned operand ring, then the top-k state
    const uint32_t raw = smem_u32(smem_raw);
    unsigned char* ring = smem_raw + (((raw + 1023u) & ~1023u) - raw);
    TopKSmem tk = topk_carve(ring + tc::STAGES * tc::STAGE_BYTES, sp.topk);

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const DevData& d = sp.d;
    if (tid == 0) {
        for (int s = 0; s < tc::STAGES; ++s) {
            mbar_init(&full_bar[s], tc::PROD_WARPS);
            mbar_init(&empty_bar[s], 1);
        }
        for (int b = 0; b < 2; ++b) {
            mbar_init(&tfull_bar[b], 1);
            mbar_init(&tempty_bar[b], tc::EPI_WARPS);
        }
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&s_tmem)),
                     "r"(tc::TMEM_COLS));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    topk_load(tk, sp, blockIdx.x, tid, tc::THREADS);
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    const uint32_t tmem = s_tmem;
    const int nch0 = d.nchunks[0], nch1 = d.nchunks[1];

    if (warp == 0) {
        // ===================== MMA issuer =====================
        if (lane == 0) {
            int stage = 0;
            uint32_t phase = 0;
            int it = 0;
            for (int64_t tile = blockIdx.x; tile < sp.ntiles; tile += gridDim.x, ++it) {
                const int buf = it & 1;
                const uint32_t tphase = (uint32_t)((it >> 1) & 1);
                mbar_wait(&tempty_bar[buf], tphase ^ 1u);   // epilogue drained this buffer
                tc_fence_after();
#pragma unroll 1
                for (int p = 0; p < 2; ++p) {
                    const uint32_t dcol = tmem + (uint32_t)(buf * 256 + p * 128);
                    const int nch = p ? nch1 : nch0;
                    for (int kc = 0; kc < nch; ++kc) {
                        mbar_wait(&full_bar[stage], phase);
                        tc_fence_after();
                        const uint32_t a0 = smem_u32(ring + stage * tc::STAGE_BYTES);
                        const uint32_t b0 = a0 + tc::A_BYTES;
#pragma unroll
                        for (int k = 0; k < tc::KCH / 32; ++k)
                            mma_i8(dcol, sw128_desc(a0 + 32 * k), sw128_desc(b0 + 32 * k), (kc | k) != 0);
                        mma_commit(&empty_bar[stage]);          // frees the smem slot when these MMAs finish
                        if (++stage == tc::STAGES) { stage = 0; phase ^= 1u; }
                    }
                }
                mma_commit(&tfull_bar[buf]);                    // accumulators of this tile are ready
            }
        }
        __syncwarp();
    } else if (warp <= tc::PROD_WARPS) {
        // ===================== producers =====================
        const int pt = tid - 32;                  // 0..95
        const int c = pt & 7;                     // 16-byte chunk of the 128-byte K row (fixed per thread)
        const int u0 = pt >> 3;                   // 0..11
        int stage = 0;
        uint32_t phase = 0;
        for (int64_t tile = blockIdx.x; tile < sp.ntiles; tile += gridDim.x) {
            const TileInfo ti = decode_tile(sp, tile);
#pragma unroll 1
            for (int p = 0; p < 2; ++p) {
                const uint8_t* E = d.expl[p];
                const int nch = p ? nch1 : nch0;
                for (int kc = 0; kc < nch; ++kc) {
                    mbar_wait(&empty_bar[stage], phase ^ 1u);
                    unsigned char* sa = ring + stage * tc::STAGE_BYTES;
                    unsigned char* sb = sa + tc::A_BYTES;
                    const uint8_t* Ek = E + (int64_t)kc * d.npad * 2 * tc::KCH;
                    const uint4 x0 = __ldg(reinterpret_cast<const uint4*>(Ek + (ti.x * 2 + 0) * tc::KCH) + c);
                    const uint4 x1 = __ldg(reinterpret_cast<const uint4*>(Ek + (ti.x * 2 + 1) * tc::KCH) + c);
                    const uint4 z0 = __ldg(reinterpret_cast<const uint4*>(Ek + (ti.z * 2 + 0) * tc::KCH) + c);
                    const uint4 z1 = __ldg(reinterpret_cast<const uint4*>(Ek + (ti.z * 2 + 1) * tc::KCH) + c);
#pragma unroll 2
                    for (int ua = u0; ua < 64; ua += 12) {
                        // A unit (i, a) -> rows i*4 + a*2 + b; B unit (j, cc) -> columns j*4 + cc*2 + dd
                        const int i = ua >> 1, a = ua & 1;
                        const uint4 wv = __ldg(reinterpret_cast<const uint4*>(Ek + ((ti.wb * EPI4_B + i) * 2 + a) * tc::KCH) + c);
                        const uint4 yv = __ldg(reinterpret_cast<const uint4*>(Ek + ((ti.yb * EPI4_B + i) * 2 + a) * tc::KCH) + c);
                        const int r0 = i * 4 + a * 2;
                        *reinterpret_cast<uint4*>(sa + sw128_off(r0, c)) = and4(wv, x0);
                        *reinterpret_cast<uint4*>(sa + sw128_off(r0 + 1, c)) = and4(wv, x1);
                        *reinterpret_cast<uint4*>(sb + sw128_off(r0, c)) = and4(yv, z0);
                        *reinterpret_cast<uint4*>(sb + sw128_off(r0 + 1, c)) = and4(yv, z1);
                    }
                    fence_proxy_async();                  // generic-proxy stores -> visible to the tensor core
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&full_bar[stage]);
                    if (++stage == tc::STAGES) { stage = 0; phase ^= 1u; }
                }
            }
        }
    } else {
        // ===================== epilogue =====================
        const int q = warp & 3;                   // TMEM lane quadrant this warp may access
        const int row = q * 32 + lane;            // = i*4 + ab
        const int i = row >> 2, t = row & 3;
        unsigned long long my_quads = 0;
        int it = 0;
        for (int64_t tile = blockIdx.x; tile < sp.ntiles; tile += gridDim.x, ++it) {
            const TileInfo ti = decode_tile(sp, tile);
            const int buf = it & 1;
            const uint32_t tphase = (uint32_t)((it >> 1) & 1);
            mbar_wait(&tfull_bar[buf], tphase);
            tc_fence_after();
            const int w = ti.wb * EPI4_B + i;
            const uint32_t tbase = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(buf * 256);
#pragma unroll 1
            for (int g = 0; g < 8; ++g) {
                uint32_t v0[16], v1[16];
                tmem_ld16(tbase + 16 * g, v0);
                tmem_ld16(tbase + 128 + 16 * g, v1);
                tmem_wait_ld();
                if (g == 7) {
                    tc_fence_before();
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&tempty_bar[buf]);
                }
                uint32_t c0[16], c1[16];
                quad_transpose(v0, c0);
                quad_transpose(v1, c1);
                const int y = ti.yb * EPI4_B + 4 * g + t;
                const bool valid = (w < ti.x) && (ti.x < y) && (y < ti.z);
                double key = 0.0;
                uint64_t idx = 0;
                if (valid) {
                    uint32_t* dump = sp.dump ? sp.dump + rank4(w, ti.x, y, ti.z) * 162 : nullptr;
                    key = score_quad(d, w, ti.x, y, ti.z, c0, c1, dump);
                    idx = pack_quad(w, ti.x, y, ti.z);
                    ++my_quads;
                }
                warp_offer(tk, valid, key, idx);
            }
        }
        unsigned long long v = my_quads;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        if (lane == 0) atomicAdd(sp.quads_done, v);
    }
    tc_fence_before();
    __syncthreads();
    tc_fence_after();
    if (warp == 0)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(tc::TMEM_COLS));
    topk_store(tk, sp, blockIdx.x, tid, tc::THREADS);
}

int32_t quad_zt(int32_t pipe) { return pipe == EPI4_PIPE_LOP3 ? 1 : 1; }

cudaError_t launch_quad_i8tc(const SearchParams& sp, int32_t grid, cudaStream_t s, int64_t* launches) {
    const size_t smem = 1024 + (size_t)tc::STAGES * tc::STAGE_BYTES + topk_smem_bytes(sp.topk);
    cudaError_t e = cudaFuncSetAttribute(k_quad_i8tc, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    k_quad_i8tc<<<grid, tc::THREADS, smem, s>>>(sp);
    if (launches) ++*launches;
    return cudaGetLastError();
}

}  // namespace epi4
