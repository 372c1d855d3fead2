// k_quad_tc.cu — the hot kernel: 4-way contraction on the 5th-generation tensor cores
// (tcgen05.mma kind::i8, {0,1} operands, s32 accumulators in TMEM) with the fused epilogue.
//
// What it computes: for a tile (w-range wr, x, y-range y0, z) and each
// phenotype p the 128 x 128 matrix
//     C_p[(w, a)][(y, b, c, d)] = sum over samples s of phenotype p of P_a(w)[s] P_b(x)[s] P_c(y)[s] P_d(z)[s]
// for the 64 SNPs w of the range and the 16 SNPs y = y0..y0+15: the 16 non-aa genotype counts of the
// 64 x 16 quads (w, x, y, z) ("a matrix with 16 values per each quad").
// Factorisation: the paper ANDs SNP pairs into both operands (combine);
// here the A operand is the raw single-SNP planes (w, a) — copied from HBM by the TMA engine, no on-chip
// production at all — and x is folded into the B operand, whose columns are triple products
// P_b(x) & P_c(y) & P_d(z) built by two producer warps.  This halves the operand bytes that must be written
// by threads (the LSU was the bottleneck of pair x pair tiles).
// Why i8: sm_100a has no native binary tensor op (ptxas emulates mma.sync ...b1.and.popc with legacy IMMA,
// SURVEY.md App. C); AND+POPC becomes an integer MAC on {0,1} bytes, exact in s32.
//
// Warp roles (CTA = 12 warps, 1 CTA per SM, persistent, static tile stride):
//   warp 0      : TMEM allocation (512 columns) + one thread running a non-blocking event loop that issues
//                 the TMA bulk copies of a stage (A: 64 SNPs x 2 planes x 128 samples = 16 KiB, pre-swizzled
//                 in HBM; the 16 y planes, x and z) and the tcgen05.mma of ready stages
//   warps 1..3  : producers — B[(y,b,c,d)] = x_b & z_d & y_c per 16-byte piece, stored K-major SW128
//   warps 4..11 : epilogue — tcgen05.ld of the control and case accumulators, pairwise lane exchange so one
//                 thread holds one quad's 2 x 16 counts, then the shared epilogue (epilogue.cuh)
// Pipelines: STAGES x {A, B, singles} (sfull: TMA bytes landed, full: B produced, empty: MMA done);
// TMEM double buffer (2 x [128 ctrl | 128 case] columns) between MMA and epilogue.
#include "epilogue.cuh"

namespace epi4 {

namespace tc {
constexpr int M = 128, N = 128;          // UMMA shape (cta_group::1), K = 32 bytes per instruction
constexpr int KCH = EPI4_CHUNK_SAMPLES;  // 128 samples (bytes) per pipeline stage
constexpr int A_BYTES = M * KCH, B_BYTES = N * KCH;
constexpr int SY_OFF = A_BYTES + B_BYTES, SY_BYTES = 2 * EPI4_YR * KCH;   // 16 y SNPs x 2 planes
constexpr int SX_OFF = SY_OFF + SY_BYTES, SZ_OFF = SX_OFF + 2 * KCH;
constexpr int STAGE_BYTES = ((SZ_OFF + 2 * KCH) + 1023) / 1024 * 1024;
constexpr int TX_BYTES = A_BYTES + SY_BYTES + 4 * KCH;                      // bytes the TMA brings per stage
// warp 0: MMA issuer; warp 1: TMA issuer; warps 2-3: producers (alternating stages); warps 4-11:
// epilogue.  384 threads keep 168 registers per thread (above 384 ptxas drops to 128).
#ifndef EPI4_TC_PROD_WARPS
#define EPI4_TC_PROD_WARPS 2
#endif
#ifndef EPI4_TC_EPI_WARPS
#define EPI4_TC_EPI_WARPS 8
#endif
constexpr int PROD_WARPS = EPI4_TC_PROD_WARPS, EPI_WARPS = EPI4_TC_EPI_WARPS;   // EPI_WARPS: 4 or 8
constexpr int PROD_WARP0 = 2, EPI_WARP0 = 2 + PROD_WARPS;
constexpr int THREADS = 32 * (2 + PROD_WARPS + EPI_WARPS);
constexpr int EPI_SPLIT = EPI_WARPS / 4;   // warps per TMEM lane quadrant (they alternate 16-column groups)
constexpr int TMEM_COLS = 512;
constexpr int CLUSTER = 2;                 // CTAs sharing A, the y slab and x through TMA multicast
                                           // (2 packs all 148 SMs; 4 strands SMs of the 18-SM GPCs)
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
__device__ __forceinline__ bool mbar_test(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\tmbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
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

__device__ __forceinline__ uint32_t cluster_rank() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t cluster_id_x() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%clusterid.x;" : "=r"(r));
    return r;
}
__device__ __forceinline__ uint32_t nclusters_x() {
    uint32_t r;
    asm volatile("mov.u32 %0, %%nclusterid.x;" : "=r"(r));
    return r;
}
__device__ __forceinline__ void cluster_sync_all() {
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

struct TileInfo {
    int32_t wr, x, y0, z;
};
// group -> this CTA's tile: the cluster's CTA of rank r takes z = first z of the group + r (>= n: dummy)
__device__ __forceinline__ TileInfo decode_tile(const SearchParams& sp, int64_t group) {
    const int64_t u = find_unit(sp.prefix, sp.nunits, group);
    const int64_t t = group - (u ? sp.prefix[u - 1] : 0);
    TileInfo ti;
    ti.wr = sp.units[u].wr;
    ti.x = sp.units[u].x;
    unit_tile_decode(sp.d.n, ti.x, t, ti.y0, ti.z, tc::CLUSTER);
    ti.z += (int32_t)cluster_rank();
    return ti;
}

// iterator over the (tile, phenotype, chunk) steps of this CTA.  The per-phenotype chunk counts are held
// in registers: indexing the kernel-parameter arrays with a runtime index spilled the parameter block to
// the local-memory stack (L1 is mostly carved out for smem, so each step paid an L2 round trip).
struct StepIt {
    int64_t tile;
    TileInfo ti;
    int p, kc;
    int nch0, nch1;
    __device__ __forceinline__ void init(const SearchParams& sp) {
        tile = cluster_id_x();
        p = 0;
        kc = 0;
        nch0 = sp.d.nchunks[0];
        nch1 = sp.d.nchunks[1];
        if (tile < sp.ntiles) ti = decode_tile(sp, tile);
    }
    __device__ __forceinline__ bool valid(const SearchParams& sp) const { return tile < sp.ntiles; }
    __device__ __forceinline__ void next(const SearchParams& sp) {
        if (++kc == (p ? nch1 : nch0)) {
            kc = 0;
            if (++p == 2) {
                p = 0;
                tile += nclusters_x();
                if (tile < sp.ntiles) ti = decode_tile(sp, tile);
            }
        }
    }
};

__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t tx) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(tx) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}

__device__ __forceinline__ void bulk_g2s_mc(void* dst, const void* src, uint32_t bytes, uint64_t* bar, uint16_t mask) {
    asm volatile(
        "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster [%0], [%1], %2, [%3], %4;" ::"r"(
            smem_u32(dst)),
        "l"(src), "r"(bytes), "r"(smem_u32(bar)), "h"(mask)
        : "memory");
}
// arrive (when this thread's prior MMAs complete) on the same-offset mbarrier of every CTA in `mask`
__device__ __forceinline__ void mma_commit_mc(uint64_t* bar, uint16_t mask) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
                     smem_u32(bar)),
                 "h"(mask)
                 : "memory");
}

template <int STAGES>
__global__ void __launch_bounds__(tc::THREADS, 1) k_quad_i8tc(SearchParams sp) {
    extern __shared__ unsigned char smem_raw[];
    __shared__ __align__(8) uint64_t sfull_bar[STAGES], full_bar[STAGES], empty_bar[STAGES];
    __shared__ __align__(8) uint64_t tfull_bar[2], tempty_bar[2];
    __shared__ uint32_t s_tmem;
    // 1024-aligned stage ring, then the fixed-point lgamma table, then the top-k state
    const uint32_t raw = smem_u32(smem_raw);
    unsigned char* ring = smem_raw + (((raw + 1023u) & ~1023u) - raw);
    int32_t* s_lfx = reinterpret_cast<int32_t*>(ring + STAGES * tc::STAGE_BYTES);
    const int lfx_words = sp.use_lfx ? ((sp.d.lfx_n + 3) & ~3) : 0;
    TopKSmem tk = topk_carve(reinterpret_cast<unsigned char*>(s_lfx + lfx_words), sp.topk);

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const DevData& d = sp.d;
    if (tid == 0) {
        for (int s = 0; s < STAGES; ++s) {
            mbar_init(&sfull_bar[s], 1);
            mbar_init(&full_bar[s], 1);          // one producer warp builds a stage's B tile
            mbar_init(&empty_bar[s], tc::CLUSTER);   // every CTA's MMA must release a stage
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
    for (int e = tid; e < lfx_words; e += tc::THREADS) s_lfx[e] = e < d.lfx_n ? __ldg(d.lfx + e) : 0;
    tc_fence_before();
    cluster_sync_all();                  // barrier inits visible cluster-wide before any multicast
    tc_fence_after();
    const bool leader = cluster_rank() == 0;
    const uint16_t cmask = (uint16_t)((1u << tc::CLUSTER) - 1);
    const int64_t first_group = cluster_id_x(), group_stride = nclusters_x();
    const uint32_t tmem = s_tmem;
    const int64_t chunk_stride = (int64_t)d.npad * 2 * tc::KCH;   // bytes of one chunk of expl
    const int nch0_r = d.nchunks[0], nch1_r = d.nchunks[1];      // (no runtime-indexed parameter arrays)
    const uint8_t* const expl0 = d.expl[0];
    const uint8_t* const expl1 = d.expl[1];

    if (warp == 0) {
        // ===================== MMA issuer =====================
        if (lane == 0) {
            int stage = 0;
            uint32_t phase = 0;
            int it = 0;
            const bool timing = (sp.debug & 8) != 0;
            long long t_wait = 0;
            for (int64_t tile = first_group; tile < sp.ntiles; tile += group_stride, ++it) {
                const int buf = it & 1;
                const uint32_t tphase = (uint32_t)((it >> 1) & 1);
                mbar_wait(&tempty_bar[buf], tphase ^ 1u);   // epilogue drained this buffer
                tc_fence_after();
#pragma unroll 1
                for (int p = 0; p < 2; ++p) {
                    const uint32_t dcol = tmem + (uint32_t)(buf * 256 + p * 128);
                    const int nch = p ? nch1_r : nch0_r;
                    for (int kc = 0; kc < nch; ++kc) {
                        const long long t0 = timing ? clock64() : 0;
                        mbar_wait(&sfull_bar[stage], phase);
                        mbar_wait(&full_bar[stage], phase);
                        if (timing) t_wait += clock64() - t0;
                        tc_fence_after();
                        const uint32_t a0 = smem_u32(ring + stage * tc::STAGE_BYTES);
                        const uint32_t b0 = a0 + tc::A_BYTES;
                        if (!(sp.debug & 4)) {
#pragma unroll
                            for (int k = 0; k < tc::KCH / 32; ++k)
                                mma_i8(dcol, sw128_desc(a0 + 32 * k), sw128_desc(b0 + 32 * k), (kc | k) != 0);
                        }
                        mma_commit_mc(&empty_bar[stage], cmask);  // frees the stage in every CTA of the cluster
                        if (++stage == STAGES) { stage = 0; phase ^= 1u; }
                    }
                }
                mma_commit(&tfull_bar[buf]);                    // accumulators of this tile are ready
            }
            if (timing) atomicAdd(sp.prof + 5, (unsigned long long)t_wait);
        }
        __syncwarp();
    } else if (warp == 1) {
        // ===================== TMA issuer =====================
        // TL lanes issue alternating steps in lockstep (lane l: steps l, l+TL, ...), each with its own stage
        // and barrier: one thread issuing every step paid each instruction latency serially (~290 cycles per
        // step, measured with debug & 64), which bounded the whole pipeline.  TL divides STAGES, so a lane's
        // successive uses of a stage are one mbarrier phase apart.
        constexpr int TL = 1;   // 2 lanes helped the pipeline-only case but not the full kernel (measured)
        if (lane < TL) {
            StepIt st;
            st.init(sp);
            int64_t step = 0;
            for (int k = 0; k < lane && st.valid(sp); ++k, ++step) st.next(sp);
            const bool timing = (sp.debug & 8) != 0;
            long long t_wait = 0;
            while (st.valid(sp)) {
                const int stage = (int)(step % STAGES);
                const uint32_t phase = (uint32_t)((step / STAGES) & 1);
                const long long t0 = timing ? clock64() : 0;
                mbar_wait(&empty_bar[stage], phase ^ 1u);
                if (timing) t_wait += clock64() - t0;
                unsigned char* sbase = ring + stage * tc::STAGE_BYTES;
                const uint8_t* E = (st.p ? expl1 : expl0) + (int64_t)st.kc * chunk_stride;
                if (sp.debug & 128) {                 // diagnostics: no copies (MMA on stale smem)
                    mbar_arrive(&sfull_bar[stage]);
                    for (int k = 0; k < TL && st.valid(sp); ++k) st.next(sp);
                    step += TL;
                    continue;
                }
                mbar_expect_tx(&sfull_bar[stage], tc::TX_BYTES);
                if (leader) {
                    // A, the y slab and x are the same for the whole cluster: one L2 read, multicast
                    bulk_g2s_mc(sbase, E + (int64_t)st.ti.wr * EPI4_WR * 2 * tc::KCH, tc::A_BYTES, &sfull_bar[stage], cmask);
                    bulk_g2s_mc(sbase + tc::SY_OFF, E + (int64_t)st.ti.y0 * 2 * tc::KCH, tc::SY_BYTES, &sfull_bar[stage], cmask);
                    bulk_g2s_mc(sbase + tc::SX_OFF, E + (int64_t)st.ti.x * 2 * tc::KCH, 2 * tc::KCH, &sfull_bar[stage], cmask);
                }
                const int zc = st.ti.z < d.n ? st.ti.z : d.n - 1;   // dummy tile: any valid row
                bulk_g2s(sbase + tc::SZ_OFF, E + (int64_t)zc * 2 * tc::KCH, 2 * tc::KCH, &sfull_bar[stage]);
                for (int k = 0; k < TL && st.valid(sp); ++k) st.next(sp);
                step += TL;
            }
            if (timing) atomicAdd(sp.prof + 6, (unsigned long long)t_wait);
        }
        __syncwarp();
    } else if (warp >= tc::PROD_WARP0 && warp < tc::PROD_WARP0 + tc::PROD_WARPS) {
        // ===================== producers =====================
        // Producer warp j builds the whole B tile of every step s with s % PW == j, so the warps'
        // per-stage latencies (shared loads, fence.proxy.async, barrier arrive) overlap.  Lane: 16-byte
        // piece cc = lane & 7 of the 128-sample K row, plane c = (lane >> 3) & 1, y_local = (lane >> 4) + 2k.
        // B[n = 8 y_local + 4b + 2c + d] = x_b & z_d & y_c (rows of smem singles keep the HBM swizzle:
        // piece cc of absolute row r sits at piece cc ^ (r & 7)).
        // A warp's successive uses of a stage must be exactly one mbarrier phase apart (parity waits alias
        // otherwise), so the number of active producer warps must divide STAGES.
        constexpr int PW = (STAGES % tc::PROD_WARPS == 0) ? tc::PROD_WARPS : (STAGES % 2 == 0 ? 2 : 1);
        const int pw = warp - tc::PROD_WARP0;
        const int cc = lane & 7;
        const int cpl = (lane >> 3) & 1;
        const bool skip = (sp.debug & 1) != 0;
        StepIt st;
        st.init(sp);
        const bool timing = (sp.debug & 8) != 0;
        long long t_wait = 0, t_busy = 0;
        for (int64_t step = 0; st.valid(sp); st.next(sp), ++step) {
            if ((int)(step % PW) != pw) continue;     // warps with pw >= PW stay idle
            const int stage = (int)(step % STAGES);
            const uint32_t phase = (uint32_t)((step / STAGES) & 1);
            const long long t0 = timing ? clock64() : 0;
            mbar_wait(&sfull_bar[stage], phase);
            const long long t1 = timing ? clock64() : 0;
            t_wait += t1 - t0;
            if (!skip) {
                unsigned char* sbase = ring + stage * tc::STAGE_BYTES;
                unsigned char* sb = sbase + tc::A_BYTES;
                const int x = st.ti.x, z = st.ti.z, y0 = st.ti.y0;
                const uint4 x0 = *reinterpret_cast<const uint4*>(sbase + tc::SX_OFF + ((cc ^ ((2 * x) & 7)) << 4));
                const uint4 x1 = *reinterpret_cast<const uint4*>(sbase + tc::SX_OFF + 128 + ((cc ^ ((2 * x + 1) & 7)) << 4));
                const uint4 z0 = *reinterpret_cast<const uint4*>(sbase + tc::SZ_OFF + ((cc ^ ((2 * z) & 7)) << 4));
                const uint4 z1 = *reinterpret_cast<const uint4*>(sbase + tc::SZ_OFF + 128 + ((cc ^ ((2 * z + 1) & 7)) << 4));
                const uint4 xz[4] = {and4(x0, z0), and4(x0, z1), and4(x1, z0), and4(x1, z1)};   // [b*2 + d]
                uint4 yv[8];
#pragma unroll
                for (int k = 0; k < 8; ++k) {
                    const int rr = 2 * ((lane >> 4) + 2 * k) + cpl;        // row inside the y slab
                    const int ra = 2 * y0 + rr;                            // absolute row (for the swizzle)
                    yv[k] = *reinterpret_cast<const uint4*>(sbase + tc::SY_OFF + rr * 128 + ((cc ^ (ra & 7)) << 4));
                }
#pragma unroll
                for (int k = 0; k < 8; ++k) {
                    const int yl = (lane >> 4) + 2 * k;
#pragma unroll
                    for (int bd = 0; bd < 4; ++bd) {
                        const int n = yl * 8 + (bd >> 1) * 4 + cpl * 2 + (bd & 1);
                        *reinterpret_cast<uint4*>(sb + sw128_off(n, cc)) = and4(yv[k], xz[bd]);
                    }
                }
                fence_proxy_async();                      // generic-proxy stores -> visible to the tensor core
            }
            __syncwarp();
            if (lane == 0) mbar_arrive(&full_bar[stage]);
            if (timing) t_busy += clock64() - t1;
        }
        if (timing && lane == 0) {
            atomicAdd(sp.prof + 3, (unsigned long long)t_busy);
            atomicAdd(sp.prof + 4, (unsigned long long)t_wait);
        }
    } else if (warp >= tc::EPI_WARP0) {
        // ===================== epilogue =====================
        // lane quadrant q holds rows 32q..32q+31 = (w_local, a) with w_local = row/2; a 16-column group g
        // holds y_local = 2g, 2g+1 x (b, c, d).  Lanes a=0/a=1 swap halves so that lane a owns the quad
        // y_local = 2g + a with all 16 counts c16[8a' + 4b + 2c + d].
        const int ew = warp - tc::EPI_WARP0;           // 0..7
        const int q = warp & 3;                         // TMEM lane quadrant this warp may access
        const int h = ew >> 2;                          // warps of one quadrant split the column groups
        const int row = q * 32 + lane;
        const int wl = row >> 1, a = row & 1;
        unsigned long long my_quads = 0, n_exact = 0;
        long long t_wait = 0, t_busy = 0;
        const bool timing = (sp.debug & 8) != 0;
        int it = 0;
        for (int64_t tile = first_group; tile < sp.ntiles; tile += group_stride, ++it) {
            const TileInfo ti = decode_tile(sp, tile);
            const int buf = it & 1;
            const uint32_t tphase = (uint32_t)((it >> 1) & 1);
            const long long t0 = timing ? clock64() : 0;
            mbar_wait(&tfull_bar[buf], tphase);
            const long long t1 = timing ? clock64() : 0;
            t_wait += t1 - t0;
            tc_fence_after();
            const int w = ti.wr * EPI4_WR + wl;
            const uint32_t tbase = tmem + ((uint32_t)(q * 32) << 16) + (uint32_t)(buf * 256);
#pragma unroll 1
            for (int g = h; g < 8; g += tc::EPI_SPLIT) {
                uint32_t v0[16], v1[16];
                tmem_ld16(tbase + 16 * g, v0);
                tmem_ld16(tbase + 128 + 16 * g, v1);
                tmem_wait_ld();
                if (g + tc::EPI_SPLIT >= 8) {
                    tc_fence_before();
                    __syncwarp();
                    if (lane == 0) mbar_arrive(&tempty_bar[buf]);
                }
                uint32_t c0[16], c1[16];
#pragma unroll
                for (int k = 0; k < 8; ++k) {
                    // send my values for the other lane's quad, keep mine
                    const uint32_t s0 = a ? v0[k] : v0[8 + k], s1 = a ? v1[k] : v1[8 + k];
                    const uint32_t r0 = __shfl_xor_sync(0xffffffffu, s0, 1);
                    const uint32_t r1 = __shfl_xor_sync(0xffffffffu, s1, 1);
                    // lane a keeps c16[8a + k] = its own v[8a + k] and takes c16[8(1-a) + k] from the partner
                    c0[k] = a ? r0 : v0[k];
                    c0[8 + k] = a ? v0[8 + k] : r0;
                    c1[k] = a ? r1 : v1[k];
                    c1[8 + k] = a ? v1[8 + k] : r1;
                }
                const int y = ti.y0 + 2 * g + a;
                const bool valid = (w < ti.x) && (y < ti.z) && (ti.z < d.n) && !(sp.debug & 2);
                double key = 0.0;
                uint64_t idx = 0;
                bool offer = false;
                if (valid) {
                    uint32_t* dump = sp.dump ? sp.dump + rank4(w, ti.x, y, ti.z) * 162 : nullptr;
                    offer = true;
                    if (dump) {
                        key = score_quad(d, w, ti.x, y, ti.z, c0, c1, dump);
                    } else if (sp.use_lfx) {
                        // exact-bounded fixed-point filter; only possible top-k members get the exact K2
                        uint32_t acc;
                        double dummy;
                        quad_eval<true, false, false>(d, w, ti.x, y, ti.z, c0, c1, s_lfx, acc, dummy, nullptr);
                        const double thr = *reinterpret_cast<volatile double*>(tk.thr);
                        offer = (double)(int32_t)acc * d.lfx_inv_scale - d.lfx_err <= thr;
                        if (offer) {
                            key = score_quad(d, w, ti.x, y, ti.z, c0, c1, nullptr);
                            ++n_exact;
                        }
                    } else {
                        key = score_quad(d, w, ti.x, y, ti.z, c0, c1, nullptr);
                    }
                    idx = pack_quad(w, ti.x, y, ti.z);
                    ++my_quads;
                }
                warp_offer(tk, offer, key, idx);
            }
            if (timing) t_busy += clock64() - t1;
        }
        unsigned long long v = my_quads, ne = n_exact;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            v += __shfl_xor_sync(0xffffffffu, v, o);
            ne += __shfl_xor_sync(0xffffffffu, ne, o);
        }
        if (lane == 0) {
            atomicAdd(sp.quads_done, v);
            atomicAdd(sp.prof + 0, ne);
            if (timing) {
                atomicAdd(sp.prof + 1, (unsigned long long)t_busy);
                atomicAdd(sp.prof + 2, (unsigned long long)t_wait);
            }
        }
    }
    tc_fence_before();
    cluster_sync_all();                  // no CTA leaves while cluster peers may still signal it
    tc_fence_after();
    if (warp == 0)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(tc::TMEM_COLS));
    topk_store(tk, sp, blockIdx.x, tid, tc::THREADS);
}

template <int STAGES>
static cudaError_t launch_cfg(SearchParams sp, size_t smem, int32_t grid, cudaStream_t s) {
    cudaError_t e = cudaFuncSetAttribute(k_quad_i8tc<STAGES>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3(tc::THREADS);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = tc::CLUSTER;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    return cudaLaunchKernelEx(&cfg, k_quad_i8tc<STAGES>, sp);
}

int32_t quad_group(int32_t pipe) { return pipe == EPI4_PIPE_I8TC ? tc::CLUSTER : 1; }

cudaError_t launch_quad_i8tc(const SearchParams& sp_in, int32_t grid, cudaStream_t s, int64_t* launches) {
    SearchParams sp = sp_in;
    grid = grid / tc::CLUSTER * tc::CLUSTER;
    int dev = 0, optin = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    const size_t fixed = 1024 + topk_smem_bytes(sp.topk) + 1024;   // alignment + static smem slack
    const size_t lfx_bytes = (size_t)((sp.d.lfx_n + 3) & ~3) * sizeof(int32_t);
    // most pipeline stages that fit; the fixed-point K2 filter table in smem is preferred, falling back to
    // exact-only scoring when it cannot fit with at least 2 stages
    int st = 0;
    for (int pass = 0; pass < 2 && !st; ++pass) {
        sp.use_lfx = pass == 0 && sp.d.lfx != nullptr && !(sp.debug & 16);   // debug 16: no table, more stages
        for (int cand = 5; cand >= 2 && !st; --cand)
            if (fixed + (size_t)cand * tc::STAGE_BYTES + (sp.use_lfx ? lfx_bytes : 0) <= (size_t)optin) st = cand;
    }
    if (!st) return cudaErrorInvalidConfiguration;
    const size_t smem = 1024 + (size_t)st * tc::STAGE_BYTES + (sp.use_lfx ? lfx_bytes : 0) + topk_smem_bytes(sp.topk);
    cudaError_t e = st == 5 ? launch_cfg<5>(sp, smem, grid, s)
                  : st == 4 ? launch_cfg<4>(sp, smem, grid, s)
                  : st == 3 ? launch_cfg<3>(sp, smem, grid, s)
                            : launch_cfg<2>(sp, smem, grid, s);
    if (launches) ++*launches;
    return e;
}

}  // namespace epi4
