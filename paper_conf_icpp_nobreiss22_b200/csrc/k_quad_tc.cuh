// k_quad_tc.cuh — the hot kernel: 4-way contraction on the 5th-generation tensor cores
// (tcgen05.mma.cta_group::2.kind::mxf4, E2M1 {0, 1.0} operands, fp32 accumulators in TMEM) with the fused
// epilogue; instantiated per tile geometry (Geom128 in k_quad_tc.cu, Geom224 in k_quad_tc_n224.cu).
#pragma once
//
// What it computes: for a tile (w-range pair wp, x, y-range y0, z) and each
// phenotype p the 256 x N matrix (N = 8 YR, YR = 16 or 28 y per tile: N = 128 or 224)
//     C_p[(w, a)][(y, b, c, d)] = sum over samples s of phenotype p of P_a(w)[s] P_b(x)[s] P_c(y)[s] P_d(z)[s]
// for the 128 SNPs w of the range pair and the YR SNPs y = y0..y0+YR-1: the 16 non-aa genotype counts of the
// 128 x YR quads (w, x, y, z) ("a matrix with 16 values per each quad").
// Factorisation: the paper ANDs SNP pairs into both operands (combine);
// here the A operand is the raw single-SNP planes (w, a), copied from HBM by the TMA engine, and x is folded
// into the B operand, whose columns are triple products P_b(x) & P_c(y) & P_d(z) built on chip.
// Why block-scaled FP4: sm_100a has no native binary tensor op (ptxas emulates mma.sync ...b1.and.popc with
// legacy IMMA).  A set bit is the E2M1 value 1.0 (nibble 0x2), so AND of packed nibbles
// is the product, and with all E8M0 block scales = 1 the MMA sums exact small integers: the fp32 accumulator
// is exact up to 2^24 per phenotype (host check; tools/probe_mxf4.cu: 0 mismatches, counts to 76800).
// kind::mxf4 runs M=256 K=64 in N/2 cycles: twice the {0,1}-MACs of kind::i8 (K=32) at half the operand
// bytes (2 samples per byte).
// Why 2-CTA: a 1-CTA M=128 MMA issues every ~97 cycles whatever N; cta_group::2 reaches the full rate.
// Why two geometries (Geom below): the A operand is streamed from L2 once per (tile, sample chunk), 128 B per
// row and 256 samples for every N columns; at N = 128 that is 64 B/clk/SM of TMA ingest and ~192 B/clk/SM of
// shared-memory traffic at the full MMA rate, above what an SM sustains (tools/probe_tma3.cu, probe_smem_bw.cu),
// while N = 224 needs 37 and ~137.  TMEM (512 columns, 480.. the scale factors) holds three regions of N = 128
// fp32 columns but only two of N = 224.  With three regions tile t accumulates its controls in region (-t) mod 3
// and its cases in the next one; when the tile is done the epilogue first packs every (control, case) pair into
// one 32-bit word in the case region and zeroes the control region (pass 1, a few hundred cycles), which the
// case accumulation of tile t+1 reuses; it then scores the quads from the packed region (pass 2), which the
// control accumulation of tile t+2 reuses.  With two regions (controls in 0, cases in 1) the controls of tile
// t+1 start after pass 1 and its cases after pass 2, so the scoring hides behind the first phenotype phase
// only: the load picks N = 224 for large sample counts (api.cu tc_tile_yr).
//
// CTA pair (cluster of 2): CTA r holds the A rows of w-range 2wp + r (64 SNPs x {AA, Aa}) and builds the
// B columns of y = y0 + r YR/2 .. y0 + (r + 1) YR/2 - 1; the leader (r = 0) issues the MMAs for both; each
// CTA's TMEM receives its 128 rows x all N columns and its epilogue scores its 64 x YR quads.
// Warp roles (each CTA: 16 warps = 4 warpgroups with setmaxnreg budgets, 1 CTA per SM, persistent, static
// tile stride over clusters):
//   warps 0..1  : leader — MMA issuers (alternating steps, one elected lane each); follower — warp 0 relays
//                 "A landed" to the leader's `full` barrier; warp 0 also allocates TMEM (cta_group::2)
//   warps 2..3  : TMA issuers (alternating steps): the CTA's A, one bulk copy per step, pre-swizzled in HBM
//   warps 4..7  : producers (one chunk of every 2nd step each at N = 128, a whole step of every 4th at N = 224)
//                 — the CTA's half of B, x_b & y_c & z_d per 16-byte piece, K-major SW128, from singles loaded
//                 into registers one step ahead; then an arrival on the leader's `full`
//   warps 8..15 : epilogue — pass 1 (pack, arrive `pk`), pass 2: tcgen05.ld of the packed counts, lane-pair
//                 exchange so one thread holds one quad's 2 x 16 counts, re-zeroing, the shared per-quad
//                 evaluation (epilogue.cuh); an arrival on the leader's `ep` barrier
// Pipelines: SA x A and SB x B-half stages per CTA (sfull: own TMA landed; full @leader: both B halves built
// and the follower's A landed; empty: the issuer's MMA commit, multicast to both CTAs); TMEM: the regions
// above (tfull -> epilogue; pk, ep -> MMA issuers).  One step = CHUNKS 256-sample fp4 chunks of one phenotype
// = 4 CHUNKS MMAs.
#include <cstdio>
#include <cstdlib>
#include <type_traits>
#include "epilogue.cuh"

namespace epi4 {

namespace tc {
constexpr int M = 256;                   // UMMA M (cta_group::2), K = 64 fp4 = 32 bytes per instruction
constexpr int ROWB = 128;                // bytes of one K-major operand row per fp4 chunk (256 samples)
constexpr int A_SUB = 128 * ROWB;        // this CTA's 128 A rows of one chunk (16 KiB)
#ifndef EPI4_A_SPLIT
#define EPI4_A_SPLIT 1
#endif
constexpr int A_SPLIT = EPI4_A_SPLIT;    // lanes issuing one A stage's bulk copy in pieces (tools/probe_tma.cu: several
                                         // concurrently issued copies ingest faster than one)
#ifndef EPI4_PROD_WARPS
#define EPI4_PROD_WARPS 4
#endif
constexpr int PROD_WARPS = EPI4_PROD_WARPS, EPI_WARPS = 8;
#ifndef EPI4_MMA_ISSUERS
#define EPI4_MMA_ISSUERS 2
#endif
constexpr int MMA_ISSUERS = EPI4_MMA_ISSUERS;   // 1: one issuer, MMAs complete in step order (any ring sizes)
constexpr int MMA_WARPS = 2;             // leader CTA: two issuers alternate steps (one thread cannot hide
                                         // its own wait/bookkeeping latency behind the blocking MMA issue)
constexpr int TMA_WARPS = 2;             // a bulk-copy issue blocks its thread ~150-200 cycles: two warps alternate
constexpr int TMA_WARP0 = MMA_WARPS, PROD_WARP0 = TMA_WARP0 + TMA_WARPS, EPI_WARP0 = PROD_WARP0 + PROD_WARPS;
constexpr int THREADS = 32 * (EPI_WARP0 + EPI_WARPS);         // 512 with 4 producer warps (128 registers each before setmaxnreg)
// register split across the 4 warpgroups (needs the 16-warp layout: MMA+TMA | producers | 2 x epilogue)
#ifndef EPI4_REGSPLIT
#define EPI4_REGSPLIT 1
#endif
#ifndef EPI4_EPI_LOW
#define EPI4_EPI_LOW 1
#endif
constexpr bool REGSPLIT = EPI4_REGSPLIT && PROD_WARPS == 4 && MMA_WARPS + TMA_WARPS == 4 && EPI_WARPS == 8;
#ifndef EPI4_REGS_CTL
#define EPI4_REGS_CTL 40
#endif
#ifndef EPI4_REGS_PROD
#define EPI4_REGS_PROD 120
#endif
constexpr int REGS_CTL = EPI4_REGS_CTL, REGS_PROD = EPI4_REGS_PROD;
constexpr int REGS_EPI = ((65536 / 128 - REGS_CTL - REGS_PROD) / 2) / 8 * 8;   // 176 with 40 / 120
// measured (C2 kernel, same box): control/producers 56/104 520 ms, 48/112 503, 40/120 499, 32/128 504; the
// epilogue needs >= 176 (48/120 -> 168: 561 ms); control 24 does not fit its code (illegal instruction)
constexpr int gcd_c(int a, int b) { return b ? gcd_c(b, a % b) : a; }
constexpr int lcm_c(int a, int b) { return a / gcd_c(a, b) * b; }
constexpr int TMEM_COLS = 512;
constexpr int SF_COL = 480;              // scale factors (all E8M0 0x7F = 1.0): columns 480..511, every lane
constexpr int CLUSTER = 2;
}  // namespace tc

// Tile geometry: YR_ y SNPs per tile (UMMA N = 8 YR_ columns), CHUNKS_ fp4 chunks of 256 samples
// per pipeline step, REGIONS_ TMEM accumulator regions of N columns, ring depths SA_ x SB_ (fallback SAF_ x SBF_
// when the top-k lists leave too little shared memory).
//   N = 128 (Geom128): 3 regions rotated per tile (the scoring of tile t overlaps both phenotype phases of
//     tile t+1); per MMA K-step each SM reads 4 KiB of A for 64 B columns: ~192 B/clk/SM of shared-memory
//     traffic at the full MMA rate (A copy + MMA reads + B stores + MMA reads), above the ~155 B/clk an SM
//     sustains (tools/probe_smem_bw.cu), and the A copy alone needs 64 B/clk/SM of TMA ingest.
//   N = 224 (Geom224): A amortised over 224 columns (~137 B/clk/SM, A ingest 37 B/clk/SM); 2 x 224 columns leave no
//     third region, so the controls of tile t+1 start once the pack pass has emptied region 0 and its cases
//     once the scoring of tile t has read region 1 — hidden when the first (larger) phenotype phase is longer
//     than the scoring, i.e. at large sample counts (selected by the load, api.cu tc_tile_yr).
template <int YR_, int CHUNKS_, int REGIONS_, int SA_, int SB_, int SAF_, int SBF_, bool LATE_ = false,
          int RCTL_ = tc::REGS_CTL, int RPROD_ = tc::REGS_PROD>
struct Geom {
    static constexpr int YR = YR_, N = 8 * YR_;                // UMMA N
    static constexpr int CHUNKS = CHUNKS_;                     // fp4 chunks per pipeline stage
    static constexpr int A_BYTES = CHUNKS * tc::A_SUB;         // this CTA's A rows of one stage
    static constexpr int B_ROWS = N / 2;                       // this CTA's B columns
    static constexpr int B_SUB = (B_ROWS + 7) / 8 * 1024;
    static constexpr int B_BYTES = CHUNKS * B_SUB;
    static constexpr int YH = YR / 2;                          // y SNPs per CTA
    static constexpr int TX_BYTES = A_BYTES;                   // bytes this CTA's TMA brings per A stage
    static constexpr int PROD_STRIDE = tc::PROD_WARPS / CHUNKS;   // steps between two steps of one producer warp
    static constexpr int REGIONS = REGIONS_;
    static constexpr int ACC_COLS = REGIONS * N;
    static constexpr int NG = N / 16;                          // 16-column groups of an accumulator
    static constexpr int SA = SA_, SB = SB_, SA_F = SAF_, SB_F = SBF_;
    // LATE: a producer issues the loads of its next step's singles after building (and publishing) this one, so
    // the two register sets do not overlap (with 28 y per tile the overlapping sets spill at 120 registers)
    static constexpr bool LATE = LATE_;
    static constexpr int REGS_CTL = RCTL_, REGS_PROD = RPROD_;                  // setmaxnreg per warpgroup
    static constexpr int REGS_EPI = ((65536 / 128 - REGS_CTL - REGS_PROD) / 2) / 8 * 8;
    // block-scaled instruction descriptor: A/B E2M1 (format 1 at bits 7 and 10), K-major, N>>3 at bit 17,
    // scale format E8M0 (bit 23), M>>4 at bit 24, scale-factor ids 0, K = 64 (bit 31 = 0)
    static constexpr uint32_t IDESC =
        (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | (1u << 23) | ((uint32_t)(tc::M >> 4) << 24);
    static_assert(tc::PROD_WARPS % CHUNKS == 0, "producer warps come in groups of CHUNKS (one chunk of a step each)");
    static_assert(REGIONS == 2 || REGIONS == 3, "2 or 3 accumulator regions");
    static_assert(ACC_COLS <= tc::SF_COL, "TMEM: accumulators overlap the scale factors");
    static_assert(YH % 2 == 0 && N % 16 == 0 && N <= 256, "two y per producer lane pair; cta_group::2 N");
};
// ring depths SA x SB, fallback SA_F x SB_F (measured, profiles/r02f_variants.log; overridable for diagnostics
// builds: nvcc splits -D values at commas, so one macro each)
#ifndef EPI4_SA_N128
#define EPI4_SA_N128 4
#define EPI4_SB_N128 4
#define EPI4_SAF_N128 2
#define EPI4_SBF_N128 2
#endif
#ifndef EPI4_SA_N224
#define EPI4_SA_N224 4
#define EPI4_SB_N224 8
#define EPI4_SAF_N224 4
#define EPI4_SBF_N224 4
#endif
#ifndef EPI4_LATE_N224
#define EPI4_LATE_N224 0
#endif
#ifndef EPI4_RCTL_N224
#define EPI4_RCTL_N224 40
#define EPI4_RPROD_N224 120
#endif
#ifndef EPI4_LATE_N128
#define EPI4_LATE_N128 0
#endif
using Geom128 = Geom<EPI4_YR_N128, EPI4_CH_N128, 3, EPI4_SA_N128, EPI4_SB_N128, EPI4_SAF_N128, EPI4_SBF_N128,
                     EPI4_LATE_N128>;
using Geom224 = Geom<EPI4_YR_N224, EPI4_CH_N224, 2, EPI4_SA_N224, EPI4_SB_N224, EPI4_SAF_N224, EPI4_SBF_N224,
                     EPI4_LATE_N224, EPI4_RCTL_N224, EPI4_RPROD_N224>;


__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_arrive_local(uint64_t* bar) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
// arrive on the same-offset barrier of cluster CTA `cta`.  Release at CTA scope (the CUTLASS remote-arrive
// form): a cluster-scope release compiles to a GPU-wide memory barrier that waits for the thread's in-flight
// cp.async prefetches (~1000 cycles per step, measured with debug 64).  What the peer consumes is this CTA's
// own shared memory, read by the tensor core after fence.proxy.async; CTA-scope completion covers it.
__device__ __forceinline__ void mbar_arrive_cluster(uint64_t* bar, uint32_t cta) {
    uint32_t remote;
    asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(smem_u32(bar)), "r"(cta));
    asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" ::"r"(remote) : "memory");
}
// CTA-scope acquire: a cluster-scope acquire compiles to an L1 invalidate (CCTL.IVALL) after every successful
// poll, which evicts the epilogue's cached tables; no waiter here reads peer data through L1 (the tensor core
// reads the peer's operands through the async proxy, ordered by the producer's fence.proxy.async + release).
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}
__device__ __forceinline__ bool mbar_try_wait_sleep(uint64_t* bar, uint32_t parity) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3;\n\tselp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity), "r"(1000000u)
        : "memory");
    return ok != 0;
}
// Bounded waits: a pipeline bug traps (kernel error) instead of hanging the GPU.  The poll loop counts
// iterations instead of reading the clock (the clock reads made every poll ~8 instructions, and the spinning
// warps took issue slots from the epilogue).  mbar_wait polls (latency-critical waiters); mbar_wait_sleep
// passes a suspend-time hint so a long waiter (the epilogue waiting for a whole tile) sleeps in the barrier
// unit until the phase completes instead of polling.
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
    uint32_t n = 0;
    while (!mbar_try_wait(bar, parity))
        if (++n == (1u << 30)) __trap();
}
#ifndef EPI4_SLEEP
#define EPI4_SLEEP 1
#endif
__device__ __forceinline__ void mbar_wait_sleep(uint64_t* bar, uint32_t parity) {
    if (!EPI4_SLEEP) return mbar_wait(bar, parity);
    uint32_t n = 0;
    while (!mbar_try_wait_sleep(bar, parity))
        if (++n == (1u << 24)) __trap();
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t tx) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(tx) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}
__device__ __forceinline__ void cp_async16(void* dst, const void* src) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }
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
// D[tmem] (+)= A[smem, both CTAs] . B[smem, both CTAs]^T for the CTA pair, E2M1 x E2M1 with the block
// scales at sf (TMEM); issued by the leader only
__device__ __forceinline__ void mma2_mxf4(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc, uint32_t idesc, uint32_t sf) {
    asm volatile(
        "{\n\t.reg .pred p;\n\tsetp.ne.b32 p, 1, 0;\n\t"
        "tcgen05.mma.cta_group::2.kind::mxf4.block_scale.block32 [%0], %1, %2, %3, [%4], [%4], p;\n\t}" ::"r"(d_tmem),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(sf));
}
// arrive (when the leader's prior MMAs complete) on the same-offset barrier of both CTAs of the pair
__device__ __forceinline__ void mma2_commit_mc(uint64_t* bar) {
    asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
                     smem_u32(bar)),
                 "h"((uint16_t)3)
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
// fill 16 columns of this warp's 32 TMEM lanes with one 32-bit value
__device__ __forceinline__ void tmem_fill16(uint32_t taddr, uint32_t v) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1,%1};" ::"r"(taddr),
        "r"(v)
        : "memory");
}
__device__ __forceinline__ void tmem_zero16(uint32_t taddr) { tmem_fill16(taddr, 0u); }
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t (&v)[16]) {
    asm volatile(
        "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(taddr),
        "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "r"(v[8]), "r"(v[9]),
        "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15])
        : "memory");
}
__device__ __forceinline__ void tmem_wait_st() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }

// byte offset of (row r, 16-byte chunk c) inside a K-major SW128 tile of 128-byte rows
__device__ __forceinline__ uint32_t sw128_off(int r, int c) {
    return (uint32_t)((r >> 3) * 1024 + (r & 7) * 128 + ((c ^ (r & 7)) << 4));
}
__device__ __forceinline__ uint4 and4(uint4 a, uint4 b) { return make_uint4(a.x & b.x, a.y & b.y, a.z & b.z, a.w & b.w); }

// one lane of the (converged) warp returns true
__device__ __forceinline__ bool elect_one() {
    uint32_t pred = 0;
    asm volatile(
        "{\n\t.reg .b32 rx;\n\t.reg .pred px;\n\telect.sync rx|px, %1;\n\t@px mov.s32 %0, 1;\n\t}"
        : "+r"(pred)
        : "r"(0xffffffffu));
    return pred != 0;
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
    int32_t wp, x, y0, z;
};
__device__ __forceinline__ TileInfo decode_tile(const SearchParams& sp, int64_t tile) {
    const int64_t u = find_unit(sp.prefix, sp.nunits, tile);
    const int64_t t = tile - (u ? sp.prefix[u - 1] : 0);
    TileInfo ti;
    ti.wp = sp.units[u].wr;
    ti.x = sp.units[u].x;
    unit_tile_decode(sp.d.n, ti.x, t, ti.y0, ti.z, sp.yr);
    return ti;
}

__device__ __forceinline__ TileInfo load_tile(const SearchParams& sp, int64_t tile) {
    const uint64_t v = __ldg(sp.tile_info + tile);
    TileInfo ti;
    ti.wp = (int32_t)(v & 0xFFFF);
    ti.x = (int32_t)((v >> 16) & 0xFFFF);
    ti.y0 = (int32_t)((v >> 32) & 0xFFFF);
    ti.z = (int32_t)(v >> 48);
    return ti;
}

// iterator over the (tile, phenotype, chunk) steps of this cluster; advance(k) moves k steps ahead.
// Chunk counts live in registers (runtime indexing of kernel-parameter arrays spills the parameter block).
template <int CH>
struct StepIt {
    int64_t tile;
    TileInfo ti;
    int p, kc;
    int nch0, nch1;
    __device__ __forceinline__ void init(const SearchParams& sp) {
        tile = cluster_id_x();
        p = 0;
        kc = 0;
        nch0 = (sp.d.nchunks4[0] + CH - 1) / CH;
        nch1 = (sp.d.nchunks4[1] + CH - 1) / CH;
        if (tile < sp.ntiles) ti = load_tile(sp, tile);
    }
    __device__ __forceinline__ bool valid(const SearchParams& sp) const { return tile < sp.ntiles; }
    // physical chunk of this step (a tile-dependent rotation of the K loop was measured slower: r01 notes)
    __device__ __forceinline__ int chunk() const { return kc; }
    __device__ __forceinline__ void advance(const SearchParams& sp, int k) {
        kc += k;
        if (kc < (p ? nch1 : nch0)) return;
        const int64_t t0 = tile;
        while (kc >= (p ? nch1 : nch0)) {
            kc -= p ? nch1 : nch0;
            if (++p == 2) {
                p = 0;
                tile += nclusters_x();
            }
        }
        if (tile != t0 && tile < sp.ntiles) ti = load_tile(sp, tile);
    }
};

// Compile-time instrumentation (build with -DEPI4_PROF=1): per-role cycle counters in prof[1..7] and, with
// debug bit 64, a per-step event trace of cluster 0 printed at exit (tools/trace_view.py).
#ifndef EPI4_PROF
#define EPI4_PROF 0
#endif
#if EPI4_PROF
constexpr int TR_STEPS = 96, TR_EV = 16;
__device__ long long g_trace[2][TR_EV][TR_STEPS];
#define TRACE(ev, step)                                                                                    \
    do {                                                                                                   \
        if (tracing && (step) < TR_STEPS) g_trace[rank][ev][(step)] = clock64() - t_base;                   \
    } while (0)
#define PCLK() clock64()
#else
#define TRACE(ev, step) do { } while (0)
#define PCLK() 0LL
#endif

// Global step s of a cluster uses A stage s % SA (phase (s / SA) & 1) and B stage s % SB.  The two MMA
// issuers may issue (and complete) the steps of the other parity out of order, so a waiter is only protected
// from phase aliasing if its previous wait on a ring was on the same issuer's steps: both ring sizes must be
// multiples of MMA_WARPS, PROD_STRIDE and TMA_WARPS.
// SMP: verification variants (dump / sample hooks compiled in); the production search has neither (their
// per-quad checks cost ~3 % at C2 in registers and branches)
// WIDE: 64-bit packed counts (bits(n0) + bits(n1) > 32, epilogue.cuh): the (control, case) pair of a count no
// longer fits one TMEM column, so there is no pack pass and no region rotation: tile t accumulates its controls
// in region 0 and its cases in region 1, the epilogue reads both, and the next tile starts once it has (the
// epilogue is a small share of a tile at the sample counts that need this mode).
template <class G, int SA, int SB, bool PK16, int FILT, bool SMP, bool WIDE>
__global__ void __launch_bounds__(tc::THREADS, 1) k_quad_tc(SearchParams sp) {
    using P = std::conditional_t<WIDE, uint64_t, uint32_t>;
    constexpr int RING_MULT = tc::lcm_c(tc::lcm_c(tc::MMA_ISSUERS, G::PROD_STRIDE), tc::TMA_WARPS);
    static_assert(SA % RING_MULT == 0 && SB % RING_MULT == 0,
                  "ring sizes must be multiples of the alternating warps' strides (phase aliasing)");
    extern __shared__ unsigned char smem_raw[];
    // A ring: afull (own TMA landed), apeer (@leader: the follower's A landed, relayed), aempty (MMA commit);
    // B ring: bfull (@leader: both CTAs' producers), bempty (MMA commit)
    __shared__ __align__(8) uint64_t afull_bar[SA], apeer_bar[SA], aempty_bar[SA], bfull_bar[SB], bempty_bar[SB];
    __shared__ __align__(8) uint64_t tfull_bar[2], pk_bar, ep_bar[2];
    __shared__ uint32_t s_tmem;
    // 1024-aligned A ring, then the B ring, then the top-k state
    // (same offsets in both CTAs of the pair: the MMA addresses the peer's operands at the same offsets)
    const uint32_t raw = smem_u32(smem_raw);
    unsigned char* ring = smem_raw + (((raw + 1023u) & ~1023u) - raw);
    unsigned char* bring = ring + SA * G::A_BYTES;
    TopKSmem tk = topk_carve(bring + SB * G::B_BYTES, sp.topk);

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    // Role index: the SMSP arbiter issues the highest eligible warp id first (B300_MICROARCH.md "multi-warp
    // arbiter"), so the latency-critical roles (MMA / TMA issuers, producers) get the high physical warp ids
    // 8..15 and the throughput-bound epilogue the low ones; rw & 3 == warp & 3 (TMEM lane quadrant) and the
    // warpgroups stay aligned for setmaxnreg.
    const int rw = EPI4_EPI_LOW ? ((warp + 8) & 15) : warp;
    const DevData& d = sp.d;
    const uint32_t rank = cluster_rank();
    const bool leader = rank == 0;
    if (tid == 0) {
        for (int s = 0; s < SA; ++s) {
            mbar_init(&afull_bar[s], 1);
            mbar_init(&apeer_bar[s], 1);                  // (leader) the follower's relay
            mbar_init(&aempty_bar[s], 1);                 // the leader's MMA commit
        }
        for (int s = 0; s < SB; ++s) {
            mbar_init(&bfull_bar[s], tc::CLUSTER * G::CHUNKS);   // (leader) both CTAs' producers
            mbar_init(&bempty_bar[s], 1);                 // the leader's MMA commit
        }
        for (int b = 0; b < 2; ++b) {
            mbar_init(&tfull_bar[b], tc::MMA_ISSUERS);    // each issuer's commit after its last step
            mbar_init(&ep_bar[b], tc::CLUSTER * tc::EPI_WARPS);   // (leader) every epilogue warp of the pair
        }
        mbar_init(&pk_bar, tc::CLUSTER * tc::EPI_WARPS);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(&s_tmem)),
                     "r"(tc::TMEM_COLS));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
    }
    if (!sp.t3_out) topk_load(tk, sp, blockIdx.x, tid, tc::THREADS);   // (also the third-order search)
    // Accumulators are zeroed by the epilogue after it reads them (and once here), so every MMA accumulates:
    // the two issuers' MMAs into one tile may then complete in any order.
    __syncthreads();                     // TMEM address visible
    if (rw >= tc::EPI_WARP0) {
        const int ew = rw - tc::EPI_WARP0, q = warp & 3, h = ew >> 2;
        const uint32_t tq = s_tmem + ((uint32_t)(q * 32) << 16);
        for (int col = 16 * h; col < G::ACC_COLS; col += 32) tmem_zero16(tq + (uint32_t)col);
        if (h == 0)                      // E8M0 scale factors 2^0 for every MMA (any layout reads 0x7F)
            for (int col = tc::SF_COL; col < tc::TMEM_COLS; col += 16) tmem_fill16(tq + (uint32_t)col, 0x7F7F7F7Fu);
        tmem_wait_st();
    }
    tc_fence_before();
    cluster_sync_all();                  // barrier inits and TMEM allocation visible to the pair
    tc_fence_after();
    const uint32_t tmem = s_tmem;
#if EPI4_PROF
    const bool tracing = (sp.debug & 64) && cluster_id_x() == 0;
    const long long t_base = clock64();
#endif
    const int64_t first_tile = cluster_id_x(), tile_stride = nclusters_x();
    const int nch0_r = (d.nchunks4[0] + G::CHUNKS - 1) / G::CHUNKS, nch1_r = (d.nchunks4[1] + G::CHUNKS - 1) / G::CHUNKS;
    const int32_t nrb = d.nrb;
    const uint8_t* const expl0 = d.expl[0];
    const uint8_t* const expl1 = d.expl[1];

    // Warp-specialised register budgets (setmaxnreg, per warpgroup): the MMA/TMA issuers and the producers
    // need few registers; the epilogue warpgroups take the rest (EPI4_REGS_EPI) so the per-quad evaluation
    // runs without spills and with more loads in flight.
    if (tc::REGSPLIT) {
        if (rw < 4) asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(G::REGS_CTL));
        else if (rw < 8) asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(G::REGS_PROD));
        else asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(G::REGS_EPI));
    }
    if (rw < tc::MMA_WARPS) {
        // ===================== MMA issuers (leader CTA) =====================
        // Issuer m takes the steps s with s % MMA_WARPS == m.  The whole warp runs the loop (warp-uniform
        // control flow keeps the descriptors in uniform registers); one elected lane issues.  Descriptors are
        // precomputed once: per MMA only a 64-bit add (tools/probe_mma3.cu).  Every MMA accumulates (the
        // epilogue re-zeroes the accumulators), so the two issuers' MMAs commute.
        if (leader && rw < tc::MMA_ISSUERS) {
            const int m = rw;
            const uint32_t ring_s = smem_u32(ring), bring_s = smem_u32(bring);
            const uint64_t adesc0 = sw128_desc(ring_s), bdesc0 = sw128_desc(bring_s);
            const uint32_t sf_addr = tmem + tc::SF_COL;
            int it = 0, gstep = 0;
            long long t_wait = 0, t_tempty = 0;
            const bool do_mma = !(sp.debug & 4);
            int r0 = 0;                                   // p0 region of this tile: (-it) mod 3; p1: r0 + 1 mod 3
            for (int64_t tile = first_tile; tile < sp.ntiles; tile += tile_stride, ++it) {
                const int buf = it & 1;
                const long long te0 = PCLK();
                // the p0 region held the packed counts of tile it - 2: both CTAs' epilogues are done with them
                if (WIDE) {          // both regions held tile it - 1
                    if (it >= 1) mbar_wait(&ep_bar[(it - 1) & 1], (uint32_t)(((it - 1) >> 1) & 1));
                } else if (G::REGIONS == 2) {   // region 0 held the controls of tile it - 1: packed out
                    if (it >= 1) mbar_wait(&pk_bar, (uint32_t)((it - 1) & 1));
                } else if (it >= 2) {
                    mbar_wait(&ep_bar[buf], (uint32_t)(((it >> 1) & 1) ^ 1));
                }
                t_tempty += PCLK() - te0;
                tc_fence_after();
                const int r1 = r0 == 2 ? 0 : r0 + 1;
#pragma unroll 1
                for (int p = 0; p < 2; ++p) {
                    if (!WIDE && p == 1 && it >= 1) {
                        if (G::REGIONS == 3)   // the p1 region held the controls of tile it - 1: packed out
                            mbar_wait(&pk_bar, (uint32_t)((it - 1) & 1));
                        else                    // region 1 held the packed counts of tile it - 1: scored
                            mbar_wait(&ep_bar[(it - 1) & 1], (uint32_t)(((it - 1) >> 1) & 1));
                        tc_fence_after();
                    }
                    const uint32_t dcol = tmem + (uint32_t)((WIDE ? p : (p ? r1 : r0)) * G::N);
                    const int nch = p ? nch1_r : nch0_r;
#pragma unroll 1
                    for (int kc = 0; kc < nch; ++kc, ++gstep) {
                        if ((gstep & (tc::MMA_ISSUERS - 1)) != m) continue;
                        const int sa = gstep % SA, sb = gstep % SB;
                        const uint32_t pa = (uint32_t)((gstep / SA) & 1), pb = (uint32_t)((gstep / SB) & 1);
                        const long long t0 = PCLK();
                        if (lane == 0) TRACE(12, gstep);
                        mbar_wait(&bfull_bar[sb], pb);              // both B halves built
                        if (lane == 0) TRACE(15, gstep);
                        mbar_wait(&apeer_bar[sa], pa);              // follower's A landed
                        mbar_wait(&afull_bar[sa], pa);              // own A landed
                        t_wait += PCLK() - t0;
                        if (lane == 0) TRACE(10, gstep);
                        tc_fence_after();
                        if (elect_one()) {
                            if (do_mma) {
                                const uint32_t aoff = (uint32_t)sa * (G::A_BYTES >> 4), boff = (uint32_t)sb * (G::B_BYTES >> 4);
#pragma unroll
                                for (int j = 0; j < G::CHUNKS; ++j)
#pragma unroll
                                    for (int k = 0; k < tc::ROWB / 32; ++k)
                                        mma2_mxf4(dcol, adesc0 + aoff + j * (tc::A_SUB >> 4) + 2 * k,
                                                  bdesc0 + boff + j * (G::B_SUB >> 4) + 2 * k, G::IDESC, sf_addr);
                            }
                            mma2_commit_mc(&aempty_bar[sa]);        // frees the A stage in both CTAs
                            mma2_commit_mc(&bempty_bar[sb]);        // and the B stage
                        }
                        __syncwarp();
                        if (lane == 0) TRACE(11, gstep);
                    }
                }
                if (elect_one()) mma2_commit_mc(&tfull_bar[buf]);   // this issuer's MMAs of the tile are done
                __syncwarp();
                if (G::REGIONS == 3) r0 = r0 == 0 ? 2 : r0 - 1;
            }
            if (EPI4_PROF && lane == 0) {
                atomicAdd(sp.prof + 5, (unsigned long long)t_wait);
                atomicAdd(sp.prof + 7, (unsigned long long)t_tempty);
            }
        } else if (rw == 0) {
            // follower: relay "my A landed" (sfull) to the leader's full barrier, off the producers' path
            StepIt<G::CHUNKS> st;
            st.init(sp);
            for (int gstep = 0; st.valid(sp); st.advance(sp, 1), ++gstep) {
                mbar_wait(&afull_bar[gstep % SA], (uint32_t)((gstep / SA) & 1));
                if (lane == 0) TRACE(14, gstep);
                if (lane == 0) mbar_arrive_cluster(&apeer_bar[gstep % SA], 0);
                __syncwarp();
            }
        }
        __syncwarp();
    } else if (rw < tc::PROD_WARP0) {
        // ===================== TMA issuers: this CTA's A (16 KiB per step) =====================
        // warp t takes the steps s with s % TMA_WARPS == t; the whole warp runs the loop (uniform operands),
        // one elected lane issues
        {
            const int tw = rw - tc::TMA_WARP0;
            StepIt<G::CHUNKS> st;
            st.init(sp);
            st.advance(sp, tw);
            long long t_wait = 0;
            const uint32_t ring_s = smem_u32(ring);
            for (int gstep = tw; st.valid(sp); st.advance(sp, tc::TMA_WARPS), gstep += tc::TMA_WARPS) {
                const int sa = gstep % SA;
                const long long t0 = PCLK();
                mbar_wait(&aempty_bar[sa], (uint32_t)((gstep / SA) & 1) ^ 1u);
                t_wait += PCLK() - t0;
                if (lane == 0) TRACE(0, gstep);
                // this CTA's 128 A rows (row block 2 wp + rank) of the step's two chunks: 32 contiguous KiB in HBM,
                // copied as A_SPLIT pieces issued by as many lanes
                const uint8_t* src = (st.p ? expl1 : expl0) +
                                     expl_off(G::CHUNKS * (int64_t)st.chunk(), (int64_t)(st.ti.wp * 2 + (int)rank) * 128, nrb);
                if (sp.debug & 128) {             // diagnostics: no copy (the MMA reads stale operands)
                    if (lane == 0) mbar_arrive_local(&afull_bar[sa]);
                    __syncwarp();
                    continue;
                }
                if (lane == 0) mbar_expect_tx(&afull_bar[sa], G::TX_BYTES);
                __syncwarp();
                if (lane < tc::A_SPLIT) {
                    constexpr uint32_t piece = G::A_BYTES / tc::A_SPLIT;
                    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                                 ::"r"(ring_s + (uint32_t)(sa * G::A_BYTES) + lane * piece), "l"(src + lane * piece),
                                 "r"(piece), "r"(smem_u32(&afull_bar[sa]))
                                 : "memory");
                }
                __syncwarp();
                if (lane == 0) TRACE(1, gstep);
            }
            if (EPI4_PROF && lane == 0) atomicAdd(sp.prof + 6, (unsigned long long)t_wait);
        }
    } else if (rw < tc::EPI_WARP0) {
        // ===================== producers =====================
        // Producer warp j builds chunk jc = j % CHUNKS of this CTA's B half of every step s with
        // s % PROD_STRIDE == j / CHUNKS.  Its singles (x, z and the CTA's YH y SNPs, two planes each, pre-swizzled
        // in HBM) are loaded straight into registers one own step ahead (no shared-memory staging).  Lane:
        // 16-byte piece cc = lane & 7 of the 256-sample K row, plane c = (lane >> 3) & 1, y_local = (lane >> 4) + 2k
        // (k = 0..YH/2-1); B[n = 8 y_local + 4b + 2c + d] = x_b & y_c & z_d (a nibble-wise AND of E2M1 {0, 1.0}
        // values is their product).  The follower's A is certified to the leader by the relay warp, so producers
        // never wait for the TMA.
        static_assert(G::YH % 2 == 0, "two y per lane pair");
        constexpr int YK = G::YH / 2;
        const int pw = rw - tc::PROD_WARP0;
        const int jc = pw % G::CHUNKS, pstep0 = pw / G::CHUNKS;   // chunk of the step, first step
        const int cc = lane & 7, cpl = (lane >> 3) & 1, yq = lane >> 4;
        const bool build = !(sp.debug & 1);
        // store offsets inside the B sub-tile for bd = 2b + d (y_local = yq; + 2048 per k)
        uint32_t boff[4];
#pragma unroll
        for (int bd = 0; bd < 4; ++bd) {
            const int n7 = (bd >> 1) * 4 + cpl * 2 + (bd & 1);
            boff[bd] = (uint32_t)(yq * 1024 + n7 * 128 + ((cc ^ n7) << 4));
        }
        long long t_wait = 0, t_busy = 0, t_arr = 0;
        StepIt<G::CHUNKS> st, pre;
        st.init(sp);
        st.advance(sp, pstep0);
        pre = st;
        // logical piece cc of absolute row r sits at piece cc ^ (r & 7) of the row in HBM
        auto ld_piece = [&](const uint8_t* E, int64_t C, int64_t r) -> uint4 {
            return __ldg(reinterpret_cast<const uint4*>(E + expl_off(C, r, nrb) + ((cc ^ (int)(r & 7)) << 4)));
        };
        uint4 nx[4], ny[YK];
        auto load = [&](const StepIt<G::CHUNKS>& it) {
            if (it.valid(sp) && build) {
                const uint8_t* E = it.p ? expl1 : expl0;
                const int64_t C = G::CHUNKS * (int64_t)it.chunk() + jc;
                nx[0] = ld_piece(E, C, 2 * (int64_t)it.ti.x);
                nx[1] = ld_piece(E, C, 2 * (int64_t)it.ti.x + 1);
                nx[2] = ld_piece(E, C, 2 * (int64_t)it.ti.z);
                nx[3] = ld_piece(E, C, 2 * (int64_t)it.ti.z + 1);
                const int64_t ry = 2 * (int64_t)(it.ti.y0 + G::YH * (int)rank + yq) + cpl;
#pragma unroll
                for (int k = 0; k < YK; ++k) ny[k] = ld_piece(E, C, ry + 4 * k);
            }
        };
        load(pre);
        pre.advance(sp, G::PROD_STRIDE);
        for (int step = pstep0; st.valid(sp); step += G::PROD_STRIDE) {
            const int sb = step % SB;
            if (lane == 0) TRACE(2, step);
            uint4 cx[4], cy[YK];
#pragma unroll
            for (int k = 0; k < 4; ++k) cx[k] = nx[k];
#pragma unroll
            for (int k = 0; k < YK; ++k) cy[k] = ny[k];
            if (!G::LATE) {
                load(pre);                                        // next own step's singles (in flight)
                pre.advance(sp, G::PROD_STRIDE);
            }
            const long long t0 = PCLK();
            mbar_wait(&bempty_bar[sb], (uint32_t)((step / SB) & 1) ^ 1u);   // B slot free (MMA of step - SB done)
            const long long t1 = PCLK();
            t_wait += t1 - t0;
            if (lane == 0) TRACE(4, step);
#if EPI4_PROF
            {   // trace event 3: this step's singles have arrived (a value-dependent branch waits for the loads)
                uint32_t dep = cx[0].x | cx[1].y | cx[2].z | cx[3].w;
#pragma unroll
                for (int k = 0; k < YK; ++k) dep |= cy[k].x;
                if (lane == 0 && dep != 0x9E3779B9u) TRACE(3, step);
            }
#endif
            if (build) {
                unsigned char* bdst = bring + sb * G::B_BYTES + jc * G::B_SUB;
                const uint4 xz[4] = {and4(cx[0], cx[2]), and4(cx[0], cx[3]), and4(cx[1], cx[2]), and4(cx[1], cx[3])};
#pragma unroll
                for (int k = 0; k < YK; ++k)
#pragma unroll
                    for (int bd = 0; bd < 4; ++bd)
                        *reinterpret_cast<uint4*>(bdst + boff[bd] + k * 2048) = and4(cy[k], xz[bd]);
                if (lane == 0) TRACE(6, step);
                fence_proxy_async();                      // generic-proxy stores -> visible to the tensor core
            }
            __syncwarp();
            const long long t2 = PCLK();
            if (lane == 0) {
                TRACE(7, step);
                if (leader) mbar_arrive_local(&bfull_bar[sb]);
                else mbar_arrive_cluster(&bfull_bar[sb], 0);             // the leader's barrier
                TRACE(9, step);
            }
            __syncwarp();
            if (G::LATE) {
                load(pre);                                        // next own step's singles, after this one is out
                pre.advance(sp, G::PROD_STRIDE);
            }
            if (EPI4_PROF) {
                const long long t3 = PCLK();
                t_busy += t3 - t1;
                t_arr += t3 - t2;
            }
            st.advance(sp, G::PROD_STRIDE);
        }
        if (EPI4_PROF && lane == 0) {
            atomicAdd(sp.prof + 3, (unsigned long long)t_busy);
            atomicAdd(sp.prof + 4, (unsigned long long)t_wait);
            (void)t_arr;
        }
    } else {
        // ===================== epilogue =====================
        // lane quadrant q holds rows 32q..32q+31 = (w_local, a) with w_local = row/2; a 16-column group g
        // holds y_local = 2g, 2g+1 x (b, c, d).  Lanes a=0/a=1 swap halves so that lane a owns the quad
        // y_local = 2g + a with all 16 counts c16[8a' + 4b + 2c + d].
        const int ew = rw - tc::EPI_WARP0;             // 0..7
        const int q = warp & 3;                         // TMEM lane quadrant this warp may access
        const int h = ew >> 2;                          // two warps per quadrant split the column groups
        const int row = q * 32 + lane;
        const int wl = row >> 1, a = row & 1;
        unsigned long long my_quads = 0, n_exact = 0;
        long long t_wait = 0, t_busy = 0;
        const bool score = !(sp.debug & 2);
        int it = 0;
        const uint32_t pks = (uint32_t)d.pk_shift;
        int r0 = 0;                                     // the MMA issuers' region rotation
        // top_k <= 32: a race-free list per warp in registers (epilogue.cuh WarpList); else the CTA's locked list
        const bool wlist = use_warp_lists(sp.topk) && !sp.t3_out;
        WarpList wlst;
        wl_init(wlst);
        if (wlist && ew == 0) wl_load(wlst, sp, blockIdx.x);   // the CTA's keys from the previous launches
        double wthr = wlist ? wl_thr(wlst, sp.topk) : 0.0;
        for (int64_t tile = first_tile; tile < sp.ntiles; tile += tile_stride, ++it) {
            const TileInfo ti = load_tile(sp, tile);
            const int buf = it & 1;
            const uint32_t tphase = (uint32_t)((it >> 1) & 1);
            const int r1 = r0 == 2 ? 0 : r0 + 1;
            const long long t0 = PCLK();
            mbar_wait_sleep(&tfull_bar[buf], tphase);
            const long long t1 = PCLK();
            t_wait += t1 - t0;
            tc_fence_after();
            const int w = (ti.wp * 2 + (int)rank) * EPI4_WR + wl;
            const uint32_t tq = tmem + ((uint32_t)(q * 32) << 16);
            const uint32_t R0 = tq + (uint32_t)((WIDE ? 0 : r0) * G::N), R1 = tq + (uint32_t)((WIDE ? 1 : r1) * G::N);
            // pass 1: pack each (control, case) count pair into one 32-bit word, in place in the case region,
            // and zero the control region, which the next tile's case accumulation reuses
#pragma unroll 1
            for (int g = h; g < (WIDE ? 0 : G::NG); g += 2) {
                uint32_t v0[16], v1[16];
                tmem_ld16(R0 + 16 * g, v0);
                tmem_ld16(R1 + 16 * g, v1);
                tmem_wait_ld();
#pragma unroll
                for (int k = 0; k < 16; ++k)              // fp32 accumulators hold exact integers < 2^23: adding
                    v1[k] = (__float_as_uint(__uint_as_float(v0[k]) + 8388608.0f) & 0x7FFFFFu) |   // 2^23 puts
                            ((__float_as_uint(__uint_as_float(v1[k]) + 8388608.0f) & 0x7FFFFFu) << pks);  // them in
                tmem_st16(R1 + 16 * g, v1);                                              // the mantissa
                tmem_zero16(R0 + 16 * g);
            }
            if (!WIDE) {
                tmem_wait_st();
                tc_fence_before();
                __syncwarp();
                if (lane == 0) {
                    if (leader) mbar_arrive_local(&pk_bar);
                    else mbar_arrive_cluster(&pk_bar, 0);   // the leader's barrier
                }
            }
            // pass 2: score the quads from the packed counts
#pragma unroll 1
            for (int g = h; g < G::NG; g += 2) {
                P v[16];
                if constexpr (WIDE) {   // unpacked fp32 counts of both regions -> 64-bit packed words
                    uint32_t v0[16], v1[16];
                    tmem_ld16(R0 + 16 * g, v0);
                    tmem_ld16(R1 + 16 * g, v1);
                    tmem_wait_ld();
                    tmem_zero16(R0 + 16 * g);
#pragma unroll
                    for (int k = 0; k < 16; ++k)
                        v[k] = (uint64_t)(__float_as_uint(__uint_as_float(v0[k]) + 8388608.0f) & 0x7FFFFFu) |
                               ((uint64_t)(__float_as_uint(__uint_as_float(v1[k]) + 8388608.0f) & 0x7FFFFFu) << 32);
                } else {
                    tmem_ld16(R1 + 16 * g, v);
                    tmem_wait_ld();
                }
                tmem_zero16(R1 + 16 * g);                 // ready for a later tile's accumulation
                if (g + 2 >= G::NG) {
                    tmem_wait_st();
                    tc_fence_before();
                    __syncwarp();
                    if (lane == 0) {
                        if (leader) mbar_arrive_local(&ep_bar[buf]);
                        else mbar_arrive_cluster(&ep_bar[buf], 0);   // the leader's barrier
                    }
                }
                P c16[16];
#pragma unroll
                for (int k = 0; k < 8; ++k) {
                    // send my values for the other lane's quad, keep mine; lane a keeps c16[8a + k] = its own
                    // v[8a + k] and takes c16[8(1-a) + k] from the partner (packed control | case words)
                    const P sv = a ? v[k] : v[8 + k];
                    const P rv = __shfl_xor_sync(0xffffffffu, sv, 1);
                    c16[k] = a ? rv : v[k];
                    c16[8 + k] = a ? v[8 + k] : rv;
                }
                const int y = ti.y0 + 2 * g + a;
                if (sp.t3_out) {
                    // 3-way-table mode (z = the all-ones SNP n): the d = AA columns are T3(w, x, y)[a b c]
                    // (PAPER.md:L118 tensorOp_3way); already packed (control | case), written in the T3 layout
                    if (w < ti.x && y < ti.z) {
                        // resident: colex rank; windowed slab FIRST(R): (w - w0) * C(n,2) + rank2(x, y)
                        const int64_t e = sp.t3_slab_w0 >= 0
                                              ? (int64_t)(w - sp.t3_slab_w0) * c2(d.n) + c2(y) + ti.x
                                              : rank3(w, ti.x, y);
                        P* o = reinterpret_cast<P*>(sp.t3_out) + e * 8;
#pragma unroll
                        for (int k = 0; k < 8; ++k) o[k] = c16[2 * k];
                    }
                    continue;
                }
                if (sp.search3) {
                    // third-order search (z = the all-ones SNP n): triple (w, x, y) from the d = AA columns
                    const bool v3 = (w < ti.x) && (y < ti.z) && score;
                    double key3 = 0.0;
                    uint64_t idx3 = 0;
                    if (v3) {
                        const P c8[8] = {c16[0], c16[2], c16[4], c16[6], c16[8], c16[10], c16[12], c16[14]};
                        key3 = score_triple<P>(d, w, ti.x, y, c8);
                        idx3 = pack_quad(w, ti.x, y, 0);
                        ++my_quads;
                    }
                    if (wlist) wl_offer(wlst, sp.topk, wthr, v3, key3, idx3);
                    else warp_offer(tk, v3, key3, idx3);
                    continue;
                }
                const bool valid = (w < ti.x) && (y < ti.z) && score;
                double key = 0.0;
                uint64_t idx = 0;
                bool offer = false;
                if (valid) {
                    uint32_t* dump = SMP && sp.dump ? sp.dump + rank4(w, ti.x, y, ti.z) * 162 : nullptr;
                    offer = true;
                    if (SMP && dump) {
                        key = score_quad_rare<P>(d, w, ti.x, y, ti.z, c16, dump);
                        if (d.objective != EPI4_OBJ_K2) key = score_quad_rare<P>(d, w, ti.x, y, ti.z, c16, nullptr);
                    } else if (SMP && sample_hit(sp, pack_quad(w, ti.x, y, ti.z))) {
                        key = sample_record_rare<P>(sp, w, ti.x, y, ti.z, c16);
                    } else if (sp.use_filter) {
                        // fp32 filter (epilogue.cuh); only possible top-k members get the exact score.
                        // FILT 0: Stirling K2 bound; FILT 1: chi-square upper bound (key = -X^2); FILT 2: MI
                        // upper bound (key = -M*I)
                        float flt;
                        double unused;
                        quad_eval<FILT == 1 ? 5 : FILT == 2 ? 6 : 0, PK16, P>(d, quad_ranks(d, w, ti.x, y, ti.z), w, ti.x, y,
                                                                              ti.z, c16, flt, unused, nullptr);
                        const double thr = wlist ? wthr : *reinterpret_cast<volatile double*>(tk.thr);
                        if (FILT == 1)
                            offer = d.chi_M - (double)flt * (1.0 + 1.0 / 4096.0) <= thr;
                        else if (FILT == 2)
                            offer = -(((double)flt + d.mi_E) * 0.69314718055994530942 + d.mi_const) <= thr;
                        else
                            offer = (double)flt * 0.69314718055994530942 + d.flt_off <= thr;
                        if (offer) {
                            // rare path: the noinline exact scorer takes the counts through local memory
                            key = score_quad_rare<P>(d, w, ti.x, y, ti.z, c16, nullptr);
                            ++n_exact;
                        }
                    } else {
                        key = score_quad_rare<P>(d, w, ti.x, y, ti.z, c16, nullptr);
                    }
                    idx = pack_quad(w, ti.x, y, ti.z);
                    ++my_quads;
                }
                if (wlist) wl_offer(wlst, sp.topk, wthr, offer, key, idx);
                else warp_offer(tk, offer, key, idx);
            }
            t_busy += PCLK() - t1;
            if (G::REGIONS == 3) r0 = r0 == 0 ? 2 : r0 - 1;
        }
        // fold the 8 warp lists into the CTA's global slot (named barrier 1 over the epilogue warps)
        if (wlist) wl_merge_store(wlst, sp.topk, ew, tc::EPI_WARPS, 1, tk.stage_k, tk.stage_i, sp, blockIdx.x);
        unsigned long long v = my_quads, ne = n_exact;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            v += __shfl_xor_sync(0xffffffffu, v, o);
            ne += __shfl_xor_sync(0xffffffffu, ne, o);
        }
        if (lane == 0) {
            atomicAdd(sp.quads_done, v);
            atomicAdd(sp.prof + 0, ne);
            if (EPI4_PROF) {
                atomicAdd(sp.prof + 1, (unsigned long long)t_busy);
                atomicAdd(sp.prof + 2, (unsigned long long)t_wait);
            }
        }
    }
    tc_fence_before();
    cluster_sync_all();                  // no CTA leaves while its peer may still signal it / read its smem
    tc_fence_after();
    if (warp == 0)
        asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(tc::TMEM_COLS));
    if (!sp.t3_out && !use_warp_lists(sp.topk)) topk_store(tk, sp, blockIdx.x, tid, tc::THREADS);
#if EPI4_PROF
    if (tracing && tid == 0) {
        for (int k = 0; k < TR_STEPS; ++k)
            printf("TR %u %d %lld %lld %lld %lld %lld %lld %lld %lld %lld %lld %lld %lld %lld %lld %lld %lld\n", rank, k,
                   g_trace[rank][0][k], g_trace[rank][1][k], g_trace[rank][2][k], g_trace[rank][3][k],
                   g_trace[rank][4][k], g_trace[rank][5][k], g_trace[rank][6][k], g_trace[rank][7][k],
                   g_trace[rank][8][k], g_trace[rank][9][k], g_trace[rank][10][k], g_trace[rank][11][k],
                   g_trace[rank][12][k], g_trace[rank][13][k], g_trace[rank][14][k], g_trace[rank][15][k]);
    }
#endif
}

template <class G, int SA, int SB, bool PK16, int FILT, bool SMP, bool WIDE = false>
static cudaError_t launch_cfg(SearchParams sp, size_t smem, int32_t grid, cudaStream_t s) {
    cudaError_t e = cudaFuncSetAttribute(k_quad_tc<G, SA, SB, PK16, FILT, SMP, WIDE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
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
    return cudaLaunchKernelEx(&cfg, k_quad_tc<G, SA, SB, PK16, FILT, SMP, WIDE>, sp);
}

// one persistent launch of the geometry G over sp's tiles (explicitly instantiated in k_quad_tc.cu / k_quad_tc_n224.cu)
template <class G>
cudaError_t launch_quad_tc_geom(const SearchParams& sp_in, int32_t grid, cudaStream_t s, int64_t* launches) {
    SearchParams sp = sp_in;
    grid = grid / tc::CLUSTER * tc::CLUSTER;
    int dev = 0, optin = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&optin, cudaDevAttrMaxSharedMemoryPerBlockOptin, dev);
    const size_t fixed = 1024 + topk_smem_bytes(sp.topk) + 1024;   // alignment + static smem slack
    // the geometry's rings if they fit beside the top-k lists, else its shallower fallback
    struct Cfg { int sa, sb; };
    const Cfg cands[] = {{G::SA, G::SB}, {G::SA_F, G::SB_F}};
    Cfg pick{0, 0};
    for (const Cfg& c : cands)
        if (!pick.sa && fixed + (size_t)c.sa * G::A_BYTES + (size_t)c.sb * G::B_BYTES <= (size_t)optin) pick = c;
    if (!pick.sa) return cudaErrorInvalidConfiguration;
    const size_t smem = 1024 + (size_t)pick.sa * G::A_BYTES + (size_t)pick.sb * G::B_BYTES + topk_smem_bytes(sp.topk);
    if (getenv("EPI4_VERBOSE"))
        fprintf(stderr, "k_quad_tc: N %d, %d regions, %d chunk(s) per step, A/B stages %d/%d, filter %d, smem %zu B, grid %d\n",
                G::N, G::REGIONS, G::CHUNKS, pick.sa, pick.sb, sp.use_filter, smem, grid);
    cudaError_t e = cudaErrorInvalidConfiguration;
    const bool pk16 = sp.d.pk_shift == 16;
    const int filt = sp.use_filter == 2 ? 1 : sp.use_filter == 3 ? 2 : 0;   // FILT 1: chi-square, 2: MI
    const bool smp = sp.dump != nullptr || sp.samp_cap > 0;
#define EPI4_LAUNCH_F(A_, B_, SM_)                                                                             \
    e = filt == 1 ? (pk16 ? launch_cfg<G, A_, B_, true, 1, SM_>(sp, smem, grid, s) : launch_cfg<G, A_, B_, false, 1, SM_>(sp, smem, grid, s)) \
      : filt == 2 ? (pk16 ? launch_cfg<G, A_, B_, true, 2, SM_>(sp, smem, grid, s) : launch_cfg<G, A_, B_, false, 2, SM_>(sp, smem, grid, s)) \
                  : (pk16 ? launch_cfg<G, A_, B_, true, 0, SM_>(sp, smem, grid, s) : launch_cfg<G, A_, B_, false, 0, SM_>(sp, smem, grid, s))
#define EPI4_LAUNCH_W(A_, B_, SM_)                                                                             \
    e = filt == 1 ? launch_cfg<G, A_, B_, false, 1, SM_, true>(sp, smem, grid, s)                              \
      : filt == 2 ? launch_cfg<G, A_, B_, false, 2, SM_, true>(sp, smem, grid, s)                              \
                  : launch_cfg<G, A_, B_, false, 0, SM_, true>(sp, smem, grid, s)
#define EPI4_LAUNCH(A_, B_) do { if (sp.d.wide) { if (smp) EPI4_LAUNCH_W(A_, B_, true); else EPI4_LAUNCH_W(A_, B_, false); } \
                                 else if (smp) EPI4_LAUNCH_F(A_, B_, true); else EPI4_LAUNCH_F(A_, B_, false); } while (0)
    if (pick.sa == G::SA && pick.sb == G::SB) EPI4_LAUNCH(G::SA, G::SB);
    else EPI4_LAUNCH(G::SA_F, G::SB_F);
#undef EPI4_LAUNCH
#undef EPI4_LAUNCH_F
#undef EPI4_LAUNCH_W
    if (launches) ++*launches;
    return e;
}

}  // namespace epi4
