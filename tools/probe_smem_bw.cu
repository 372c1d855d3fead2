// Probe: does the 2-CTA tcgen05.mma kind::mxf4 rate share the SM's shared-memory bandwidth with the operand
// writes that feed it?  The MMA loop (static operands, M=256 N=NN K=64) runs on the leader while other warps of
// BOTH CTAs stream:
//   bit 1: TMA bulk copies global(L2-resident) -> smem, 32 KiB each, 4 in flight (warps 2, 3)
//   bit 2: STS.128 stores (warps 4..7)
//   bit 4: TMA at a throttled rate: one 32 KiB copy per `gap` cycles (the A-operand pattern of k_quad_tc)
// Reports clk per MMA (ideal N/2), and the traffic each CTA moved into its shared memory (B/clk/SM).
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o probe_smem_bw probe_smem_bw.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t sw128_desc(uint32_t saddr) {
    uint64_t d = (uint64_t)((saddr & 0x3FFFFu) >> 4);
    d |= (uint64_t)1 << 16;
    d |= (uint64_t)(1024 >> 4) << 32;
    d |= (uint64_t)1 << 46;
    d |= (uint64_t)2 << 61;
    return d;
}
__device__ __forceinline__ bool try_bar(uint64_t* bar, uint32_t ph) {
    uint32_t ok;
    asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                 : "=r"(ok) : "r"(su32(bar)), "r"(ph) : "memory");
    return ok != 0;
}
__device__ __forceinline__ void wait_bar(uint64_t* bar, uint32_t ph) { while (!try_bar(bar, ph)) {} }
__device__ __forceinline__ uint32_t hash32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352du; x ^= x >> 15; x *= 0x846ca68bu; x ^= x >> 16;
    return x;
}

constexpr int OPND = 32768;            // A (16 KiB) + B (16 KiB)
constexpr int SLOT = 32768, NSLOT = 4; // TMA landing slots
constexpr int STS_BYTES = 16384;

template <int NN>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(256, 1)
k_probe(int iters, int mode, int gap, const uint8_t* src, int nblk, unsigned long long* out /*[grid][4]*/) {
    extern __shared__ __align__(1024) uint8_t sm_raw[];
    __shared__ uint32_t s_tmem;
    __shared__ __align__(8) uint64_t bar, full[NSLOT];
    __shared__ volatile int s_done;
    __shared__ unsigned long long s_tma, s_sts;
    const uint32_t raw = su32(sm_raw);
    uint8_t* sm = sm_raw + (((raw + 1023u) & ~1023u) - raw);
    uint8_t* A = sm;
    uint8_t* B = sm + 16384;
    uint8_t* T = sm + OPND;                      // TMA slots
    uint8_t* S = T + NSLOT * SLOT;               // STS region
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    uint32_t rank;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
    for (int i = threadIdx.x; i < OPND / 4; i += blockDim.x)
        reinterpret_cast<uint32_t*>(sm)[i] = (i * 2654435761u) & 0x22222222u;
    if (threadIdx.x == 0) {
        s_done = 0;
        s_tma = 0;
        s_sts = 0;
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
        for (int s = 0; s < NSLOT; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[s])));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(su32(&s_tmem)), "r"(512));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tmem = s_tmem;
    if (warp < 4) {
        const uint32_t t = tmem + ((uint32_t)(warp * 32) << 16) + 480;
        const uint32_t v = 0x7F7F7F7Fu;
        for (int c = 0; c < 32; c += 8)
            asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%1,%1,%1,%1,%1,%1,%1};" ::"r"(t + c), "r"(v) : "memory");
        asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t idesc = (1u << 7) | (1u << 10) | ((uint32_t)(NN >> 3) << 17) | (1u << 23) | (16u << 24);
    const uint64_t ad0 = sw128_desc(su32(A)), bd0 = sw128_desc(su32(B));
    const uint32_t sf = tmem + 480;
    long long t_mma = 0, t_run = 0;
    const long long t_start = clock64();
    if (warp == 0) {
        if (lane == 0 && rank == 0) {
            for (int i = 0; i < iters; i += 4) {
#pragma unroll
                for (int k = 0; k < 4; ++k)
                    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, 1, 0;\n\t"
                                 "tcgen05.mma.cta_group::2.kind::mxf4.block_scale.block32 [%0], %1, %2, %3, [%4], [%4], p;\n\t}"
                                 ::"r"(tmem), "l"(ad0 + 2 * k), "l"(bd0 + 2 * k), "r"(idesc), "r"(sf));
            }
            asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                         ::"r"(su32(&bar)), "h"((uint16_t)3) : "memory");
            wait_bar(&bar, 0);
            t_mma = clock64() - t_start;
            s_done = 1;
        } else if (lane == 0) {
            wait_bar(&bar, 0);
            s_done = 1;
        }
    } else if (warp == 2 && (mode & (2 | 16))) {
        // TMA: 4 slots, each reissued as soon as its previous copy landed (mode 2) or every `gap` cycles (mode 16)
        unsigned long long bytes = 0;
        if (lane == 0) {
            uint32_t ph[NSLOT] = {0, 0, 0, 0};
            bool pend[NSLOT] = {false, false, false, false};
            int i = 0;
            long long next = clock64();
            while (!s_done) {
                const int s = i % NSLOT;
                if (pend[s]) {
                    while (!try_bar(&full[s], ph[s]) && !s_done) {}
                    if (s_done) break;
                    ph[s] ^= 1;
                    pend[s] = false;
                }
                if (mode & 16) {
                    while (clock64() < next && !s_done) {}
                    next += gap;
                }
                const int blk = (int)(hash32((uint32_t)blockIdx.x * 7919u + (uint32_t)i) % (uint32_t)nblk);
                asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(SLOT) : "memory");
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                             ::"r"(su32(T + s * SLOT)), "l"(src + (size_t)blk * SLOT), "r"(SLOT), "r"(su32(&full[s])) : "memory");
                pend[s] = true;
                ++i;
                bytes += SLOT;
            }
            for (int s = 0; s < NSLOT; ++s)   // drain: no copy may land after the CTA exits
                if (pend[s]) wait_bar(&full[s], ph[s]);
            s_tma = bytes;
        }
    } else if (warp >= 4 && warp < 8 && (mode & 4)) {
        const int tw = warp - 4;
        unsigned long long n = 0;
        uint32_t h = lane * 2654435761u + tw;
        while (!s_done) {
#pragma unroll 8
            for (int r = 0; r < 16; ++r)
                *reinterpret_cast<uint4*>(S + ((tw * 16 + r) * 512 + lane * 16) % STS_BYTES) = make_uint4(h, r, tw, lane);
            n += 16 * 512;
        }
        if (lane == 0) atomicAdd(&s_sts, n);
    }
    t_run = clock64() - t_start;
    __syncthreads();
    if (threadIdx.x == 0) {
        out[blockIdx.x * 4 + 0] = rank == 0 ? t_mma : 0;
        out[blockIdx.x * 4 + 1] = s_tma;
        out[blockIdx.x * 4 + 2] = s_sts;
        out[blockIdx.x * 4 + 3] = t_run;
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    asm volatile("tcgen05.fence::after_thread_sync;");
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512));
}

int main() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    const int grid = nsm / 2 * 2;
    unsigned long long* out;
    cudaMalloc(&out, grid * 4 * sizeof(unsigned long long));
    const int nblk = 1024;   // 32 MiB L2-resident source
    uint8_t* src;
    cudaMalloc(&src, (size_t)nblk * SLOT);
    cudaMemset(src, 0x22, (size_t)nblk * SLOT);
    auto run = [&](auto kern, int N, int mode, int gap) {
        const size_t smem = OPND + NSLOT * SLOT + STS_BYTES + 1024;
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        const int iters = 40000;
        kern<<<grid, 256, smem>>>(iters, mode, gap, src, nblk, out);
        cudaError_t e = cudaDeviceSynchronize();
        static unsigned long long h[4 * 1024];
        cudaMemcpy(h, out, grid * 4 * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
        double cyc = 0, tma = 0, sts = 0, run = 0;
        for (int i = 0; i < grid; ++i) {
            cyc += h[i * 4];
            tma += h[i * 4 + 1];
            sts += h[i * 4 + 2];
            run += h[i * 4 + 3];
        }
        cyc /= grid / 2;
        run /= grid;
        const double clk = cyc / iters, ideal = N / 2.0;
        printf("N=%3d mode=%2d gap=%5d  %6.1f clk/MMA (ideal %5.1f, %5.1f%%)  TMA %5.1f B/clk/SM  STS %5.1f B/clk/SM  "
               "MMA-operand smem reads ~%5.1f B/clk/SM (%s)\n",
               N, mode, gap, clk, ideal, 100.0 * ideal / clk, tma / grid / run, sts / grid / run,
               (128.0 * 32 + N / 2.0 * 32) / clk, cudaGetErrorString(e));
    };
    const int gaps[] = {1024, 512, 400};
    auto sweep = [&](auto k, int N) {
        run(k, N, 0, 0);
        run(k, N, 2, 0);
        run(k, N, 4, 0);
        run(k, N, 6, 0);
        for (int g : gaps) run(k, N, 16, g);
        for (int g : gaps) run(k, N, 16 | 4, g);
    };
    sweep(k_probe<128>, 128);
    sweep(k_probe<256>, 256);
    return 0;
}
