// Microbenchmark: 2-CTA i8 MMA (M=256, N=128, K=32) issue rate when a multicast tcgen05.commit follows every
// 4 MMAs (one pipeline step), with operands rotating over a ring of stages, as in k_quad_tc.cu.
// mode 0: no commits; 1: commit per step to a ring barrier (nobody waits);
// 2: commit per step, and the issuer waits for the commit of step s - D (D = STAGES) before issuing step s.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o probe_mma2 probe_mma2.cu
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
__device__ __forceinline__ void wait_bar(uint64_t* bar, uint32_t ph) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                     : "=r"(ok) : "r"(su32(bar)), "r"(ph) : "memory");
}

constexpr int STAGES = 6, STAGE_BYTES = 24576;
__global__ void __cluster_dims__(2, 1, 1) k_mma2(int steps, int mode, unsigned long long* cyc) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ uint32_t s_tmem;
    __shared__ __align__(8) uint64_t bar[STAGES], fin;
    const int warp = threadIdx.x >> 5;
    uint32_t rank;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
    for (int i = threadIdx.x; i < (mode == 3 ? 1 : STAGES) * STAGE_BYTES; i += blockDim.x) sm[i] = (uint8_t)(i & 1);
    if (threadIdx.x == 0) {
        for (int s = 0; s < STAGES; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[s])));
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&fin)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(su32(&s_tmem)), "r"(512));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;");
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tmem = s_tmem;
    if (threadIdx.x == 0 && rank == 0) {
        const uint32_t idesc = (2u << 4) | ((uint32_t)(128 >> 3) << 17) | (16u << 24);   // i8, M = 256, N = 128
        const uint64_t adesc0 = sw128_desc(su32(sm)), bdesc0 = sw128_desc(su32(sm) + 16384);
        long long t0 = clock64();
        int stage = 0;
        uint32_t phase = 0;
        for (int s = 0; s < steps; ++s) {
            if (mode == 2 && s >= STAGES) wait_bar(&bar[stage], phase ^ 1u);
            const int st_eff = (mode == 3) ? 0 : stage;
            const uint32_t a0 = su32(sm + st_eff * STAGE_BYTES), b0 = a0 + 16384;
            const uint32_t dcol = (mode == 4) ? 0u : (uint32_t)((s & 1) * 128);
            const uint64_t soff = (uint64_t)((st_eff * STAGE_BYTES) >> 4);
#pragma unroll
            for (int k = 0; k < 4; ++k) {
                const uint32_t acc = (s | k) != 0;
                const uint64_t ad = mode >= 6 ? adesc0 + soff + 2 * k : sw128_desc(a0 + 32 * k);
                const uint64_t bd = mode >= 6 ? bdesc0 + soff + 2 * k : sw128_desc(b0 + 32 * k);
                asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %3, 0;\n\ttcgen05.mma.cta_group::2.kind::i8 [%0], %1, %2, %4, p;\n\t}"
                             ::"r"(tmem + dcol), "l"(ad), "l"(bd), "r"(acc), "r"(idesc));
            }
            if ((mode >= 1 && mode <= 2) || mode == 6)
                asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                             ::"r"(su32(&bar[stage])), "h"((uint16_t)3) : "memory");
            if (++stage == STAGES) { stage = 0; phase ^= 1u; }
        }
        asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                     ::"r"(su32(&fin)), "h"((uint16_t)3) : "memory");
        wait_bar(&fin, 0);
        cyc[blockIdx.x / 2] = clock64() - t0;
    } else if (threadIdx.x == 0) {
        wait_bar(&fin, 0);
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    asm volatile("tcgen05.fence::after_thread_sync;");
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512));
}

int main() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    unsigned long long* cyc;
    cudaMalloc(&cyc, nsm * sizeof(unsigned long long));
    const int steps = 5000;
    const size_t smem = (size_t)STAGES * STAGE_BYTES + 1024;
    cudaFuncSetAttribute(k_mma2, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    for (int mode : {0, 1, 2, 3, 4, 5, 6}) {
        const size_t sm_b = mode == 5 ? (size_t)STAGE_BYTES + 1024 : smem;   // mode 5 = mode 3 with a small smem footprint
        k_mma2<<<nsm, 128, sm_b>>>(steps, mode == 5 ? 3 : mode, cyc);
        k_mma2<<<nsm, 128, sm_b>>>(steps, mode == 5 ? 3 : mode, cyc);
        cudaDeviceSynchronize();
        unsigned long long h[256];
        cudaMemcpy(h, cyc, nsm / 2 * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
        double avg = 0;
        for (int i = 0; i < nsm / 2; ++i) avg += h[i];
        avg /= nsm / 2;
        printf("mode %d: %.1f clk/step (4 MMAs M256 N128 K32), %.1f clk/MMA (%s)\n", mode, avg / steps, avg / steps / 4,
               cudaGetErrorString(cudaGetLastError()));
    }
    return 0;
}
