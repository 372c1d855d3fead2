// Microbenchmark: 2-CTA i8 MMA issue loop as in k_quad_tc.cu (M=256, N=128, K=32; 4 MMAs + one multicast
// commit per step; operands rotating over 6 stages), descriptors precomputed (template ISSUE = 1) or
// rebuilt per MMA from the smem address (ISSUE = 0).  Reports cycles per step and per MMA.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o probe_mma3 probe_mma3.cu
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
__device__ __forceinline__ void mma(uint32_t d, uint64_t a, uint64_t b, uint32_t acc, uint32_t idesc) {
    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %3, 0;\n\ttcgen05.mma.cta_group::2.kind::i8 [%0], %1, %2, %4, p;\n\t}"
                 ::"r"(d), "l"(a), "l"(b), "r"(acc), "r"(idesc));
}

constexpr int STAGES = 4, STAGE_BYTES = 24576;
template <int ISSUE, int KPER, int INTERF>
__global__ void __cluster_dims__(2, 1, 1) k_mma3(int steps, unsigned long long* cyc, const uint8_t* gsrc) {
    extern __shared__ __align__(1024) uint8_t sm_raw[];
    __shared__ uint32_t s_tmem;
    __shared__ __align__(8) uint64_t bar[STAGES], fin;
    const uint32_t raw = su32(sm_raw);
    uint8_t* sm = sm_raw + (((raw + 1023u) & ~1023u) - raw);
    const int warp = threadIdx.x >> 5;
    uint32_t rank;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
    for (int i = threadIdx.x; i < STAGES * STAGE_BYTES; i += blockDim.x) sm[i] = (uint8_t)(i & 1);
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
    __shared__ __align__(8) uint64_t tbar[4];
    __shared__ volatile int done_flag;
    if (threadIdx.x == 0) done_flag = 0;
    __syncthreads();
    if ((INTERF & 1) && threadIdx.x == 32) {
        // TMA: 16 KiB copies into a 4 x 16 KiB region after the stages, until the MMA issuer is done
        uint8_t* dst = sm + STAGES * STAGE_BYTES;
        for (int i = 0; i < 4; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&tbar[i])));
        int i = 0;
        while (!done_flag) {
            const int b = i & 3;
            if (i >= 4) wait_bar(&tbar[b], ((i - 4) >> 2) & 1);
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&tbar[b])), "r"(16384) : "memory");
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                         ::"r"(su32(dst + b * 16384)), "l"(gsrc + ((size_t)((blockIdx.x * 131 + i * 7) & 1023) << 14)), "r"(16384), "r"(su32(&tbar[b])) : "memory");
            ++i;
        }
        for (int k = (i > 4 ? i - 4 : 0); k < i; ++k) wait_bar(&tbar[k & 3], (k >> 2) & 1);
    }
    if ((INTERF & 2) && threadIdx.x >= 64) {
        // STS.128 traffic from warps 2-3 into the extra region (16 B per lane per store)
        uint4* dst = reinterpret_cast<uint4*>(sm + STAGES * STAGE_BYTES + 65536);
        const uint4 v = make_uint4(threadIdx.x, 1, 2, 3);
        int i = 0;
        while (!done_flag) {
#pragma unroll
            for (int k = 0; k < 16; ++k) dst[((threadIdx.x - 64) + 64 * ((i * 16 + k) & 15))] = v;
            ++i;
        }
    }
    if (threadIdx.x == 0 && rank == 0) {
        const uint32_t idesc = (2u << 4) | ((uint32_t)(128 >> 3) << 17) | (16u << 24);
        const uint64_t adesc0 = sw128_desc(su32(sm)), bdesc0 = sw128_desc(su32(sm) + 16384);
        long long t0 = clock64();
        int stage = 0;
        for (int s = 0; s < steps; ++s) {
            const uint32_t dcol = tmem + (uint32_t)((s & 1) * 128);
#pragma unroll
            for (int k = 0; k < KPER; ++k) {
                const uint32_t acc = (s | k) != 0;
                if (ISSUE) {
                    const uint64_t soff = (uint64_t)(stage * (STAGE_BYTES >> 4));
                    mma(dcol, adesc0 + soff + 2 * (k & 3), bdesc0 + soff + 2 * (k & 3), acc, idesc);
                } else {
                    const uint32_t a0 = su32(sm + stage * STAGE_BYTES), b0 = a0 + 16384;
                    mma(dcol, sw128_desc(a0 + 32 * (k & 3)), sw128_desc(b0 + 32 * (k & 3)), acc, idesc);
                }
            }
            asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                         ::"r"(su32(&bar[stage])), "h"((uint16_t)3) : "memory");
            if (++stage == STAGES) stage = 0;
        }
        asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                     ::"r"(su32(&fin)), "h"((uint16_t)3) : "memory");
        wait_bar(&fin, 0);
        cyc[blockIdx.x / 2] = clock64() - t0;
        done_flag = 1;
    } else if (threadIdx.x == 0) {
        wait_bar(&fin, 0);
        done_flag = 1;
    }
    __syncthreads();
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
    const size_t smem = (size_t)STAGES * STAGE_BYTES + 1024 + 65536 + 16384;
    uint8_t* gsrc;
    cudaMalloc(&gsrc, (size_t)1024 << 14);
    cudaMemset(gsrc, 1, (size_t)1024 << 14);
    auto run = [&](auto kern, const char* name, int kper) {
        const int steps = 20000 / kper;
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        kern<<<nsm, 128, smem>>>(steps, cyc, gsrc);
        kern<<<nsm, 128, smem>>>(steps, cyc, gsrc);
        cudaDeviceSynchronize();
        unsigned long long h[256];
        cudaMemcpy(h, cyc, nsm / 2 * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
        double avg = 0;
        for (int i = 0; i < nsm / 2; ++i) avg += h[i];
        avg /= nsm / 2;
        printf("%-28s: %.1f clk/step, %.1f clk/MMA (%s)\n", name, avg / steps, avg / steps / kper,
               cudaGetErrorString(cudaGetLastError()));
    };
    run(k_mma3<0, 4, 0>, "rebuilt desc, 4/commit", 4);
    run(k_mma3<1, 4, 0>, "precomputed desc, 4/commit", 4);
    run(k_mma3<1, 16, 0>, "precomputed desc, 16/commit", 16);
    run(k_mma3<1, 4, 1>, "4/commit + TMA 16K stream", 4);
    run(k_mma3<1, 4, 2>, "4/commit + STS stream", 4);
    run(k_mma3<1, 4, 3>, "4/commit + TMA + STS", 4);
    return 0;
}
