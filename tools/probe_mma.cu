// Microbenchmark: tcgen05.mma.cta_group::1.kind::i8 throughput from shared memory (SW128 K-major operands),
// back-to-back issue by one thread with one commit at the end.  Reports cycles per MMA and MAC/clk/SM for
// N = 64, 128, 256 (M = 128, K = 32 per instruction).  1 CTA per SM, all SMs.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o probe_mma probe_mma.cu
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

template <int N>
__global__ void k_mma(int iters, unsigned long long* cyc, int kind) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ uint32_t s_tmem;
    __shared__ __align__(8) uint64_t bar;
    const int warp = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < (128 + N) * 128; i += blockDim.x) sm[i] = (uint8_t)(i & 1);
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    if (warp == 0) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(su32(&s_tmem)), "r"(512));
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    const uint32_t tmem = s_tmem;
    if (threadIdx.x == 0) {
        const uint32_t a0 = su32(sm), b0 = a0 + 128 * 128;
        const uint32_t idesc = kind == 0 ? ((2u << 4) | ((uint32_t)(N >> 3) << 17) | (8u << 24))     // i8 -> s32
                                         : ((1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | (8u << 24));  // bf16 -> f32
        long long t0 = clock64();
        for (int i = 0; i < iters; ++i) {
            const int k = i & 3;
            const uint64_t ad = sw128_desc(a0 + 32 * k), bd = sw128_desc(b0 + 32 * k);
            const uint32_t acc = i > 0;
            if (kind == 0)
                asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %3, 0;\n\ttcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %4, p;\n\t}"
                             ::"r"(tmem), "l"(ad), "l"(bd), "r"(acc), "r"(idesc));
            else
                asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %3, 0;\n\ttcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %4, p;\n\t}"
                             ::"r"(tmem), "l"(ad), "l"(bd), "r"(acc), "r"(idesc));
        }
        asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar)) : "memory");
        uint32_t ok = 0;
        while (!ok)
            asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0,1,0,p;}"
                         : "=r"(ok) : "r"(su32(&bar)) : "memory");
        cyc[blockIdx.x] = clock64() - t0;
    }
    asm volatile("tcgen05.fence::before_thread_sync;");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;");
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512));
}

// cta_group::2: a 2-CTA cluster, M = 256 (128 rows per CTA), N columns split N/2 per CTA; the leader issues.
template <int N>
__global__ void __cluster_dims__(2, 1, 1) k_mma2(int iters, unsigned long long* cyc) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ uint32_t s_tmem;
    __shared__ __align__(8) uint64_t bar;
    const int warp = threadIdx.x >> 5;
    uint32_t rank;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
    for (int i = threadIdx.x; i < (128 + N / 2) * 128; i += blockDim.x) sm[i] = (uint8_t)(i & 1);
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
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
        const uint32_t a0 = su32(sm), b0 = a0 + 128 * 128;
        const uint32_t idesc = (2u << 4) | ((uint32_t)(N >> 3) << 17) | (16u << 24);   // i8, M = 256
        long long t0 = clock64();
        for (int i = 0; i < iters; ++i) {
            const int k = i & 3;
            const uint64_t ad = sw128_desc(a0 + 32 * k), bd = sw128_desc(b0 + 32 * k);
            const uint32_t acc = i > 0;
            asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.b32 p, %3, 0;\n\ttcgen05.mma.cta_group::2.kind::i8 [%0], %1, %2, %4, p;\n\t}"
                         ::"r"(tmem), "l"(ad), "l"(bd), "r"(acc), "r"(idesc));
        }
        asm volatile("tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;"
                     ::"r"(su32(&bar)), "h"((uint16_t)3) : "memory");
        uint32_t ok = 0;
        while (!ok)
            asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0,1,0,p;}"
                         : "=r"(ok) : "r"(su32(&bar)) : "memory");
        cyc[blockIdx.x / 2] = clock64() - t0;
    } else if (threadIdx.x == 0) {
        uint32_t ok = 0;
        while (!ok)
            asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0,1,0,p;}"
                         : "=r"(ok) : "r"(su32(&bar)) : "memory");
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
    const int iters = 20000;
    auto run = [&](auto kern, int N, int kind) {
        size_t smem = (size_t)(128 + N) * 128 + 1024;
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        kern<<<nsm, 128, smem>>>(iters, cyc, kind);
        kern<<<nsm, 128, smem>>>(iters, cyc, kind);
        cudaDeviceSynchronize();
        unsigned long long h[256];
        cudaMemcpy(h, cyc, nsm * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
        double avg = 0;
        for (int i = 0; i < nsm; ++i) avg += h[i];
        avg /= nsm;
        const double macs = 128.0 * N * (kind == 0 ? 32 : 16);
        printf("%s M=128 N=%3d: %.1f clk/MMA, %.0f MAC/clk/SM (%s)\n", kind == 0 ? "i8  " : "bf16", N, avg / iters,
               macs * iters / avg, cudaGetErrorString(cudaGetLastError()));
    };
    for (int kind : {0}) {
        run(k_mma<64>, 64, kind);
        run(k_mma<128>, 128, kind);
        run(k_mma<256>, 256, kind);
    }
    auto run2 = [&](auto kern, int N) {
        size_t smem = (size_t)(128 + N / 2) * 128 + 1024;
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        kern<<<nsm, 128, smem>>>(iters, cyc);
        kern<<<nsm, 128, smem>>>(iters, cyc);
        cudaDeviceSynchronize();
        unsigned long long h[256];
        cudaMemcpy(h, cyc, nsm / 2 * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
        double avg = 0;
        for (int i = 0; i < nsm / 2; ++i) avg += h[i];
        avg /= nsm / 2;
        const double macs = 256.0 * N * 32 / 2;   // per SM
        printf("i8 2-CTA M=256 N=%3d: %.1f clk/MMA, %.0f MAC/clk/SM (%s)\n", N, avg / iters, macs * iters / avg,
               cudaGetErrorString(cudaGetLastError()));
    };
    run2(k_mma2<64>, 64);
    run2(k_mma2<128>, 128);
    run2(k_mma2<256>, 256);
    return 0;
}
