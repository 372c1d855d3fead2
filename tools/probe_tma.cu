// Microbenchmark: per-SM ingest bandwidth of cp.async.bulk (TMA bulk copy) global -> shared, L2-resident
// source, 1 CTA per SM, a ring of S stages of B bytes each; also the i8 tcgen05 MMA issue rate.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o probe_tma probe_tma.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int S>
__global__ void k_ingest(const uint8_t* src, size_t src_bytes, int bytes, int iters, unsigned long long* cyc) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ __align__(8) uint64_t bar[S];
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[s])));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    if (threadIdx.x != 0) return;
    const size_t nblk = src_bytes / bytes;
    long long t0 = clock64();
    for (int i = 0; i < iters + S; ++i) {
        const int s = i % S;
        if (i >= S) {   // wait for the copy issued S iterations ago
            const uint32_t ph = ((i - S) / S) & 1;
            uint32_t ok = 0;
            while (!ok)
                asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                             : "=r"(ok) : "r"(su32(&bar[s])), "r"(ph) : "memory");
        }
        if (i < iters) {
            const uint8_t* g = src + ((size_t)(blockIdx.x * 7919 + i * 131) % nblk) * bytes;
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[s])), "r"(bytes) : "memory");
            asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                         ::"r"(su32(sm + (size_t)s * bytes)), "l"(g), "r"(bytes), "r"(su32(&bar[s])) : "memory");
        }
    }
    cyc[blockIdx.x] = clock64() - t0;
}

int main() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    size_t src_bytes = 32u << 20;   // 32 MiB: L2 resident
    uint8_t* src;
    cudaMalloc(&src, src_bytes);
    cudaMemset(src, 1, src_bytes);
    unsigned long long* cyc;
    cudaMalloc(&cyc, nsm * sizeof(unsigned long long));
    int sizes[] = {4096, 8192, 16384, 32768};
    for (int bytes : sizes) {
        const int S = 4;
        const int iters = 4000;
        size_t smem = (size_t)S * bytes;
        cudaFuncSetAttribute(k_ingest<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        for (int grid : {1, nsm}) {
            k_ingest<4><<<grid, 32, smem>>>(src, src_bytes, bytes, iters, cyc);
            cudaEvent_t e0, e1;
            cudaEventCreate(&e0); cudaEventCreate(&e1);
            cudaEventRecord(e0);
            k_ingest<4><<<grid, 32, smem>>>(src, src_bytes, bytes, iters, cyc);
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms = 0;
            cudaEventElapsedTime(&ms, e0, e1);
            unsigned long long h[256];
            cudaMemcpy(h, cyc, grid * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
            double avg = 0;
            for (int i = 0; i < grid; ++i) avg += h[i];
            avg /= grid;
            printf("bulk %6d B x %d stages, grid %3d: %.1f B/clk/SM, chip %.2f TB/s (%s)\n", bytes, S, grid,
                   (double)bytes * iters / avg, (double)bytes * iters * grid / (ms * 1e-3) / 1e12,
                   cudaGetErrorString(cudaGetLastError()));
        }
    }
    return 0;
}
