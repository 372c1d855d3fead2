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

// variants: mode 0 = wait+expect+copy per iteration (baseline); 1 = no wait (barrier reuse unchecked, timing
// only); 2 = expect_tx + copy only, no wait, no barrier (copy issue cost); 3 = L lanes issue L stages per
// warp-iteration (each lane: wait + expect + copy on its own stage)
template <int S>
__global__ void k_variant(const uint8_t* src, size_t src_bytes, int bytes, int iters, int mode, int L,
                          unsigned long long* cyc) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ __align__(8) uint64_t bar[S];
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[s])));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    const int lane = threadIdx.x;
    if (lane >= (mode == 3 ? L : 1)) return;
    const size_t nblk = src_bytes / bytes;
    long long t0 = clock64();
    const int step = (mode == 3) ? L : 1;
    for (int i0 = 0; i0 < iters; i0 += step) {
        const int i = i0 + (mode == 3 ? lane : 0);
        const int s = i % S;
        if ((mode == 0 || mode == 3) && i >= S) {
            const uint32_t ph = ((i - S) / S) & 1;
            uint32_t ok = 0;
            while (!ok)
                asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                             : "=r"(ok) : "r"(su32(&bar[s])), "r"(ph) : "memory");
        }
        const uint8_t* g = src + ((size_t)(blockIdx.x * 7919 + i * 131) % nblk) * bytes;
        if (mode != 2)
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[s])), "r"(bytes) : "memory");
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                     ::"r"(su32(sm + (size_t)s * bytes)), "l"(g), "r"(bytes), "r"(su32(&bar[s])) : "memory");
        if (mode == 1 && (i % S) == S - 1) {   // drain every S iterations
            for (int k = 0; k < S; ++k) {
                const uint32_t ph = (i / S) & 1;
                uint32_t ok = 0;
                while (!ok)
                    asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                                 : "=r"(ok) : "r"(su32(&bar[k])), "r"(ph) : "memory");
            }
        }
    }
    if (lane == 0) cyc[blockIdx.x] = clock64() - t0;
}

int main1() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    size_t src_bytes = 32u << 20;   // 32 MiB: L2 resident
    uint8_t* src;
    cudaMalloc(&src, src_bytes);
    cudaMemset(src, 1, src_bytes);
    unsigned long long* cyc;
    cudaMalloc(&cyc, nsm * sizeof(unsigned long long));
    auto run = [&](auto kern, int S, int bytes) {
        const int iters = 4000;
        size_t smem = (size_t)S * bytes;
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        kern<<<nsm, 32, smem>>>(src, src_bytes, bytes, iters, cyc);
        kern<<<nsm, 32, smem>>>(src, src_bytes, bytes, iters, cyc);
        cudaDeviceSynchronize();
        unsigned long long h[256];
        cudaMemcpy(h, cyc, nsm * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
        double avg = 0;
        for (int i = 0; i < nsm; ++i) avg += h[i];
        avg /= nsm;
        printf("ingest %6d B x %2d stages, grid %3d: %.0f clk/iter, %.1f B/clk/SM (%s)\n", bytes, S, nsm, avg / iters,
               (double)bytes * iters / avg, cudaGetErrorString(cudaGetLastError()));
    };
    auto runv = [&](int mode, int L, int bytes) {
        const int iters = 4096, S = 8;
        size_t smem = (size_t)S * bytes;
        cudaFuncSetAttribute(k_variant<8>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        k_variant<8><<<nsm, 32, smem>>>(src, src_bytes, bytes, iters, mode, L, cyc);
        k_variant<8><<<nsm, 32, smem>>>(src, src_bytes, bytes, iters, mode, L, cyc);
        cudaDeviceSynchronize();
        unsigned long long h[256];
        cudaMemcpy(h, cyc, nsm * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
        double avg = 0;
        for (int i = 0; i < nsm; ++i) avg += h[i];
        avg /= nsm;
        printf("variant mode=%d lanes=%d %6d B: %.0f clk/copy, %.1f B/clk/SM (%s)\n", mode, L, bytes, avg / iters,
               (double)bytes * iters / avg, cudaGetErrorString(cudaGetLastError()));
    };
    for (int bytes : {4096, 16384}) {
        runv(0, 1, bytes);
        runv(1, 1, bytes);
        runv(2, 1, bytes);
        runv(3, 2, bytes);
        runv(3, 4, bytes);
        runv(3, 8, bytes);
    }
    return 0;
}

// ---- kernel-like pattern: per step 4 copies (16 KiB, 4 KiB, 256 B, 256 B) into one stage, S stages ----
template <int S>
__global__ void k_pattern(const uint8_t* src, size_t src_bytes, int iters, int ncopies, unsigned long long* cyc,
                          int align_a, int stage_bytes, int src_mode) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ __align__(8) uint64_t bar[S];
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[s])));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    if (threadIdx.x != 0) return;
    const int sizes[4] = {16384, 4096, 256, 256};
    const int offs[4] = {0, 16384, 20480, 20736};
    int tx = 0;
    for (int c = 0; c < ncopies; ++c) tx += sizes[c];
    long long t0 = clock64();
    for (int i = 0; i < iters + S; ++i) {
        const int s = i % S;
        if (i >= S) {
            const uint32_t ph = ((i - S) / S) & 1;
            uint32_t ok = 0;
            while (!ok)
                asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                             : "=r"(ok) : "r"(su32(&bar[s])), "r"(ph) : "memory");
        }
        if (i < iters) {
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[s])), "r"(tx) : "memory");
            for (int c = 0; c < ncopies; ++c) {
                size_t off = ((size_t)(blockIdx.x * 7919 + i * 131 + c * 17) * 256) % (src_bytes - 16384);
                if (src_mode == 1) off = ((size_t)(blockIdx.x * 7919 + i * 131) % (src_bytes / 16384 - 1)) * 16384;
                if (c == 0) off = off / align_a * align_a;     // alignment of the big (A) copy
                const uint8_t* g = src + off;
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                             ::"r"(su32(sm + (size_t)s * stage_bytes + offs[c])), "l"(g), "r"(sizes[c]), "r"(su32(&bar[s])) : "memory");
            }
        }
    }
    cyc[blockIdx.x] = clock64() - t0;
}

int main2() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    size_t src_bytes = 32u << 20;
    uint8_t* src;
    cudaMalloc(&src, src_bytes);
    cudaMemset(src, 1, src_bytes);
    unsigned long long* cyc;
    cudaMalloc(&cyc, nsm * sizeof(unsigned long long));
    const int iters = 4000;
    for (int sm_mode : {1})
    for (int sb : {16384, 21504})
    for (int nc : {1}) {
        auto run = [&](auto kern, int S) {
            size_t smem = (size_t)S * sb;
            if (smem > 227 * 1024 || (nc > 1 && sb < 21504)) return;
            cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
            kern<<<nsm, 32, smem>>>(src, src_bytes, iters, nc, cyc, 256, sb, sm_mode);
            kern<<<nsm, 32, smem>>>(src, src_bytes, iters, nc, cyc, 256, sb, sm_mode);
            cudaDeviceSynchronize();
            unsigned long long h[256];
            cudaMemcpy(h, cyc, nsm * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
            double avg = 0;
            for (int i = 0; i < nsm; ++i) avg += h[i];
            avg /= nsm;
            printf("pattern srcmode=%d stage_bytes=%5d copies=%d stages=%d: %.0f clk/step (%s)\n", sm_mode, sb, nc, S, avg / iters, cudaGetErrorString(cudaGetLastError()));
        };
        run(k_pattern<4>, 4);
        run(k_pattern<6>, 6);
    }
    return 0;
}
int main() { main1(); return 0; }
