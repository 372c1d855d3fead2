// Microbenchmark: issue cost of cp.async.bulk (global -> shared) from one thread vs several warps.
// Thread(s) issue C copies of B bytes back-to-back onto one mbarrier (expect_tx once), then wait.
// Reports issue clocks per copy (clock64 around the issue loop) and total clocks to completion.
// Source offsets use a power-of-two mask (no 64-bit modulo in the loop).  1 CTA per SM, all SMs.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o probe_tma2 probe_tma2.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void wait_bar(uint64_t* bar, uint32_t ph) {
    uint32_t ok = 0;
    while (!ok)
        asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                     : "=r"(ok) : "r"(su32(bar)), "r"(ph) : "memory");
}

// W issuing warps (lane 0 of each), each issues C/W copies per round; R rounds (alternating 2 barriers)
__global__ void k_issue(const uint8_t* src, uint64_t mask, int bytes, int C, int W, int R, int cta_dst,
                        unsigned long long* out) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ __align__(8) uint64_t bar[2];
    __shared__ unsigned long long s_issue[32];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(&bar[0])), "r"(W));
        asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(&bar[1])), "r"(W));
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    __syncthreads();
    unsigned long long issue = 0;
    long long t0 = clock64();
    if (lane == 0 && warp < W) {
        const int per = C / W;
        for (int r = 0; r < R; ++r) {
            uint64_t* b = &bar[r & 1];
            if (r >= 2) wait_bar(b, ((r - 2) >> 1) & 1);
            const long long a = clock64();
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(b)), "r"(per * bytes) : "memory");
            for (int c = 0; c < per; ++c) {
                const int slot = (r & 1) * C + warp * per + c;
                const uint64_t off = ((uint64_t)(blockIdx.x * 7919 + (r * C + warp * per + c) * 131) * bytes) & mask;
                if (cta_dst)
                    asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                                 ::"r"(su32(sm + (size_t)slot * bytes)), "l"(src + off), "r"(bytes), "r"(su32(b)) : "memory");
                else
                    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                                 ::"r"(su32(sm + (size_t)slot * bytes)), "l"(src + off), "r"(bytes), "r"(su32(b)) : "memory");
            }
            issue += clock64() - a;
        }
        wait_bar(&bar[(R - 1) & 1], ((R - 1) >> 1) & 1);
        if (R >= 2) wait_bar(&bar[(R - 2) & 1], ((R - 2) >> 1) & 1);
        s_issue[warp] = issue;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long mx = 0;
        for (int w = 0; w < W; ++w) mx = s_issue[w] > mx ? s_issue[w] : mx;
        out[2 * blockIdx.x] = mx;
        out[2 * blockIdx.x + 1] = clock64() - t0;
    }
}

int main() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    const size_t src_bytes = 64u << 20;   // 64 MiB: L2 resident
    uint8_t* src;
    cudaMalloc(&src, src_bytes);
    cudaMemset(src, 1, src_bytes);
    unsigned long long* out;
    cudaMalloc(&out, 2 * nsm * sizeof(unsigned long long));
    auto run = [&](int bytes, int C, int W, int R, int cta_dst, int grid) {
        const size_t smem = (size_t)2 * C * bytes;
        if (smem > 200 * 1024) return;
        cudaFuncSetAttribute(k_issue, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        const uint64_t mask = (src_bytes - 1) & ~(uint64_t)(bytes - 1) & ~(uint64_t)127;
        k_issue<<<grid, 32 * (W > 1 ? W : 1), smem>>>(src, mask, bytes, C, W, R, cta_dst, out);
        k_issue<<<grid, 32 * (W > 1 ? W : 1), smem>>>(src, mask, bytes, C, W, R, cta_dst, out);
        cudaDeviceSynchronize();
        unsigned long long h[512];
        cudaMemcpy(h, out, 2 * grid * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
        double is = 0, tot = 0;
        for (int i = 0; i < grid; ++i) is += h[2 * i], tot += h[2 * i + 1];
        is /= grid, tot /= grid;
        printf("bytes %6d copies/round %2d warps %d dst %s grid %3d: issue %.0f clk/copy, total %.0f clk/copy, %.1f B/clk/SM (%s)\n",
               bytes, C, W, cta_dst ? "cta    " : "cluster", grid, is / ((double)R * C / W), tot / ((double)R * C),
               (double)bytes * R * C / tot, cudaGetErrorString(cudaGetLastError()));
    };
    const int R = 400;
    for (int grid : {1, nsm}) {
        for (int bytes : {256, 2048, 4096, 16384}) {
            run(bytes, 1, 1, R, 0, grid);
            run(bytes, 4, 1, R, 0, grid);
            run(bytes, 4, 1, R, 1, grid);
            run(bytes, 4, 4, R, 0, grid);
        }
    }
    return 0;
}
