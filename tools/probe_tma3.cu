// Probe: chip-wide TMA bulk-copy ingest (global -> shared, L2-resident source like the A operand of
// k_quad_tc: a ~9 MB array re-read by every SM), S stages of 16 KiB per CTA, 1 CTA per SM.
//   mode 0: every CTA copies whole 16 KiB blocks (no multicast)
//   mode 1: clusters of 2; each CTA issues one 8 KiB half of the block multicast to both CTAs
//   mode 2: clusters of 4 (2 x 2): each CTA issues a quarter... here: 8 KiB half multicast to CTA r and r^2
//           (the layout a 2-pair cluster would use), i.e. L2 reads halved, each CTA still ingests 16 KiB
// Reports per-SM ingest (B/clk/SM, bytes landed in this CTA's smem) and the implied latency S*16K / rate.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o probe_tma3 probe_tma3.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint32_t cta_rank() { uint32_t r; asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r)); return r; }
__device__ __forceinline__ uint32_t hash32(uint32_t x) {
    x ^= x >> 16; x *= 0x7feb352du; x ^= x >> 15; x *= 0x846ca68bu; x ^= x >> 16;
    return x;
}

template <int S, int MODE, int BLK>
__global__ void k_tma(const uint8_t* src, int nblk, int iters, unsigned long long* cyc) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ __align__(8) uint64_t full[S], empty[S];
    const uint32_t r = MODE ? cta_rank() : 0;
    const int csize = MODE == 0 ? 1 : MODE == 1 ? 2 : 4;
    if (threadIdx.x == 0) {
        for (int s = 0; s < S; ++s) {
            asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&full[s])));
            asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(&empty[s])), "r"(MODE == 0 ? 1 : 2));
        }
        asm volatile("fence.mbarrier_init.release.cluster;");
    }
    if (MODE) asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    else __syncthreads();
    const int cl = blockIdx.x / csize;
    // multicast partner set: mode 1: {0,1}; mode 2: {r&1, (r&1)+2}
    const uint16_t mask = MODE == 1 ? (uint16_t)3 : (uint16_t)((1u << (r & 1)) | (1u << ((r & 1) + 2)));
    const uint32_t piece = MODE == 1 ? r : (r >> 1);    // which 8 KiB half this CTA issues
    long long t0 = 0;
    if (threadIdx.x == 0) {
        t0 = clock64();
        for (int i = 0; i < iters; ++i) {
            const int s = i % S;
            const uint32_t ph = (i / S) & 1;
            // wait until the slot is free in every destination CTA (their consumer arrived on our empty[s])
            if (i >= S) {
                uint32_t ok = 0;
                while (!ok)
                    asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                                 : "=r"(ok) : "r"(su32(&empty[s])), "r"(ph ^ 1) : "memory");
            }
            // the block this cluster reads at step i (same for all CTAs of a cluster; pairs (r, r^2) share it in mode 2)
            const uint32_t grp = MODE == 2 ? (uint32_t)cl * 2 + (r & 1) : (uint32_t)cl;
            const int blk = (int)(hash32(grp * 7919u + (uint32_t)i) % (uint32_t)nblk);
            const uint8_t* g = src + (size_t)blk * BLK;
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&full[s])), "r"(BLK) : "memory");
            if (MODE == 0) {
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                             ::"r"(su32(sm + s * BLK)), "l"(g), "r"(BLK), "r"(su32(&full[s])) : "memory");
            } else {
                asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.multicast::cluster [%0], [%1], %2, [%3], %4;"
                             ::"r"(su32(sm + s * BLK + piece * (BLK / 2))), "l"(g + piece * (BLK / 2)), "r"(BLK / 2),
                             "r"(su32(&full[s])), "h"(mask) : "memory");
            }
            // consume: wait for the data, then release the slot in every CTA that writes into ours
            uint32_t ok = 0;
            const int j = i - (S - 1);   // consume with a lag of S-1 (keeps S copies in flight)
            if (j >= 0) {
                const int sj = j % S;
                const uint32_t phj = (j / S) & 1;
                while (!ok)
                    asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                                 : "=r"(ok) : "r"(su32(&full[sj])), "r"(phj) : "memory");
                if (MODE == 0) {
                    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(&empty[sj])) : "memory");
                } else {
                    // our slot is written by ourselves and by the partner: release it in both
                    const uint32_t partner = MODE == 1 ? (r ^ 1) : (r ^ 2);
                    for (uint32_t t : {r, partner}) {
                        uint32_t remote;
                        asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(su32(&empty[sj])), "r"(t));
                        asm volatile("mbarrier.arrive.shared::cluster.b64 _, [%0];" ::"r"(remote) : "memory");
                    }
                }
            }
        }
        // drain
        for (int j = iters - (S - 1); j < iters; ++j) {
            if (j < 0) continue;
            const int sj = j % S;
            const uint32_t phj = (j / S) & 1;
            uint32_t ok = 0;
            while (!ok)
                asm volatile("{.reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p;}"
                             : "=r"(ok) : "r"(su32(&full[sj])), "r"(phj) : "memory");
        }
        cyc[blockIdx.x] = clock64() - t0;
    }
    if (MODE) asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

template <int S, int MODE, int BLK>
void run(const uint8_t* src, int nblk, unsigned long long* cyc, int nsm) {
    auto k = k_tma<S, MODE, BLK>;
    const size_t smem = (size_t)S * BLK;
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    const int csize = MODE == 0 ? 1 : MODE == 1 ? 2 : 4;
    const int grid = nsm / csize * csize;
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(32);
    cfg.dynamicSmemBytes = smem;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = csize;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    const int iters = 4000;
    cudaLaunchKernelEx(&cfg, k, src, nblk, iters, cyc);
    cudaError_t e = cudaDeviceSynchronize();
    unsigned long long h[256];
    cudaMemcpy(h, cyc, grid * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
    double avg = 0;
    for (int i = 0; i < grid; ++i) avg += h[i];
    avg /= grid;
    const double bpc = (double)iters * BLK / avg;
    printf("blk %5d mode %d S=%2d grid %3d src %5.1f MB: %5.1f B/clk/SM ingest, L2 reads %5.1f B/clk/SM, latency ~%5.0f clk (%s)\n",
           BLK, MODE, S, grid, nblk * (double)BLK / 1e6, bpc, MODE == 0 ? bpc : bpc / 2, S * BLK / bpc, cudaGetErrorString(e));
}

int main() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    uint8_t* src;
    const size_t bytes = 9437184;   // 9.4 MB, like expl at C2
    cudaMalloc(&src, bytes);
    cudaMemset(src, 1, bytes);
    unsigned long long* cyc;
    cudaMalloc(&cyc, 256 * sizeof(unsigned long long));
    run<4, 0, 16384>(src, bytes / 16384, cyc, nsm);
    run<8, 0, 16384>(src, bytes / 16384, cyc, nsm);
    run<2, 0, 32768>(src, bytes / 32768, cyc, nsm);
    run<4, 0, 32768>(src, bytes / 32768, cyc, nsm);
    run<6, 0, 32768>(src, bytes / 32768, cyc, nsm);
    run<2, 0, 65536>(src, bytes / 65536, cyc, nsm);
    run<3, 0, 65536>(src, bytes / 65536, cyc, nsm);
    run<4, 1, 32768>(src, bytes / 32768, cyc, nsm);
    run<4, 2, 32768>(src, bytes / 32768, cyc, nsm);
    run<6, 1, 32768>(src, bytes / 32768, cyc, nsm);
    run<6, 2, 32768>(src, bytes / 32768, cyc, nsm);
    // a 64 MB source (less reuse across SMs)
    uint8_t* big;
    const size_t bbytes = (size_t)64 << 20;
    cudaMalloc(&big, bbytes);
    cudaMemset(big, 1, bbytes);
    run<4, 0, 32768>(big, bbytes / 32768, cyc, nsm);
    run<6, 0, 32768>(big, bbytes / 32768, cyc, nsm);
    run<4, 1, 32768>(big, bbytes / 32768, cyc, nsm);
    run<4, 2, 32768>(big, bbytes / 32768, cyc, nsm);
    return 0;
}
