// Probe: 2-CTA tcgen05.mma kind::mxf4 rate vs N, and its sensitivity to concurrent shared-memory traffic
// from other warps of the same CTA (LDS.128 / STS.128 streams), i.e. whether the tensor core's operand reads
// share the SM's shared-memory bandwidth with the producers / epilogue.
//   mode 0: MMA only;  mode 1: + 8 warps LDS.128 stream;  mode 2: + 8 warps STS.128 stream;
//   mode 3: + 8 warps random 4-byte LDS gathers (the epilogue's table-lookup pattern)
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o probe_mxf4b probe_mxf4b.cu
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

constexpr int TRAFFIC_BYTES = 32768;

template <int N>
__global__ void __cluster_dims__(2, 1, 1) __launch_bounds__(320, 1)
k_rate(int iters, int mode, unsigned long long* out /*[grid/2][4]*/) {
    extern __shared__ __align__(1024) uint8_t sm_raw[];
    __shared__ uint32_t s_tmem;
    __shared__ __align__(8) uint64_t bar;
    __shared__ volatile int s_done;
    const uint32_t raw = su32(sm_raw);
    uint8_t* sm = sm_raw + (((raw + 1023u) & ~1023u) - raw);
    uint8_t* A = sm;                      // 128 rows x 128 B
    uint8_t* B = sm + 16384;              // up to 128 rows x 128 B
    uint8_t* T = sm + 32768;              // traffic buffer
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    uint32_t rank;
    asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(rank));
    for (int i = threadIdx.x; i < (32768 + TRAFFIC_BYTES) / 4; i += blockDim.x)
        reinterpret_cast<uint32_t*>(sm)[i] = (i * 2654435761u) & 0x22222222u;
    if (threadIdx.x == 0) {
        s_done = 0;
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
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
    const uint32_t idesc = (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | (1u << 23) | (16u << 24);
    const uint64_t ad0 = sw128_desc(su32(A)), bd0 = sw128_desc(su32(B));
    const uint32_t sf = tmem + 480;
    unsigned long long traffic_ops = 0;
    long long t_mma = 0;
    if (warp == 0) {
        if (lane == 0 && rank == 0) {
            const long long t0 = clock64();
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
            t_mma = clock64() - t0;
            s_done = 1;
        } else if (lane == 0) {
            wait_bar(&bar, 0);
            s_done = 1;
        }
    } else if (warp >= 2 && mode != 0) {
        // traffic warps: stream until the MMAs finish
        const int tw = warp - 2;
        uint4 acc = make_uint4(0, 0, 0, 0);
        uint32_t h = lane * 2654435761u + tw;
        while (!s_done) {
#pragma unroll 4
            for (int r = 0; r < 16; ++r) {
                if (mode == 1) {
                    const uint4 v = *reinterpret_cast<const uint4*>(T + ((tw * 16 + r) * 512 + lane * 16) % TRAFFIC_BYTES);
                    acc.x ^= v.x; acc.y += v.y; acc.z ^= v.z; acc.w += v.w;
                } else if (mode == 2) {
                    *reinterpret_cast<uint4*>(T + ((tw * 16 + r) * 512 + lane * 16) % TRAFFIC_BYTES) = make_uint4(h, r, tw, lane);
                } else {
                    h = h * 1664525u + 1013904223u;
                    acc.x += *reinterpret_cast<const uint32_t*>(T + ((h >> 8) & (TRAFFIC_BYTES / 4 - 1)) * 4);
                }
            }
            traffic_ops += 16;
        }
        if (acc.x == 0x12345 && acc.y == 7) out[0] = 1;   // keep the loads
    }
    __syncthreads();
    if (threadIdx.x == 0 && rank == 0) out[(blockIdx.x / 2) * 4 + 0] = t_mma;
    __shared__ unsigned long long s_ops;
    if (threadIdx.x == 0) s_ops = 0;
    __syncthreads();
    if (warp >= 2 && lane == 0) atomicAdd(&s_ops, traffic_ops);
    __syncthreads();
    if (threadIdx.x == 0 && rank == 0) out[(blockIdx.x / 2) * 4 + 1] = s_ops;
    asm volatile("tcgen05.fence::before_thread_sync;");
    asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
    asm volatile("tcgen05.fence::after_thread_sync;");
    if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(512));
}

int main() {
    int nsm = 0;
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
    unsigned long long* out;
    cudaMalloc(&out, nsm * 4 * sizeof(unsigned long long));
    const char* names[] = {"mma only", "+LDS.128 x8 warps", "+STS.128 x8 warps", "+LDS.32 random x8 warps"};
    auto run = [&](auto kern, int N, int mode) {
        const size_t smem = 32768 + TRAFFIC_BYTES + 2048;
        cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
        const int iters = 40000;
        kern<<<nsm / 2 * 2, 320, smem>>>(iters, mode, out);
        cudaError_t e = cudaDeviceSynchronize();
        unsigned long long h[1024];
        cudaMemcpy(h, out, nsm / 2 * 4 * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
        double cyc = 0, ops = 0;
        for (int i = 0; i < nsm / 2; ++i) { cyc += h[i * 4]; ops += h[i * 4 + 1]; }
        cyc /= nsm / 2;
        ops /= nsm / 2;
        const double clk_per_mma = cyc / iters;
        const double ideal = N / 2.0;   // 2-CTA fp4: 128 x N x 64 per SM at 16384 MAC/clk
        // traffic: warp-instructions per cycle on the leader CTA (x 512 B for .128)
        printf("N=%3d %-26s %6.1f clk/MMA (ideal %5.1f, %4.0f%%)  traffic %.3f warp-ops/clk  (%s)\n", N, names[mode],
               clk_per_mma, ideal, 100.0 * ideal / clk_per_mma, ops / cyc, cudaGetErrorString(e));
    };
    for (int mode = 0; mode < 4; ++mode) {
        run(k_rate<64>, 64, mode);
        run(k_rate<112>, 112, mode);
        run(k_rate<128>, 128, mode);
        run(k_rate<192>, 192, mode);
        run(k_rate<256>, 256, mode);
    }
    return 0;
}
