// k_quad_lop3.cu — CUDA-core contraction (EPI4_PIPE_LOP3): AND + POPC on bit planes.
//
// The cross-check pipe of SURVEY.md §8(a) a5: for each tile (64-SNP half wr of a unit's w-range, x,
// y-range y0, z) the 64 x 16
// (w, y) combinations are counted directly: for each 32-sample word, the pair rows
// (w,x,a,b) = P_a(w) & P_b(x) ("combine") are ANDed with the pair columns
// (y,z,c,d) and popcounted (3 ANDs + POPC per sample and genotype).  This is the
// computation the paper maps to binary tensor-core GEMMs; on sm_100a there is
// no native b1 tensor op, so this pipe runs on the integer ALUs.  The fused
// epilogue (epilogue.cuh) recovers the aa cells, scores K2 and updates the CTA's top-k list.
//
// CTA = 256 threads; thread (i = tid%64, jg = tid/64) owns quads (64wr+i, x, y0+jg+4m, z), m<4.
#include "epilogue.cuh"

namespace epi4 {

constexpr int LOP3_THREADS = 256;
constexpr int LOP3_Q = 4;   // quads per thread per tile

__global__ void __launch_bounds__(LOP3_THREADS, 1) k_quad_lop3(SearchParams sp) {
    extern __shared__ __align__(16) unsigned char smem[];
    // [0, 128 KiB): per-thread contraction counts staged for the epilogue: cnt[c][tid]
    uint32_t* s_cnt = reinterpret_cast<uint32_t*>(smem);
    TopKSmem tk = topk_carve(smem + sizeof(uint32_t) * 2 * LOP3_Q * 16 * LOP3_THREADS, sp.topk);
    __shared__ long long s_tile;
    const int tid = threadIdx.x;
    topk_load(tk, sp, blockIdx.x, tid, LOP3_THREADS);
    __syncthreads();
    const DevData& d = sp.d;
    unsigned long long my_quads = 0;
    // top_k <= 32: race-free per-warp register lists (epilogue.cuh WarpList), else the CTA's locked list
    const bool wlist = use_warp_lists(sp.topk);
    WarpList wlst;
    wl_init(wlst);
    if (wlist && tid < 32) wl_load(wlst, sp, blockIdx.x);
    double wthr = wlist ? wl_thr(wlst, sp.topk) : 0.0;

    for (;;) {
        if (tid == 0) s_tile = (long long)atomicAdd(sp.tile_counter, 1ull);
        __syncthreads();
        const long long tile = s_tile;
        __syncthreads();
        if (tile >= sp.ntiles) break;
        const int64_t u = find_unit(sp.prefix, sp.nunits, tile);
        const int64_t t = tile - (u ? sp.prefix[u - 1] : 0);   // = 2 * unit tile + half
        const int32_t wr = sp.units[u].wr * 2 + (int32_t)(t & 1), x = sp.units[u].x;
        int32_t y0, z;
        unit_tile_decode(d.n, x, t >> 1, y0, z, EPI4_YR);
        const int i = tid & 63, jg = tid >> 6;
        const int w = wr * EPI4_WR + i;

        uint32_t cnt[2][LOP3_Q][16];
#pragma unroll
        for (int p = 0; p < 2; ++p)
#pragma unroll
            for (int m = 0; m < LOP3_Q; ++m)
#pragma unroll
                for (int c = 0; c < 16; ++c) cnt[p][m][c] = 0;

#pragma unroll
        for (int p = 0; p < 2; ++p) {
            const uint32_t* P = d.planes[p];
            const int nch = d.nchunks[p];
            for (int kc = 0; kc < nch; ++kc) {
                const uint4 w0 = __ldg(reinterpret_cast<const uint4*>(P + plane_off(kc, d.npad, w, 0, 0)));
                const uint4 w1 = __ldg(reinterpret_cast<const uint4*>(P + plane_off(kc, d.npad, w, 1, 0)));
                const uint4 x0 = __ldg(reinterpret_cast<const uint4*>(P + plane_off(kc, d.npad, x, 0, 0)));
                const uint4 x1 = __ldg(reinterpret_cast<const uint4*>(P + plane_off(kc, d.npad, x, 1, 0)));
                const uint4 z0 = __ldg(reinterpret_cast<const uint4*>(P + plane_off(kc, d.npad, z, 0, 0)));
                const uint4 z1 = __ldg(reinterpret_cast<const uint4*>(P + plane_off(kc, d.npad, z, 1, 0)));
                const uint32_t wv[2][4] = {{w0.x, w0.y, w0.z, w0.w}, {w1.x, w1.y, w1.z, w1.w}};
                const uint32_t xv[2][4] = {{x0.x, x0.y, x0.z, x0.w}, {x1.x, x1.y, x1.z, x1.w}};
                const uint32_t zv[2][4] = {{z0.x, z0.y, z0.z, z0.w}, {z1.x, z1.y, z1.z, z1.w}};
#pragma unroll
                for (int m = 0; m < LOP3_Q; ++m) {
                    const int y = y0 + jg + 4 * m;
                    const uint4 ya = __ldg(reinterpret_cast<const uint4*>(P + plane_off(kc, d.npad, y, 0, 0)));
                    const uint4 yb = __ldg(reinterpret_cast<const uint4*>(P + plane_off(kc, d.npad, y, 1, 0)));
                    const uint32_t yv[2][4] = {{ya.x, ya.y, ya.z, ya.w}, {yb.x, yb.y, yb.z, yb.w}};
#pragma unroll
                    for (int wd = 0; wd < 4; ++wd) {
                        uint32_t wx[4], yz[4];
#pragma unroll
                        for (int a = 0; a < 2; ++a)
#pragma unroll
                            for (int b = 0; b < 2; ++b) {
                                wx[a * 2 + b] = wv[a][wd] & xv[b][wd];
                                yz[a * 2 + b] = yv[a][wd] & zv[b][wd];
                            }
#pragma unroll
                        for (int ab = 0; ab < 4; ++ab)
#pragma unroll
                            for (int cd = 0; cd < 4; ++cd) cnt[p][m][ab * 4 + cd] += __popc(wx[ab] & yz[cd]);
                    }
                }
            }
        }
        // stage the counts so the epilogue's register budget is free
#pragma unroll
        for (int p = 0; p < 2; ++p)
#pragma unroll
            for (int m = 0; m < LOP3_Q; ++m)
#pragma unroll
                for (int c = 0; c < 16; ++c) s_cnt[((p * LOP3_Q + m) * 16 + c) * LOP3_THREADS + tid] = cnt[p][m][c];

        for (int m = 0; m < LOP3_Q; ++m) {
            const int y = y0 + jg + 4 * m;
            const bool valid = (w < x) && (y > x) && (y < z);
            double key = 0.0;
            uint64_t idx = 0;
            if (valid) {
                uint32_t c0[16], c1[16];
#pragma unroll
                for (int c = 0; c < 16; ++c) {
                    c0[c] = s_cnt[((0 * LOP3_Q + m) * 16 + c) * LOP3_THREADS + tid];
                    c1[c] = s_cnt[((1 * LOP3_Q + m) * 16 + c) * LOP3_THREADS + tid];
                }
                uint32_t* dump = sp.dump ? sp.dump + rank4(w, x, y, z) * 162 : nullptr;
                auto eval = [&](auto tag) {
                    using P = decltype(tag);
                    P c16[16];
                    pack16<P>(d, c0, c1, c16);
                    if (!dump && sample_hit(sp, pack_quad(w, x, y, z))) return sample_record<P>(sp, w, x, y, z, c16);
                    double k = score_quad<P>(d, w, x, y, z, c16, dump);
                    if (dump && d.objective != EPI4_OBJ_K2) k = score_quad<P>(d, w, x, y, z, c16, nullptr);
                    return k;
                };
                key = d.wide ? eval(uint64_t{}) : eval(uint32_t{});
                idx = pack_quad(w, x, y, z);
                ++my_quads;
            }
            if (wlist) wl_offer(wlst, sp.topk, wthr, valid, key, idx);
            else warp_offer(tk, valid, key, idx);
        }
    }
    __syncthreads();
    if (wlist) wl_merge_store(wlst, sp.topk, tid >> 5, LOP3_THREADS / 32, 1, tk.stage_k, tk.stage_i, sp, blockIdx.x);
    else topk_store(tk, sp, blockIdx.x, tid, LOP3_THREADS);
    // useful-quad counter
    unsigned long long v = my_quads;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if ((tid & 31) == 0) atomicAdd(sp.quads_done, v);
}

cudaError_t launch_quad_lop3(const SearchParams& sp, int32_t grid, cudaStream_t s, int64_t* launches) {
    const size_t smem = sizeof(uint32_t) * 2 * LOP3_Q * 16 * LOP3_THREADS + topk_smem_bytes(sp.topk);
    cudaError_t e = cudaFuncSetAttribute(k_quad_lop3, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    k_quad_lop3<<<grid, LOP3_THREADS, smem, s>>>(sp);
    if (launches) ++*launches;
    return cudaGetLastError();
}

}  // namespace epi4
