// k_quad_tc.cu — the tensor-core contraction kernel (k_quad_tc.cuh) in its N = 128 geometry, the tile table,
// and the geometry dispatch (the N = 224 instantiation is compiled in parallel in k_quad_tc_n224.cu).
#include "k_quad_tc.cuh"

namespace epi4 {

extern template cudaError_t launch_quad_tc_geom<Geom224>(const SearchParams&, int32_t, cudaStream_t, int64_t*);
template cudaError_t launch_quad_tc_geom<Geom128>(const SearchParams&, int32_t, cudaStream_t, int64_t*);

// The tile table (one uint64 per tile, filled by k_tile_table before the search): a tile change in the hot
// kernel costs one load instead of decode_tile's binary search over the unit prefix (~log2(units) dependent
// global loads) and the y-range loop, which stalled the TMA / producer / epilogue warps at every tile change.
// tiles [t0, t1) of the launch's units (one launch per chunk of at most epi4_ctx::tile_chunk tiles)
__global__ void __launch_bounds__(256) k_tile_table(SearchParams sp, int64_t t0, int64_t t1, uint64_t* __restrict__ out) {
    const int64_t t = t0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= t1) return;
    const TileInfo ti = decode_tile(sp, t);
    out[t - t0] = (uint64_t)(uint16_t)ti.wp | ((uint64_t)(uint16_t)ti.x << 16) | ((uint64_t)(uint16_t)ti.y0 << 32) |
                  ((uint64_t)(uint16_t)ti.z << 48);
}
cudaError_t launch_tile_table(const SearchParams& sp, int64_t t0, int64_t t1, uint64_t* out, cudaStream_t s,
                              int64_t* launches) {
    if (t1 <= t0) return cudaSuccess;
    k_tile_table<<<(unsigned)((t1 - t0 + 255) / 256), 256, 0, s>>>(sp, t0, t1, out);
    if (launches) ++*launches;
    return cudaGetLastError();
}
// tiles per unit tile: the tensor-core kernel pairs the two 64-SNP halves of a 128-SNP w-range in one
// cluster (1 tile); the CUDA-core kernel processes them as 2 tiles
int32_t quad_split(int32_t pipe) { return pipe == EPI4_PIPE_LOP3 ? 2 : 1; }

// sp.yr selects the geometry (api.cu tc_tile_yr)
cudaError_t launch_quad_tc(const SearchParams& sp, int32_t grid, cudaStream_t s, int64_t* launches) {
    if (sp.yr == Geom224::YR) return launch_quad_tc_geom<Geom224>(sp, grid, s, launches);
    if (sp.yr == Geom128::YR) return launch_quad_tc_geom<Geom128>(sp, grid, s, launches);
    return cudaErrorInvalidValue;
}

}  // namespace epi4
