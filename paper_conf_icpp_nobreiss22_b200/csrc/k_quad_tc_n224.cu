// k_quad_tc_n224.cu — the tensor-core contraction kernel (k_quad_tc.cuh) in its N = 224 geometry (large sample
// counts), a translation unit of its own so that the two geometries compile in parallel.
#include "k_quad_tc.cuh"

namespace epi4 {
template cudaError_t launch_quad_tc_geom<Geom224>(const SearchParams&, int32_t, cudaStream_t, int64_t*);
}  // namespace epi4
