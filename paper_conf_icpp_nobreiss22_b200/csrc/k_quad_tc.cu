// k_quad_tc.cu — tcgen05 kind::i8 contraction (placeholder until the kernel lands).
#include "epilogue.cuh"

namespace epi4 {
int32_t quad_zt(int32_t pipe) { return pipe == EPI4_PIPE_LOP3 ? 1 : 1; }
cudaError_t launch_quad_i8tc(const SearchParams&, int32_t, cudaStream_t, int64_t*) { return cudaErrorNotSupported; }
}  // namespace epi4
