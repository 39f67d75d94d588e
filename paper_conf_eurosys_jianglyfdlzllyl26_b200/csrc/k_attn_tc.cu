// Tensor-core varlen merged-key attention (placeholder until the tcgen05 kernel lands).
#include "kernels.h"
namespace fps {
bool attention_tc_supported(int dtype, int head_dim) { (void)dtype; (void)head_dim; return false; }
fps_status launch_attention_tc(const void*, const void*, void*, int, int, const int32_t*,
                               const int32_t*, const int32_t*, int, int, cudaStream_t) {
  return fail(FPS_EUNSUPPORTED, "attention_tc not built");
}
}  // namespace fps
