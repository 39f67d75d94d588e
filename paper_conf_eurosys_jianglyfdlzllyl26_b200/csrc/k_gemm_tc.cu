// tcgen05 GEMM (placeholder).
#include "kernels.h"
namespace fps {
bool gemm_tc_supported(int dtype, int M, int N, int K) { (void)dtype; (void)M; (void)N; (void)K; return false; }
fps_status launch_gemm_tc(const void*, const void*, int, int, int, const Epilogue&, cudaStream_t) {
  return fail(FPS_EUNSUPPORTED, "gemm_tc not built");
}
}  // namespace fps
