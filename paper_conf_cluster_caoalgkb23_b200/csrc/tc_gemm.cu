// Placeholder until the tcgen05 kernels land: reports "unavailable" so the engine uses the
// DMMA path (FP64 arithmetic on operands rounded to the class precision).
#include "tc_gemm.h"
namespace mpgeo {
bool tc_gemm_available() { return false; }
cudaError_t tc_gemm_tf32x3_launch(const TcArgs&, int, cudaStream_t) { return cudaErrorNotSupported; }
cudaError_t tc_gemm_f16_launch(const TcArgs&, int, cudaStream_t) { return cudaErrorNotSupported; }
}  // namespace mpgeo
