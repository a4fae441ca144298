// tcgen05 / TMEM / TMA GEMMs for sm_100a (placeholder until the tensor-core
// kernels land; returning false routes to the CUDA-core kernels).
#include "wg_internal.cuh"

namespace wg {
bool tc_gemm_nt(wg_dtype, int64_t, int, const GemmPart*, int, const GemmEpi&, cudaStream_t, wg_status*) {
  return false;
}
bool tc_gemm_tn(int64_t, int, int, const void*, int64_t, const void*, int64_t, float*, float*, cudaStream_t,
                wg_status*) {
  return false;
}
}  // namespace wg
