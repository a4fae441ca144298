// RGCN layer (placeholder: implemented in a later milestone).
#include "plan.h"
namespace wg {
wg_status rgcn_plan(wg_plan_s*, cudaStream_t) { set_error("RGCN not implemented yet"); return WG_ERR_UNSUPPORTED; }
void rgcn_plan_free(wg_plan_s*) {}
wg_status rgcn_forward(wg_plan_s*, const wg_params*, const wg_fwd_args*, cudaStream_t) { return WG_ERR_UNSUPPORTED; }
wg_status rgcn_backward(wg_plan_s*, const wg_params*, const wg_bwd_args*, const wg_grads*, cudaStream_t) {
  return WG_ERR_UNSUPPORTED;
}
}  // namespace wg
