// GAT layer (placeholder: implemented in a later milestone).
#include "plan.h"
namespace wg {
void gat_layout(wg_plan_s* p) { p->saved = Layout(); p->ws = Layout(); }
wg_status gat_forward(wg_plan_s*, const wg_params*, const wg_fwd_args*, cudaStream_t) {
  set_error("GAT not implemented yet"); return WG_ERR_UNSUPPORTED;
}
wg_status gat_backward(wg_plan_s*, const wg_params*, const wg_bwd_args*, const wg_grads*, cudaStream_t) {
  set_error("GAT not implemented yet"); return WG_ERR_UNSUPPORTED;
}
}  // namespace wg
