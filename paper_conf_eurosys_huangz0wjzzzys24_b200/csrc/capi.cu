// C-ABI glue: status strings, thread-local error text, launch counter and
// the forward / backward dispatch by model.
#include "plan.h"

namespace wg {
namespace {
thread_local std::string g_err;
thread_local int64_t g_launches = 0;
}  // namespace
void set_error(const std::string& msg) { g_err = msg; }
int64_t& launch_counter() { return g_launches; }

namespace {
struct ProfRec {
  int kind;
  cudaEvent_t a, b;
  double bytes, flops;
};
struct Profiler {
  bool on = false;
  std::vector<cudaEvent_t> pool;
  std::vector<ProfRec> recs;
  cudaEvent_t get() {
    if (!pool.empty()) { cudaEvent_t e = pool.back(); pool.pop_back(); return e; }
    cudaEvent_t e;
    cudaEventCreate(&e);
    return e;
  }
};
Profiler g_prof;
}  // namespace

ProfScope::ProfScope(int kind, cudaStream_t s, double bytes, double flops) : s_(s) {
  if (!g_prof.on) return;
  ProfRec r{kind, g_prof.get(), g_prof.get(), bytes, flops};
  cudaEventRecord(r.a, s);
  rec_ = (int)g_prof.recs.size();
  g_prof.recs.push_back(r);
}

ProfScope::~ProfScope() {
  if (rec_ >= 0 && rec_ < (int)g_prof.recs.size()) cudaEventRecord(g_prof.recs[rec_].b, s_);
}
}  // namespace wg

extern "C" {

const char* wg_status_string(wg_status s) {
  switch (s) {
    case WG_OK: return "ok";
    case WG_ERR_INVALID: return "invalid argument";
    case WG_ERR_RANGE: return "out of range";
    case WG_ERR_NOMEM: return "out of device memory";
    case WG_ERR_CUDA: return "CUDA error";
    case WG_ERR_UNSUPPORTED: return "unsupported";
    case WG_ERR_STATE: return "invalid state";
  }
  return "unknown status";
}

const char* wg_last_error(void) { return wg::g_err.c_str(); }

int64_t wg_launch_count(void) { return wg::launch_counter(); }

wg_status wg_profile(int cmd, double* out) {
  using namespace wg;
  if (cmd == 0 || cmd == 1) {
    for (auto& r : g_prof.recs) { cudaEventSynchronize(r.b); g_prof.pool.push_back(r.a); g_prof.pool.push_back(r.b); }
    g_prof.recs.clear();
    g_prof.on = cmd == 1;
    return WG_OK;
  }
  WG_REQ(cmd == 2 && out, WG_ERR_INVALID, "wg_profile: cmd must be 0, 1 or 2 (with out)");
  for (int i = 0; i < 4 * PK_KINDS; ++i) out[i] = 0.0;
  for (auto& r : g_prof.recs) {
    WG_CK(cudaEventSynchronize(r.b));
    float ms = 0.f;
    WG_CK(cudaEventElapsedTime(&ms, r.a, r.b));
    out[4 * r.kind + 0] += ms;
    out[4 * r.kind + 1] += 1;
    out[4 * r.kind + 2] += r.bytes;
    out[4 * r.kind + 3] += r.flops;
    g_prof.pool.push_back(r.a);
    g_prof.pool.push_back(r.b);
  }
  g_prof.recs.clear();
  return WG_OK;
}

wg_status wg_conv_forward(wg_plan p, const wg_params* params, const wg_fwd_args* a, wg_stream stream) {
  WG_REQ(p && params && a, WG_ERR_INVALID, "wg_conv_forward: null argument");
  WG_REQ(a->phase == WG_PHASE_ALL || a->phase == WG_PHASE_PRE || a->phase == WG_PHASE_POST, WG_ERR_INVALID,
         "wg_conv_forward: bad phase");
  WG_REQ(a->phase == WG_PHASE_ALL || (p->d.model != WG_GAT && p->d.model != WG_SAGE_LSTM), WG_ERR_UNSUPPORTED,
         "wg_conv_forward: PRE / POST phases are for GCN / SAGE / GIN / RGCN");
  WG_CK(cudaSetDevice(p->g->device));
  WG_CK(cudaGetLastError());
  cudaStream_t s = (cudaStream_t)stream;
  switch (p->d.model) {
    case WG_GCN: case WG_SAGE: case WG_GIN: return wg::lin_forward(p, params, a, s);
    case WG_GAT: return wg::gat_forward(p, params, a, s);
    case WG_RGCN: return wg::rgcn_forward(p, params, a, s);
    case WG_SAGE_LSTM: return wg::lstm_forward(p, params, a, s);
  }
  return WG_ERR_INVALID;
}

wg_status wg_conv_backward(wg_plan p, const wg_params* params, const wg_bwd_args* a, const wg_grads* grads,
                           wg_stream stream) {
  WG_REQ(p && params && a, WG_ERR_INVALID, "wg_conv_backward: null argument");
  WG_REQ(a->phase == WG_PHASE_ALL || a->phase == WG_PHASE_PRE || a->phase == WG_PHASE_POST, WG_ERR_INVALID,
         "wg_conv_backward: bad phase");
  WG_REQ(a->phase == WG_PHASE_ALL || (p->d.model != WG_GAT && p->d.model != WG_SAGE_LSTM), WG_ERR_UNSUPPORTED,
         "wg_conv_backward: PRE / POST phases are for GCN / SAGE / GIN / RGCN");
  WG_CK(cudaSetDevice(p->g->device));
  WG_CK(cudaGetLastError());
  cudaStream_t s = (cudaStream_t)stream;
  switch (p->d.model) {
    case WG_GCN: case WG_SAGE: case WG_GIN: return wg::lin_backward(p, params, a, grads, s);
    case WG_GAT: return wg::gat_backward(p, params, a, grads, s);
    case WG_RGCN: return wg::rgcn_backward(p, params, a, grads, s);
    case WG_SAGE_LSTM: return wg::lstm_backward(p, params, a, grads, s);
  }
  return WG_ERR_INVALID;
}

}  // extern "C"
