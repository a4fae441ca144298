// GraphSAGE with the LSTM aggregator -- the paper's fifth model, SAGE-LSTM
// (readings Q26 in DESIGN.md):
//   h_N(v) = LSTM over x[s_e], e in in(v) in edge-id order (H = f_in),
//   y[v]   = b + x[v] W_s + h_N(v) W_n.
//
// gTasks of uniq(dst-degree) = min & uniq(dst) = K: the
// destinations are ordered by decreasing in-degree, so at LSTM step t the
// rows still running (deg > t) are a PREFIX of that order -- step t is one
// dense batch of n_t rows.  Per step: one tcgen05 GEMM (3xTF32)
//   Z_t = [X_t | H_{t-1}] [W_ih ; W_hh] + b_l   (X_t gathered once, step-major)
// and one cell kernel (gate nonlinearities, c / h update).  The backward is
// the same walk reversed (BPTT): a cell-backward kernel per step and
// dH_{t-1} = dZ_t W_hh^T; dX = dZ W_ih^T, dW_ih = X^T dZ, dW_hh = H_prev^T dZ
// and db_l are single GEMMs / column sums over all steps; dx[u] gathers the
// per-edge dX rows over the transposed gTask partition (no atomics).
// fp32 (3xTF32 tensor cores); full graphs only.
#include <algorithm>

#include "plan.h"

namespace wg {

struct LstmPlan {
  int64_t T = 0, S = 0;                 // steps (max in-degree), step-major rows (padded)
  std::vector<int64_t> n, off;          // rows and first row of every step
  int32_t* order = nullptr;             // [rows] vertex (local row) by decreasing degree
  int32_t* pos = nullptr;               // [rows] position of a row in `order`
  int32_t* deg = nullptr;               // [rows] in-degree (local rows)
  int32_t* src_tm = nullptr;            // [S + 128] source of every step-major row (pads 0)
  int32_t* tpos = nullptr;              // [E_T] step-major row of each transposed-partition edge
  std::vector<void*> allocs;
};

namespace {

__global__ void k_lstm_steps(const int32_t* order, int64_t rows, const int32_t* deg, const int64_t* off,
                             const int64_t* row_ptr, const int32_t* idx, const int32_t* perm, int32_t* src_tm,
                             int32_t* epos) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < rows; j += (int64_t)gridDim.x * blockDim.x) {
    const int32_t v = order[j];
    const int64_t b = row_ptr[v];
    for (int32_t t = 0; t < deg[v]; ++t) {   // in-edges of v in edge-id order (the forward partition order)
      const int64_t k = off[t] + j;
      src_tm[k] = idx[b + t];
      epos[perm[b + t]] = (int32_t)k;
    }
  }
}

__global__ void k_tpos(const int32_t* permT, int64_t n, const int32_t* epos, int32_t* tpos) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    tpos[i] = epos[permT[i]];
}

// rows of a [n x F] fp32 table gathered by index: out[k] = tab[idx[k]]
__global__ void k_gather_rows(const float* tab, int64_t ldt, const int32_t* idx, int64_t n, int F, float* out,
                              int64_t ldo) {
  const int64_t tot = n * (int64_t)F;
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < tot; q += (int64_t)gridDim.x * blockDim.x) {
    const int64_t k = q / F;
    const int c = (int)(q % F);
    out[k * ldo + c] = tab[(int64_t)idx[k] * ldt + c];
  }
}

__device__ __forceinline__ float sigm(float z) { return 1.f / (1.f + __expf(-z)); }

// forward cell, rows j < n of step t: Z (pre-activations, ld 4H) -> activated
// gates in place; c, h state update; c_t / h_t kept per step for the backward
__global__ void k_lstm_cell(float* Z, int64_t ldz, int64_t n, int H, float* Cst, float* Hst, int64_t lds, float* Call,
                            float* Hseq, int64_t ldc) {
  const int64_t tot = n * (int64_t)H;
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < tot; q += (int64_t)gridDim.x * blockDim.x) {
    const int64_t j = q / H;
    const int k = (int)(q % H);
    float* z = Z + j * ldz;
    const float i = sigm(z[k]), f = sigm(z[H + k]), g = tanhf(z[2 * H + k]), o = sigm(z[3 * H + k]);
    z[k] = i; z[H + k] = f; z[2 * H + k] = g; z[3 * H + k] = o;
    const float c = f * Cst[j * lds + k] + i * g;
    const float h = o * tanhf(c);
    Cst[j * lds + k] = c;
    Hst[j * lds + k] = h;
    Call[j * ldc + k] = c;
    Hseq[j * ldc + k] = h;
  }
}

// backward cell, rows j < n of step t.  A row whose sequence ends at step t
// (deg == t + 1) starts from dh = dH_N[v], dc = 0; the others continue from
// the step t + 1 state.  G: activated gates of step t; Ct: c_t; Cp: c_{t-1}
// (nullptr at t = 0).  Writes dZ_t and the dc state.
__global__ void k_lstm_cell_bwd(const float* G, int64_t ldg, const float* Ct, const float* Cp, int64_t ldc, int64_t n,
                                int H, int t, const int32_t* order, const int32_t* deg, const float* dHN, int64_t ldh,
                                const float* dhst, float* dcst, int64_t lds, float* dZ, int64_t ldz) {
  const int64_t tot = n * (int64_t)H;
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < tot; q += (int64_t)gridDim.x * blockDim.x) {
    const int64_t j = q / H;
    const int k = (int)(q % H);
    const int32_t v = order[j];
    const bool last = deg[v] == t + 1;
    const float dh = last ? dHN[(int64_t)v * ldh + k] : dhst[j * lds + k];
    const float dc0 = last ? 0.f : dcst[j * lds + k];
    const float* g = G + j * ldg;
    const float i = g[k], f = g[H + k], gg = g[2 * H + k], o = g[3 * H + k];
    const float tc = tanhf(Ct[j * ldc + k]);
    const float cp = Cp ? Cp[j * ldc + k] : 0.f;
    const float dO = dh * tc;
    const float dC = dc0 + dh * o * (1.f - tc * tc);
    float* z = dZ + j * ldz;
    z[k] = dC * gg * i * (1.f - i);
    z[H + k] = dC * cp * f * (1.f - f);
    z[2 * H + k] = dC * i * (1.f - gg * gg);
    z[3 * H + k] = dO * o * (1.f - o);
    dcst[j * lds + k] = dC * f;
  }
}

// H_prev of every step-major row: h_{t-1} of the same row (0 at t = 0)
__global__ void k_hprev(const float* Hseq, int64_t ld, const int64_t* off, const int64_t* n, int64_t T, int H,
                        float* Hp) {
  const int64_t t = blockIdx.y;
  if (t >= T) return;
  const int64_t tot = n[t] * (int64_t)H;
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < tot; q += (int64_t)gridDim.x * blockDim.x) {
    const int64_t j = q / H;
    const int k = (int)(q % H);
    Hp[(off[t] + j) * ld + k] = t > 0 ? Hseq[(off[t - 1] + j) * ld + k] : 0.f;
  }
}

unsigned grid_for(int64_t n) { return (unsigned)std::max<int64_t>(1, std::min<int64_t>(cdiv(n, 256), 148 * 16)); }

}  // namespace

wg_status lstm_plan(wg_plan_s* p, cudaStream_t st) {
  wg_graph_s* g = p->g;
  const wg_conv_desc& d = p->d;
  WG_REQ(d.dtype == WG_F32, WG_ERR_UNSUPPORTED, "SAGE-LSTM: fp32 only (3xTF32 gates)");
  WG_REQ(g->vb == 0 && g->ve == g->V && !g->by_type, WG_ERR_UNSUPPORTED, "SAGE-LSTM: full untyped graphs only");
  WG_REQ(4 * d.f_in <= 1024, WG_ERR_UNSUPPORTED, "SAGE-LSTM: f_in <= 256");
  auto* L = new LstmPlan();
  p->lstm = L;
  const int64_t rows = g->V;
  const auto& rp = g->fwd.h_row_ptr;
  std::vector<int32_t> deg(rows), order(rows), pos(rows);
  for (int64_t v = 0; v < rows; ++v) deg[v] = (int32_t)(rp[v + 1] - rp[v]);
  for (int64_t v = 0; v < rows; ++v) order[v] = (int32_t)v;
  std::stable_sort(order.begin(), order.end(), [&](int32_t a, int32_t b) { return deg[a] > deg[b]; });
  for (int64_t j = 0; j < rows; ++j) pos[order[j]] = (int32_t)j;
  L->T = rows ? deg[order[0]] : 0;
  L->n.assign(L->T, 0);
  L->off.assign(L->T + 1, 0);
  for (int64_t j = 0, t = L->T - 1; t >= 0; --t) {       // n_t = #rows with deg > t
    while (j < rows && deg[order[j]] > t) ++j;
    L->n[t] = j;
  }
  for (int64_t t = 0; t < L->T; ++t) L->off[t + 1] = L->off[t] + rup(L->n[t], 4);   // 16-byte aligned steps
  L->S = L->off[L->T];
  auto up = [&](const void* h, size_t bytes, void** o) -> wg_status {
    WG_CK(cudaMalloc(o, std::max<size_t>(bytes, 256)));
    L->allocs.push_back(*o);
    if (bytes) WG_CK(cudaMemcpy(*o, h, bytes, cudaMemcpyHostToDevice));
    return WG_OK;
  };
  int64_t* doff = nullptr;
  int32_t* epos = nullptr;
  WG_TRY(up(order.data(), 4 * rows, (void**)&L->order));
  WG_TRY(up(pos.data(), 4 * rows, (void**)&L->pos));
  WG_TRY(up(deg.data(), 4 * rows, (void**)&L->deg));
  WG_TRY(up(L->off.data(), 8 * (L->T + 1), (void**)&doff));
  WG_CK(cudaMalloc((void**)&L->src_tm, 4 * (L->S + 128)));
  L->allocs.push_back(L->src_tm);
  WG_CK(cudaMemset(L->src_tm, 0, 4 * (L->S + 128)));
  WG_CK(cudaMalloc((void**)&epos, 4 * std::max<int64_t>(g->E_total, 1)));
  WG_CK(cudaMalloc((void**)&L->tpos, 4 * std::max<int64_t>(g->bwd.E, 1)));
  L->allocs.push_back(L->tpos);
  if (g->fwd.E) {
    WG_LAUNCH(k_lstm_steps, grid_for(rows), 256, 0, st, L->order, rows, L->deg, doff, g->fwd.row_ptr, g->fwd.idx,
              g->fwd.perm, L->src_tm, epos);
    WG_LAUNCH(k_tpos, grid_for(g->bwd.E), 256, 0, st, g->bwd.perm, g->bwd.E, epos, L->tpos);
  }
  WG_CK(cudaStreamSynchronize(st));
  cudaFree(epos);                               // (doff stays in L->allocs)
  // layouts (fp32; row pitches 32-byte padded)
  const int H = d.f_in;
  p->pi = pitch(d.f_in, d.dtype);
  p->po = pitch(d.f_out, d.dtype);
  const int64_t p4 = pitch(4 * H, d.dtype), ph = pitch(H, d.dtype);
  Layout& S = p->saved;
  Layout& W = p->ws;
  S = Layout();
  W = Layout();
  S.add("xall", 4 * (size_t)(L->S + 128) * p->pi);   // x[src] of every step-major row
  S.add("gall", 4 * (size_t)L->S * p4);             // activated gates
  S.add("call", 4 * (size_t)L->S * ph);             // c_t
  S.add("hseq", 4 * (size_t)L->S * ph);             // h_t
  S.add("hnat", 4 * (size_t)rows * ph);             // h_N(v), vertex order
  W.add("hst", 4 * (size_t)rows * ph);
  W.add("cst", 4 * (size_t)rows * ph);
  W.add("wiht", 4 * (size_t)4 * H * p->pi);         // W_ih^T [4H x f_in]
  W.add("whht", 4 * (size_t)4 * H * ph);            // W_hh^T [4H x H]
  W.add("wst", 4 * (size_t)rup(d.f_out, 16) * p->pi);
  W.add("wnt", 4 * (size_t)rup(d.f_out, 16) * ph);
  W.add("wih", 4 * (size_t)rup(d.f_in, 16) * p4);   // W_ih [f_in x 4H]
  W.add("whh", 4 * (size_t)rup(H, 16) * p4);
  W.add("wn", 4 * (size_t)rup(H, 16) * p->po);
  W.add("ws", 4 * (size_t)rup(d.f_in, 16) * p->po);
  W.add("dt", 4 * (size_t)rows * p->po);
  W.add("dhn", 4 * (size_t)rows * ph);
  W.add("dxs", 4 * (size_t)rows * p->pi);
  W.add("dhst", 4 * (size_t)rows * ph);
  W.add("dcst", 4 * (size_t)rows * ph);
  W.add("dz", 4 * (size_t)(L->S + 128) * p4);
  W.add("dxall", 4 * (size_t)(L->S + 128) * p->pi);
  W.add("hprev", 4 * (size_t)(L->S + 128) * ph);
  W.add("colsum", bias_grad_scratch(std::max<int64_t>(L->S, rows), (int)std::max<int64_t>(p4, p->po)));
  W.add("tn", std::max(gemm_tn_scratch(std::max<int64_t>(L->S, rows), d.f_in, 4 * H),
                       gemm_tn_scratch(rows, d.f_in, d.f_out)));
  W.add("part", 4 * (size_t)std::max(1, p->n_slots_t) * rup(std::max(d.f_in, d.f_out), 8));
  return WG_OK;
}

void lstm_plan_free(wg_plan_s* p) {
  auto* L = static_cast<LstmPlan*>(p->lstm);
  if (!L) return;
  for (void* q : L->allocs) cudaFree(q);
  delete L;
  p->lstm = nullptr;
}

wg_status lstm_forward(wg_plan_s* p, const wg_params* P, const wg_fwd_args* A, cudaStream_t st) {
  auto* L = static_cast<LstmPlan*>(p->lstm);
  const wg_conv_desc& d = p->d;
  wg_graph_s* g = p->g;
  WG_REQ(A->phase == WG_PHASE_ALL, WG_ERR_UNSUPPORTED, "SAGE-LSTM: WG_PHASE_ALL only");
  WG_REQ(P && P->W && P->W_self && P->Wih && P->Whh, WG_ERR_INVALID, "SAGE-LSTM needs W, W_self, Wih, Whh");
  WG_REQ(A->x && A->y && A->saved && A->workspace, WG_ERR_INVALID, "x / y / saved / workspace is NULL");
  WG_REQ(A->ldx % 4 == 0 && A->ldx >= d.f_in && A->ldy % 4 == 0 && A->ldy >= d.f_out, WG_ERR_INVALID,
         "ldx / ldy must be >= F and 16-byte multiples");
  const int H = d.f_in;
  const int64_t rows = g->V, p4 = pitch(4 * H, d.dtype), ph = pitch(H, d.dtype);
  const Layout& S = p->saved;
  const Layout& W = p->ws;
  void* sv = A->saved;
  void* ws = A->workspace;
  float *xall = S.at<float>(sv, "xall"), *gall = S.at<float>(sv, "gall"), *call = S.at<float>(sv, "call");
  float *hseq = S.at<float>(sv, "hseq"), *hnat = S.at<float>(sv, "hnat");
  float *hst = W.at<float>(ws, "hst"), *cst = W.at<float>(ws, "cst");
  void* wiht = W.at<void>(ws, "wiht");
  void* whht = W.at<void>(ws, "whht");
  WG_TRY(prep_weight(d.dtype, P->Wih, d.f_in, 4 * H, 1, wiht, p->pi, 4 * H, st));
  WG_TRY(prep_weight(d.dtype, P->Whh, H, 4 * H, 1, whht, ph, 4 * H, st));
  WG_CK(cudaMemsetAsync(hst, 0, 4 * rows * ph, st));
  WG_CK(cudaMemsetAsync(cst, 0, 4 * rows * ph, st));
  // X rows of every step, gathered once (step-major)
  if (L->S) {
    ProfScope ps(PK_AGG, st, (double)L->S * (4.0 + 4.0 * d.f_in) * 2, 0.0);
    WG_LAUNCH(k_gather_rows, grid_for(L->S * d.f_in), 256, 0, st, static_cast<const float*>(A->x), A->ldx, L->src_tm,
              L->S, d.f_in, xall, p->pi);
  }
  for (int64_t t = 0; t < L->T; ++t) {
    const int64_t n = L->n[t], o = L->off[t];
    GemmPart parts[2];
    int np = 0;
    parts[np++] = GemmPart{xall + o * p->pi, p->pi, wiht, p->pi, d.f_in, 4 * H};
    if (t > 0) parts[np++] = GemmPart{hst, ph, whht, ph, H, 4 * H};
    GemmEpi e;
    e.bias = P->bl;
    e.D = gall + o * p4; e.ldd = p4;
    WG_TRY(gemm_nt(d.dtype, n, 4 * H, parts, np, e, nullptr, 0, st));
    ProfScope ps(PK_MISC, st, (double)n * H * 4 * 10, 0.0);
    WG_LAUNCH(k_lstm_cell, grid_for(n * H), 256, 0, st, gall + o * p4, p4, n, H, cst, hst, ph, call + o * ph,
              hseq + o * ph, ph);
  }
  // h_N in vertex order, then y = x W_s + h_N W_n + b
  WG_LAUNCH(k_gather_rows, grid_for(rows * H), 256, 0, st, hst, ph, L->pos, rows, H, hnat, ph);
  void* wst = W.at<void>(ws, "wst");
  void* wnt = W.at<void>(ws, "wnt");
  WG_TRY(prep_weight(d.dtype, P->W_self, d.f_in, d.f_out, 1, wst, p->pi, (int)rup(d.f_out, 16), st));
  WG_TRY(prep_weight(d.dtype, P->W, H, d.f_out, 1, wnt, ph, (int)rup(d.f_out, 16), st));
  GemmPart parts[2] = {GemmPart{A->x, A->ldx, wst, p->pi, d.f_in, (int)rup(d.f_out, 16)},
                       GemmPart{hnat, ph, wnt, ph, H, (int)rup(d.f_out, 16)}};
  GemmEpi e;
  e.bias = d.bias ? P->bias : nullptr;
  e.relu = d.fuse_relu;
  e.D = A->y; e.ldd = A->ldy;
  return gemm_nt(d.dtype, rows, (int)rup(d.f_out, 4), parts, 2, e, nullptr, 0, st);
}

wg_status lstm_backward(wg_plan_s* p, const wg_params* P, const wg_bwd_args* A, const wg_grads* G, cudaStream_t st) {
  auto* L = static_cast<LstmPlan*>(p->lstm);
  const wg_conv_desc& d = p->d;
  wg_graph_s* g = p->g;
  WG_REQ(A->phase == WG_PHASE_ALL, WG_ERR_UNSUPPORTED, "SAGE-LSTM: WG_PHASE_ALL only");
  WG_REQ(P && P->W && P->W_self && P->Wih && P->Whh && A->dy && A->x && A->saved && A->workspace, WG_ERR_INVALID,
         "SAGE-LSTM backward: null argument");
  const bool mask_dy = d.fuse_relu && !A->dy_masked;
  WG_REQ(!mask_dy || A->y, WG_ERR_INVALID, "fuse_relu backward needs y");
  WG_REQ(!d.need_dx || A->dx, WG_ERR_INVALID, "need_dx but dx is NULL");
  const int H = d.f_in;
  const int64_t rows = g->V, p4 = pitch(4 * H, d.dtype), ph = pitch(H, d.dtype);
  const Layout& S = p->saved;
  const Layout& W = p->ws;
  const void* sv = A->saved;
  void* ws = A->workspace;
  const float *xall = S.at<float>(sv, "xall"), *gall = S.at<float>(sv, "gall"), *call = S.at<float>(sv, "call");
  const float *hseq = S.at<float>(sv, "hseq"), *hnat = S.at<float>(sv, "hnat");
  float* colsum = W.at<float>(ws, "colsum");
  void* tn = W.at<void>(ws, "tn");
  // dT = dy (ReLU-masked), db
  float* dtb = W.at<float>(ws, "dt");
  WG_TRY(bias_grad_mask(d.dtype, rows, d.f_out, A->dy, A->lddy, mask_dy ? A->y : nullptr, A->ldy, dtb, p->po,
                        (G && d.bias) ? G->bias : nullptr, colsum, st));
  const float* dT = dtb;
  const int64_t lddT = p->po;
  if (G && G->W_self) WG_TRY(gemm_tn(d.dtype, rows, d.f_in, d.f_out, A->x, A->ldx, dT, lddT, G->W_self, tn, st));
  if (G && G->W) WG_TRY(gemm_tn(d.dtype, rows, H, d.f_out, hnat, ph, dT, lddT, G->W, tn, st));
  // dH_N = dT W_n^T, dx_self = dT W_s^T
  void* wn = W.at<void>(ws, "wn");
  void* wsb = W.at<void>(ws, "ws");
  WG_TRY(prep_weight(d.dtype, P->W, H, d.f_out, 0, wn, p->po, (int)rup(H, 16), st));
  WG_TRY(prep_weight(d.dtype, P->W_self, d.f_in, d.f_out, 0, wsb, p->po, (int)rup(d.f_in, 16), st));
  float* dhn = W.at<float>(ws, "dhn");
  {
    GemmPart part{dT, lddT, wn, p->po, d.f_out, (int)rup(H, 16)};
    GemmEpi e;
    e.D = dhn; e.ldd = ph;
    WG_TRY(gemm_nt(d.dtype, rows, (int)rup(H, 4), &part, 1, e, nullptr, 0, st));
  }
  float* dxs = W.at<float>(ws, "dxs");
  if (d.need_dx) {
    GemmPart part{dT, lddT, wsb, p->po, d.f_out, (int)rup(d.f_in, 16)};
    GemmEpi e;
    e.D = dxs; e.ldd = p->pi;
    WG_TRY(gemm_nt(d.dtype, rows, (int)rup(d.f_in, 4), &part, 1, e, nullptr, 0, st));
  }
  // backpropagation through time over the degree-ordered prefixes
  void* whh = W.at<void>(ws, "whh");
  void* wih = W.at<void>(ws, "wih");
  WG_TRY(prep_weight(d.dtype, P->Whh, H, 4 * H, 0, whh, p4, (int)rup(H, 16), st));
  WG_TRY(prep_weight(d.dtype, P->Wih, d.f_in, 4 * H, 0, wih, p4, (int)rup(d.f_in, 16), st));
  float *dhst = W.at<float>(ws, "dhst"), *dcst = W.at<float>(ws, "dcst"), *dz = W.at<float>(ws, "dz");
  WG_CK(cudaMemsetAsync(dz, 0, 4 * (size_t)(L->S + 128) * p4, st));
  for (int64_t t = L->T - 1; t >= 0; --t) {
    const int64_t n = L->n[t], o = L->off[t];
    {
      ProfScope ps(PK_MISC, st, (double)n * H * 4 * 12, 0.0);
      WG_LAUNCH(k_lstm_cell_bwd, grid_for(n * H), 256, 0, st, gall + o * p4, p4, call + o * ph,
                t > 0 ? call + L->off[t - 1] * ph : nullptr, ph, n, H, (int)t, L->order, L->deg, dhn, ph, dhst, dcst,
                ph, dz + o * p4, p4);
    }
    if (t > 0) {   // dh of step t-1 = dZ_t W_hh^T
      GemmPart part{dz + o * p4, p4, whh, p4, 4 * H, (int)rup(H, 16)};
      GemmEpi e;
      e.D = dhst; e.ldd = ph;
      WG_TRY(gemm_nt(d.dtype, n, (int)rup(H, 4), &part, 1, e, nullptr, 0, st));
    }
  }
  // weight gradients of the LSTM over every step at once
  if (G && G->Wih) WG_TRY(gemm_tn(d.dtype, L->S, d.f_in, 4 * H, xall, p->pi, dz, p4, G->Wih, tn, st));
  if (G && G->Whh) {
    float* hp = W.at<float>(ws, "hprev");
    std::vector<int64_t> hn(L->n.begin(), L->n.end());
    int64_t *don = nullptr;
    // device copies of n / off for k_hprev (small, per call; stream-ordered)
    WG_CK(cudaMallocAsync((void**)&don, 16 * (L->T + 1), st));
    WG_CK(cudaMemcpyAsync(don, hn.data(), 8 * L->T, cudaMemcpyHostToDevice, st));
    WG_CK(cudaMemcpyAsync(don + L->T, L->off.data(), 8 * (L->T + 1), cudaMemcpyHostToDevice, st));
    WG_CK(cudaMemsetAsync(hp, 0, 4 * (size_t)(L->S + 128) * ph, st));
    if (L->T) {
      dim3 grid(grid_for(rows * H), (unsigned)L->T);
      WG_LAUNCH(k_hprev, grid, 256, 0, st, hseq, ph, don + L->T, don, L->T, H, hp);
    }
    WG_CK(cudaFreeAsync(don, st));
    WG_TRY(gemm_tn(d.dtype, L->S, H, 4 * H, hp, ph, dz, p4, G->Whh, tn, st));
  }
  if (G && G->bl)
    WG_TRY(bias_grad_mask(d.dtype, std::max<int64_t>(L->S, 1), 4 * H, dz, p4, nullptr, 0, nullptr, 0, G->bl, colsum,
                          st));
  if (!d.need_dx) return WG_OK;
  // dX of every step-major row = dZ W_ih^T; dx[u] = dx_self[u] + sum over u's out-edges (transposed gTasks)
  float* dxall = W.at<float>(ws, "dxall");
  if (L->S) {
    GemmPart part{dz, p4, wih, p4, 4 * H, (int)rup(d.f_in, 16)};
    GemmEpi e;
    e.D = dxall; e.ldd = p->pi;
    WG_TRY(gemm_nt(d.dtype, L->S, (int)rup(d.f_in, 4), &part, 1, e, nullptr, 0, st));
  }
  AggArgs a{};
  a.items = p->bt.d; a.n_items = p->bt.n;
  a.row_ptr = g->bwd.row_ptr; a.idx = L->tpos; a.key = g->bwd.key;
  a.row_base = 0; a.self_coef = 1.f; a.E_max = g->E_max;
  a.n_edges = p->bt.n_edges; a.n_rows = p->bt.n_rows;
  a.table = dxall; a.ld_tab = p->pi;
  a.self_tab = dxs; a.ld_self = p->pi;
  a.mask_ref = A->dx_mask; a.ld_mask = A->ld_dx_mask;
  a.out = A->dx; a.ld_out = A->lddx;
  a.partial = W.at<float>(ws, "part"); a.ld_part = rup(std::max(d.f_in, d.f_out), 8);
  a.F = d.f_in;
  WG_TRY(launch_agg(d.dtype, a, st));
  CombineArgs b{};
  b.rows = p->bt.split; b.n_rows = p->bt.n_split;
  b.partial = a.partial; b.ld_part = a.ld_part;
  b.self_tab = dxs; b.ld_self = p->pi; b.self_coef = 1.f;
  b.mask_ref = A->dx_mask; b.ld_mask = A->ld_dx_mask;
  b.out = A->dx; b.ld_out = A->lddx;
  b.F = d.f_in; b.plan_filter = -1;
  return launch_combine(d.dtype, b, st);
}

}  // namespace wg
