// GCN / GraphSAGE-mean / GIN layers: forward (a5-a8) and backward (a9-a11).
//
// All three are "aggregate + linear transform" layers, so the two operation
// plans of the paper apply (T2 indexing swapping):
//   EDGE   (gather-then-transform): Agg = A_hat x   ->  y = Agg W
//   VERTEX (transform-before-gather): Y = x W      ->  y = A_hat Y
// chosen per gTask by the plan (plan.cu).  A mixed plan writes Agg rows for
// EDGE gTasks and Z rows for VERTEX gTasks (each row belongs to exactly one
// gTask or SPLIT row) and the final GEMM computes y = Agg W + Z + b.
//
// Backward (the paper is silent, Q8; exact gradients of the definitions in
// DESIGN.md "Backward") runs the same gather pattern over the transposed gTask
// partition, in one of two orders:
//   dAgg path (all-EDGE forward, Agg saved):  dAgg = dT W^T, dx = A_hat^T dAgg,
//                                             dW = Agg^T dT
//   G path (otherwise):                       G = A_hat^T dT, dx = G W^T,
//                                             dW = x^T G
// where dT is dy masked by the fused ReLU.
#include "plan.h"

namespace wg {

namespace {

struct Ctx {
  wg_plan_s* p;
  wg_graph_s* g;
  wg_dtype dt;
  int s;        // dtype bytes
  int fi, fo;
  int64_t pi, po, nr, Vg, vb;
  int64_t wrows_o, wrows_i;   // padded weight row counts
};

Ctx mk(wg_plan_s* p) {
  Ctx c;
  c.p = p; c.g = p->g; c.dt = p->d.dtype; c.s = dsize(c.dt);
  c.fi = p->d.f_in; c.fo = p->d.f_out;
  c.pi = p->pi; c.po = p->po;
  c.nr = c.g->ve - c.g->vb; c.Vg = c.g->V; c.vb = c.g->vb;
  c.wrows_o = rup(c.fo, 16); c.wrows_i = rup(c.fi, 16);
  return c;
}

int64_t part_ld(const Ctx& c) { return rup(std::max(c.fi, c.fo), 8); }

char* off(const void* base, int64_t rows, int64_t ld, int s) {
  return (char*)base + rows * ld * s;
}

}  // namespace

void lin_layout(wg_plan_s* p) {
  const wg_conv_desc& d = p->d;
  p->pi = pitch(d.f_in, d.dtype);
  p->po = pitch(d.f_out, d.dtype);
  Ctx c = mk(p);
  const int s = c.s;
  Layout& S = p->saved;
  Layout& W = p->ws;
  S = Layout();
  W = Layout();
  const bool sage = d.model == WG_SAGE, gin = d.model == WG_GIN;
  if (edge_path(p)) S.add("agg", (size_t)c.nr * c.pi * s);
  if (gin) S.add("h", (size_t)c.nr * c.po * s);
  // prepped weights (forward: transposed [rows_o x pi]; backward: [rows_i x po])
  W.add("wt", (size_t)c.wrows_o * c.pi * s);          // W^T (GCN W, SAGE W_n, GIN W1)
  W.add("w", (size_t)c.wrows_i * c.po * s);           // W
  if (sage) {
    W.add("wst", (size_t)c.wrows_o * c.pi * s);
    W.add("ws", (size_t)c.wrows_i * c.po * s);
    W.add("wys", (size_t)2 * c.po * c.pi * s);       // [W_n^T ; W_s^T] stacked along N
    W.add("wbs", (size_t)2 * c.pi * c.po * s);       // [W_n ; W_s] stacked along N
    W.add("s", (size_t)c.nr * c.po * s);             // x W_s (all-VERTEX forward)
    W.add("dxs", (size_t)c.nr * c.pi * s);           // dy W_s^T (dAgg path)
  }
  if (gin) {
    W.add("w2t", (size_t)c.wrows_o * c.po * s);
    W.add("w2", (size_t)c.wrows_o * c.po * s);
    W.add("da", (size_t)c.nr * c.po * s);
  }
  // tables the gathers read (Y, dT, dAgg, GIN da) live here only on a full
  // graph (nr == V); on a 1-D partition they are the caller's exchange
  // tables (global rows), so these buffers hold owned rows only
  if (p->n_vert_tasks > 0) W.add("y", (size_t)c.nr * c.po * s);
  if (p->mixed) W.add("z", (size_t)c.nr * c.po * s);
  const int64_t pl = part_ld(c);
  W.add("part", sizeof(float) * (size_t)std::max(1, p->n_slots_f) * pl);
  W.add("partT", sizeof(float) * (size_t)std::max(1, p->n_slots_t) * pl);
  // backward
  W.add("dt", (size_t)c.nr * c.po * s);
  W.add("colsum", bias_grad_scratch(c.nr, (int)std::max(c.po, c.pi)));
  W.add("tn", gemm_tn_scratch(c.nr, (int)c.fi, (int)c.fo) + gemm_tn_scratch(c.nr, (int)c.fo, (int)c.fo));
  W.add("dagg", (size_t)c.nr * c.pi * s);
  W.add("g", (size_t)c.nr * c.po * s);
}

namespace {

AggArgs agg_base(const Ctx& c, const ItemList& L, const Side& S) {
  AggArgs a{};
  a.items = L.d;
  a.n_items = L.n;
  a.row_ptr = S.row_ptr;
  a.idx = S.idx;
  a.key = S.key;
  a.row_base = c.vb;
  a.self_coef = 1.f;
  a.E_max = c.g->E_max;
  a.n_edges = L.n_edges;
  a.n_rows = L.n_rows;
  return a;
}

CombineArgs comb_from(const AggArgs& a, const ItemList& L, int plan_filter) {
  CombineArgs b{};
  b.rows = L.split; b.n_rows = L.n_split;
  b.partial = a.partial; b.ld_part = a.ld_part;
  b.rscale = a.rscale; b.row_base = a.row_base;
  b.self_tab = a.self_tab; b.ld_self = a.ld_self; b.self_coef = a.self_coef;
  b.bias = a.bias; b.relu = a.relu; b.mask_ref = a.mask_ref; b.ld_mask = a.ld_mask;
  b.out = a.out; b.ld_out = a.ld_out;
  b.zero_out = a.zero_out; b.ld_zero = a.ld_zero; b.zero_cols = a.zero_cols;
  b.F = a.F; b.plan_filter = plan_filter;
  return b;
}

wg_status run_agg(const Ctx& c, AggArgs a, const ItemList& L, cudaStream_t st) {
  return launch_agg_outliers(c.dt, a, L.n_split_items, L.split, L.n_split, comb_from(a, L, -1), st);
}

// Gather over an exchange table in layout X (chunk k = [V x Fc] at k * V * Fc
// elements): one gather + combine per column chunk, writing columns
// [k Fc, k Fc + Fc) of the output (aggregation is column-separable); before
// chunk k the stream waits for its arrival (hook).  The self / mask / bias
// operands are ordinary row-major [rows x ld] tensors.
wg_status run_agg_x(const Ctx& c, AggArgs a, const ItemList& L, cudaStream_t st, const XLayout& X,
                    const XHook* hk) {
  if (X.C <= 1) {
    if (hk) hk->wait(0, st);
    return run_agg(c, a, L, st);
  }
  const int F = a.F;
  for (int k = 0; k < X.C; ++k) {
    const int64_t c0 = k * X.Fc;
    if (c0 >= F) break;
    if (hk) hk->wait(k, st);
    AggArgs b = a;
    b.table = static_cast<const char*>(a.table) + (size_t)k * c.Vg * X.Fc * c.s;
    b.ld_tab = X.Fc;
    b.F = (int)std::min<int64_t>(X.Fc, F - c0);
    b.out = static_cast<char*>(a.out) + c0 * c.s;
    if (a.bias) b.bias = a.bias + c0;
    if (a.self_tab) b.self_tab = static_cast<const char*>(a.self_tab) + c0 * c.s;
    if (a.mask_ref) b.mask_ref = static_cast<const char*>(a.mask_ref) + c0 * c.s;
    WG_TRY(run_agg(c, b, L, st));
  }
  return WG_OK;
}

// GEMM output into this rank's rows of an exchange table (layout X, caller
// pitch ld when X.C == 1)
void epi_xchg(const Ctx& c, GemmEpi* e, void* tab, int64_t ld, const XLayout& X) {
  if (X.C > 1) {
    e->D = off(tab, c.vb, X.Fc, c.s);
    e->ldd = X.Fc;
    e->d_chunk_cols = (int)X.Fc;
    e->d_chunk_stride = c.Vg * X.Fc;
  } else {
    e->D = off(tab, c.vb, ld, c.s);
    e->ldd = ld;
  }
}

// GCN edge coefficient c_e = gs[src] * rs[dst] (Q3)
void gcn_scales(const Ctx& c, const float** gs_src, const float** rs_dst) {
  *gs_src = nullptr; *rs_dst = nullptr;
  if (c.p->d.model == WG_SAGE) { *rs_dst = c.g->inv_in; return; }
  if (c.p->d.model != WG_GCN) return;
  if (c.p->d.norm == WG_NORM_BOTH) { *gs_src = c.g->rs_out; *rs_dst = c.g->rs_in; }
  else if (c.p->d.norm == WG_NORM_RIGHT) { *rs_dst = c.g->inv_in; }
}

}  // namespace

wg_status lin_forward(wg_plan_s* p, const wg_params* P, const wg_fwd_args* A, cudaStream_t st, const XHook* hk) {
  Ctx c = mk(p);
  const wg_conv_desc& d = p->d;
  const bool sage = d.model == WG_SAGE, gin = d.model == WG_GIN;
  const bool pre = A->phase != WG_PHASE_POST, post = A->phase != WG_PHASE_PRE;
  WG_REQ(P && P->W, WG_ERR_INVALID, "params->W is NULL");
  WG_REQ(!sage || P->W_self, WG_ERR_INVALID, "SAGE needs W_self");
  WG_REQ(!gin || P->W2, WG_ERR_INVALID, "GIN needs W2");
  WG_REQ(A->x && A->y && A->workspace, WG_ERR_INVALID, "x / y / workspace is NULL");
  WG_REQ(!edge_path(p) || A->saved, WG_ERR_INVALID, "saved is NULL");
  WG_REQ((A->ldx * c.s) % 16 == 0 && A->ldx >= c.fi && (A->ldy * c.s) % 16 == 0 && A->ldy >= c.fo, WG_ERR_INVALID,
         "ldx / ldy must be >= F and 16-byte multiples");
  const bool dist = c.nr != c.Vg;
  WG_REQ(!dist || !p->mixed, WG_ERR_UNSUPPORTED, "mixed EDGE/VERTEX plans are not supported with a 1-D partition");
  // on a 1-D partition the VERTEX gathers read Y rows other ranks own: the
  // exchange table is required (the workspace holds owned rows only)
  WG_REQ(!dist || !post || p->n_vert_tasks == 0 || A->xchg, WG_ERR_INVALID,
         "a VERTEX layer on a 1-D partition needs the exchange table (xchg)");
  const XLayout xl = A->xchg ? p->xf : XLayout{};
  WG_REQ(!A->xchg || ((A->ld_xchg * c.s) % 16 == 0 && (xl.C > 1 || A->ld_xchg >= c.fo)), WG_ERR_INVALID,
         "ld_xchg must be >= f_out (the chunk pitch for a chunked table) and a 16-byte multiple");
  WG_REQ(xl.C <= 1 || A->ld_xchg == xl.Fc, WG_ERR_INVALID,
         "chunked exchange table: ld_xchg must be the chunk width (wg_plan_xchg)");
  void* ws = A->workspace;
  const Layout& L = p->ws;
  const char* x_own = off(A->x, c.vb, A->ldx, c.s);
  const float *gs, *rs;
  gcn_scales(c, &gs, &rs);
  const bool all_vertex = !edge_path(p);
  const bool has_bias = d.bias && P->bias;
  // prepped weights
  void* wt = L.at<void>(ws, "wt");
  WG_TRY(prep_weight(c.dt, P->W, c.fi, c.fo, 1, wt, c.pi, (int)c.wrows_o, st));
  void* wst = nullptr;
  if (sage) {
    wst = L.at<void>(ws, "wst");
    WG_TRY(prep_weight(c.dt, P->W_self, c.fi, c.fo, 1, wst, c.pi, (int)c.wrows_o, st));
  }
  // ---- VERTEX table: Y = x W (own rows), exchanged in the distributed case
  void* ytab = nullptr;
  int64_t ldY = c.po;
  // a rank with no VERTEX gTask of its own (e.g. no in-edge at all) still
  // writes its rows of the exchanged Y table when the caller passes one:
  // the other ranks' VERTEX gathers read them
  if (p->n_vert_tasks > 0 || (A->xchg && pre)) {
    ytab = A->xchg ? A->xchg : L.at<void>(ws, "y");
    ldY = A->xchg ? A->ld_xchg : c.po;
    if (pre && sage && all_vertex) {
      // [Y | S] = x [W_n | W_s] in one GEMM (x read once); S = self term
      void* wys = L.at<void>(ws, "wys");
      WG_TRY(prep_weight(c.dt, P->W, c.fi, c.fo, 1, wys, c.pi, (int)c.po, st));
      WG_TRY(prep_weight(c.dt, P->W_self, c.fi, c.fo, 1, off(wys, c.po, c.pi, c.s), c.pi, (int)c.po, st));
      GemmPart part{x_own, A->ldx, wys, c.pi, c.fi, (int)(2 * c.po)};
      GemmEpi e;
      epi_xchg(c, &e, ytab, ldY, xl);
      e.D2 = L.at<void>(ws, "s");
      e.ldd2 = c.po;
      e.n_split = (int)c.po;
      WG_TRY(gemm_nt(c.dt, c.nr, (int)(2 * c.po), &part, 1, e, nullptr, 0, st));
    } else if (pre) {
      GemmPart part{x_own, A->ldx, wt, c.pi, c.fi, (int)c.wrows_o};
      GemmEpi e;
      epi_xchg(c, &e, ytab, ldY, xl);
      WG_TRY(gemm_nt(c.dt, c.nr, (int)rup(c.fo, 16 / c.s), &part, 1, e, nullptr, 0, st));
    }
  }
  if (!post) return WG_OK;
  void* agg = edge_path(p) ? p->saved.at<void>(A->saved, "agg") : nullptr;
  void* z = p->mixed ? L.at<void>(ws, "z") : nullptr;
  void* h = gin ? p->saved.at<void>(A->saved, "h") : nullptr;
  const int64_t pl = part_ld(c);
  // ---- EDGE gTasks: Agg = A_hat x  (GIN: z = (1+eps) x + A x)
  if (edge_path(p)) {
    AggArgs a = agg_base(c, p->fe, c.g->fwd);
    a.table = A->x; a.ld_tab = A->ldx;
    a.gscale = gs; a.rscale = rs;
    if (gin) { a.self_tab = x_own; a.ld_self = A->ldx; a.self_coef = 1.f + d.gin_eps; }
    a.out = agg; a.ld_out = c.pi;
    a.zero_out = z; a.ld_zero = c.po; a.zero_cols = (int)c.po;
    a.partial = L.at<float>(ws, "part"); a.ld_part = pl;
    a.F = c.fi;
    WG_TRY(run_agg(c, a, p->fe, st));
  }
  // ---- VERTEX gTasks: out = A_hat Y (+ self, bias, relu when all-VERTEX)
  if (p->n_vert_tasks > 0) {
    AggArgs a = agg_base(c, p->fv, c.g->fwd);
    a.table = ytab; a.ld_tab = ldY;
    a.gscale = gs; a.rscale = rs;
    a.partial = L.at<float>(ws, "part"); a.ld_part = pl;
    a.F = c.fo;
    if (gin) { a.self_tab = off(ytab, c.vb, ldY, c.s); a.ld_self = ldY; a.self_coef = 1.f + d.gin_eps; }
    if (all_vertex) {
      if (sage) { a.self_tab = L.at<void>(ws, "s"); a.ld_self = c.po; a.self_coef = 1.f; }
      if (gin) {  // a = A_hat-stage output + b1 -> h = relu(a)
        a.bias = P->bias; a.relu = 1; a.out = h; a.ld_out = c.po;
      } else {
        a.bias = has_bias ? P->bias : nullptr; a.relu = d.fuse_relu; a.out = A->y; a.ld_out = A->ldy;
      }
    } else {
      a.out = z; a.ld_out = c.po;
      a.zero_out = agg; a.ld_zero = c.pi; a.zero_cols = (int)c.pi;
    }
    WG_TRY(run_agg_x(c, a, p->fv, st, xl, hk));
  }
  // ---- EDGE transform: y = Agg W (+ x W_s) + Z + b
  if (edge_path(p)) {
    GemmPart parts[2];
    int np = 0;
    if (sage) parts[np++] = GemmPart{x_own, A->ldx, wst, c.pi, c.fi, (int)c.wrows_o};
    parts[np++] = GemmPart{agg, c.pi, wt, c.pi, c.fi, (int)c.wrows_o};
    GemmEpi e;
    e.addend = z; e.ld_add = c.po;
    if (gin) {
      e.bias = P->bias; e.relu = 1; e.D = h; e.ldd = c.po;
    } else {
      e.bias = has_bias ? P->bias : nullptr; e.relu = d.fuse_relu; e.D = A->y; e.ldd = A->ldy;
    }
    WG_TRY(gemm_nt(c.dt, c.nr, (int)rup(c.fo, 16 / c.s), parts, np, e, nullptr, 0, st));
  }
  // ---- GIN second linear: y = h W2 + b2
  if (gin) {
    void* w2t = L.at<void>(ws, "w2t");
    WG_TRY(prep_weight(c.dt, P->W2, c.fo, c.fo, 1, w2t, c.po, (int)c.wrows_o, st));
    GemmPart part{h, c.po, w2t, c.po, c.fo, (int)c.wrows_o};
    GemmEpi e;
    e.bias = P->b2; e.relu = d.fuse_relu; e.D = A->y; e.ldd = A->ldy;
    WG_TRY(gemm_nt(c.dt, c.nr, (int)rup(c.fo, 16 / c.s), &part, 1, e, nullptr, 0, st));
  }
  return WG_OK;
}

wg_status lin_backward(wg_plan_s* p, const wg_params* P, const wg_bwd_args* A, const wg_grads* G, cudaStream_t st,
                       const XHook* hk) {
  Ctx c = mk(p);
  const wg_conv_desc& d = p->d;
  const bool sage = d.model == WG_SAGE, gin = d.model == WG_GIN;
  const bool pre = A->phase != WG_PHASE_POST, post = A->phase != WG_PHASE_PRE;
  WG_REQ(P && P->W && A->dy && A->x && A->workspace, WG_ERR_INVALID, "backward: null argument");
  WG_REQ(!d.fuse_relu || A->y || A->dy_masked, WG_ERR_INVALID, "fuse_relu backward needs y");
  WG_REQ(!d.need_dx || A->dx, WG_ERR_INVALID, "need_dx but dx is NULL");
  WG_REQ(!edge_path(p) || A->saved, WG_ERR_INVALID, "saved is NULL");
  // dy already masked by the next layer (dx_mask fusion): no mask pass here
  const bool mask_dy = d.fuse_relu && !A->dy_masked;
  const bool dist = c.nr != c.Vg;
  // on a 1-D partition the transposed gather reads rows other ranks own
  // (dT / dAgg / GIN da): the exchange table is required
  WG_REQ(!dist || !post || (p->bwd_path == 0 && !d.need_dx) || A->xchg, WG_ERR_INVALID,
         "backward on a 1-D partition needs the exchange table (xchg)");
  WG_REQ(!A->xchg || (A->ld_xchg * c.s) % 16 == 0, WG_ERR_INVALID, "ld_xchg must be a 16-byte multiple");
  void* ws = A->workspace;
  const Layout& L = p->ws;
  const char* x_own = off(A->x, c.vb, A->ldx, c.s);
  const float *gs, *rs;
  gcn_scales(c, &gs, &rs);
  const int path = p->bwd_path;
  void* xchg = A->xchg;
  const int64_t pl = part_ld(c);
  float* colsum = L.at<float>(ws, "colsum");
  void* tn = L.at<void>(ws, "tn");
  // prepped weights for backward
  void* w = L.at<void>(ws, "w");
  WG_TRY(prep_weight(c.dt, P->W, c.fi, c.fo, 0, w, c.po, (int)c.wrows_i, st));
  void* wsb = nullptr;
  if (sage) {
    wsb = L.at<void>(ws, "ws");
    WG_TRY(prep_weight(c.dt, P->W_self, c.fi, c.fo, 0, wsb, c.po, (int)c.wrows_i, st));
  }
  // ---- dT = dy (masked by the fused ReLU); db
  // The table the transposed gather reads (dT in the G path, dAgg in the
  // dAgg path) lives in the exchange buffer when distributed.
  // (single GPU: vb == 0 and every table is indexed by global == local rows)
  const bool gpath_lin = (path == 1 && !gin);
  // 1-D partition: the destination scale rs[d] of the transposed gather is
  // folded into the exchanged rows by their owner in PRE (dT rs on the G
  // path, dAgg rs on the dAgg path), so the POST gather reads no per-edge
  // scale -- a random 4-byte load per edge from a V-sized array (444 MB at C5)
  const bool fold = xchg != nullptr && rs != nullptr && !gin;
  const float* rs_own = rs ? rs + c.vb : nullptr;
  const XLayout xl = xchg ? p->xb : XLayout{};
  WG_REQ(xl.C <= 1 || A->ld_xchg == xl.Fc, WG_ERR_INVALID,
         "chunked exchange table: ld_xchg must be the chunk width (wg_plan_xchg)");
  void* dt_buf = nullptr;                  // dT of the owned rows (row-major), when dy itself is not it
  int64_t ld_dtb = c.po;
  void* dt_x = nullptr;                    // G path: this rank's rows of the exchange table, dT (* rs)
  if (gpath_lin && xchg) dt_x = xl.C > 1 ? off(xchg, c.vb, xl.Fc, c.s) : off(xchg, c.vb, A->ld_xchg, c.s);
  if (mask_dy) dt_buf = L.at<void>(ws, "dt");             // owned rows, local indexing
  if (pre) {
    float* db = gin ? (G ? G->b2 : nullptr) : (G ? G->bias : nullptr);
    if (dt_buf || db || dt_x)
      WG_TRY(bias_grad_mask(c.dt, c.nr, c.fo, A->dy, A->lddy, mask_dy ? A->y : nullptr, A->ldy, dt_buf, ld_dtb,
                            db, colsum, st, fold ? rs_own : nullptr, dt_x, xl.C > 1 ? xl.Fc : A->ld_xchg,
                            xl.C > 1 ? (int)xl.Fc : 0, c.Vg * xl.Fc));
  }
  const void* dT = dt_buf ? dt_buf : A->dy;
  const int64_t lddT = dt_buf ? ld_dtb : A->lddy;
  const void* dTT;        // gradient w.r.t. the swappable transform's output
  int64_t lddTT;
  const void* gtab = nullptr;   // G-path gathered table (global rows)
  int64_t ldg = lddT;
  if (gpath_lin) { gtab = xchg ? xchg : dT; ldg = xchg ? A->ld_xchg : lddT; }
  dTT = dT; lddTT = lddT;
  // ---- GIN MLP tail: dW2 = h^T dT, da = (dT W2^T) * [h > 0], db1 = sum da
  void* gin_tab = nullptr;
  int64_t ld_gin = c.po;
  if (gin) {
    void* h = p->saved.at<void>(A->saved, "h");
    gin_tab = (path == 1 && xchg) ? xchg : L.at<void>(ws, "da");
    ld_gin = (path == 1 && xchg) ? A->ld_xchg : c.po;
    void* da = off(gin_tab, (path == 1 && xchg) ? c.vb : 0, ld_gin, c.s);   // ws "da": owned rows
    if (pre) {
      if (G && G->W2) WG_TRY(gemm_tn(c.dt, c.nr, c.fo, c.fo, h, c.po, dT, lddT, G->W2, tn, st));
      void* w2 = L.at<void>(ws, "w2");
      WG_TRY(prep_weight(c.dt, P->W2, c.fo, c.fo, 0, w2, c.po, (int)c.wrows_o, st));
      GemmPart part{dT, lddT, w2, c.po, c.fo, (int)c.wrows_o};
      GemmEpi e;
      e.mask_ref = h; e.ld_mask = c.po; e.D = da; e.ldd = ld_gin;
      WG_TRY(gemm_nt(c.dt, c.nr, (int)rup(c.fo, 16 / c.s), &part, 1, e, nullptr, 0, st));
      if (G && G->bias) WG_TRY(bias_grad_mask(c.dt, c.nr, c.fo, da, ld_gin, nullptr, 0, nullptr, 0, G->bias, colsum, st));
    }
    dTT = da; lddTT = ld_gin;
    if (path == 1) { gtab = gin_tab; ldg = ld_gin; }
  }
  // ---- dAgg path
  if (path == 0) {
    void* agg = p->saved.at<void>(A->saved, "agg");
    void* dtab = xchg ? xchg : L.at<void>(ws, "dagg");
    const int64_t ldd = xchg ? A->ld_xchg : c.pi;
    if (pre) {
      if (G && G->W) WG_TRY(gemm_tn(c.dt, c.nr, c.fi, c.fo, agg, c.pi, dTT, lddTT, G->W, tn, st));
      if (sage && G && G->W_self) WG_TRY(gemm_tn(c.dt, c.nr, c.fi, c.fo, x_own, A->ldx, dT, lddT, G->W_self, tn, st));
      if (d.need_dx && sage) {
        // [dAgg | dXs] = dT [W_n ; W_s]^T in one GEMM (dT read once)
        void* wbs = L.at<void>(ws, "wbs");
        WG_TRY(prep_weight(c.dt, P->W, c.fi, c.fo, 0, wbs, c.po, (int)c.pi, st));
        WG_TRY(prep_weight(c.dt, P->W_self, c.fi, c.fo, 0, off(wbs, c.pi, c.po, c.s), c.po, (int)c.pi, st));
        GemmPart part{dT, lddT, wbs, c.po, c.fo, (int)(2 * c.pi)};
        GemmEpi e;
        epi_xchg(c, &e, dtab, ldd, xl);
        e.rscale = fold ? rs_own : nullptr;    // dAgg only (D), not dX_s (D2)
        e.D2 = L.at<void>(ws, "dxs"); e.ldd2 = c.pi; e.n_split = (int)c.pi;
        WG_TRY(gemm_nt(c.dt, c.nr, (int)(2 * c.pi), &part, 1, e, nullptr, 0, st));
      } else if (d.need_dx) {
        GemmPart part{dTT, lddTT, w, c.po, c.fo, (int)c.wrows_i};
        GemmEpi e;
        epi_xchg(c, &e, dtab, ldd, xl);
        e.rscale = fold ? rs_own : nullptr;
        WG_TRY(gemm_nt(c.dt, c.nr, (int)rup(c.fi, 16 / c.s), &part, 1, e, nullptr, 0, st));
      }
    }
    if (post && d.need_dx) {
      AggArgs a = agg_base(c, p->bt, c.g->bwd);
      a.table = dtab; a.ld_tab = ldd;
      a.gscale = fold ? nullptr : rs; a.rscale = gs;   // transposed: c_e = gs[u] * rs[d]
      if (sage) { a.self_tab = L.at<void>(ws, "dxs"); a.ld_self = c.pi; a.self_coef = 1.f; }
      if (gin) { a.self_tab = off(dtab, c.vb, ldd, c.s); a.ld_self = ldd; a.self_coef = 1.f + d.gin_eps; }
      a.out = A->dx; a.ld_out = A->lddx;
      a.mask_ref = A->dx_mask; a.ld_mask = A->ld_dx_mask;
      a.partial = L.at<float>(ws, "partT"); a.ld_part = pl;
      a.F = c.fi;
      WG_TRY(run_agg_x(c, a, p->bt, st, xl, hk));
    }
    return WG_OK;
  }
  // ---- G path
  if (pre && sage && G && G->W_self) WG_TRY(gemm_tn(c.dt, c.nr, c.fi, c.fo, x_own, A->ldx, dT, lddT, G->W_self, tn, st));
  if (!post) return WG_OK;
  void* gbuf = L.at<void>(ws, "g");
  {
    AggArgs a = agg_base(c, p->bt, c.g->bwd);
    a.table = gtab; a.ld_tab = ldg;
    a.gscale = fold ? nullptr : rs; a.rscale = gs;
    if (gin) { a.self_tab = off(gtab, c.vb, ldg, c.s); a.ld_self = ldg; a.self_coef = 1.f + d.gin_eps; }
    a.out = gbuf; a.ld_out = c.po;
    a.partial = L.at<float>(ws, "partT"); a.ld_part = pl;
    a.F = c.fo;
    WG_TRY(run_agg_x(c, a, p->bt, st, xl, hk));
  }
  if (G && G->W) WG_TRY(gemm_tn(c.dt, c.nr, c.fi, c.fo, x_own, A->ldx, gbuf, c.po, G->W, tn, st));
  if (d.need_dx) {
    GemmPart parts[2];
    int np = 0;
    parts[np++] = GemmPart{gbuf, c.po, w, c.po, c.fo, (int)c.wrows_i};
    if (sage) parts[np++] = GemmPart{dT, lddT, wsb, c.po, c.fo, (int)c.wrows_i};
    GemmEpi e;
    e.D = A->dx; e.ldd = A->lddx;
    e.mask_ref = A->dx_mask; e.ld_mask = A->ld_dx_mask;
    WG_TRY(gemm_nt(c.dt, c.nr, (int)rup(c.fi, 16 / c.s), parts, np, e, nullptr, 0, st));
  }
  return WG_OK;
}

}  // namespace wg
