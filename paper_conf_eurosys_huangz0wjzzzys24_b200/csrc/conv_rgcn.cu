// RGCN layer, Eq. (1): h^{l+1}[e.dst] += MLP(h^l[e.src], W^l[e.type]),
// Schlichtkrull et al. [34] (readings Q2): optional c_e = 1/|in_r(v)|,
// self-loop W_0 and bias.
//
// gTasks are (destination tile x relation) blocks (Fig 7(c)(d)).
// Per gTask the plan (a4) chooses:
//   EDGE   (gather-then-transform): one stage-1 row per (dst, relation)
//          segment, S = sum_e c_e x[src_e]; the row is transformed by W_r and
//          contributes once to y[dst];
//   VERTEX (transform-before-gather): one Y row per unique (source, relation)
//          pair over all VERTEX gTasks of the relation (T1 unique extraction,
//          src-id_unique / src-id_map), Y = x[src] W_r computed
//          once (T2 indexing swapping, Index-2D A[B] x C[D] = (A x C)[B, D],
//          P:L1867-1876); every edge contributes c_e Y[map(e)].  The GEMM
//          gathers its A rows straight from x (TMA tile::gather4): the unique
//          rows are never materialised.
// Y rows and EDGE segment rows are laid out grouped by relation (each group
// padded to 128 rows), so one grouped GEMM per block applies W_r to every row
// of group r ("a batch of K src rows becomes a matrix-matrix product",
// P:L2159-2189); stage 3 is the contribution-list gather-reduce into
// destination rows.  Backward mirrors this on the transposed partition
// (source tile x relation): G = sum over (src, relation) segments of c_e
// dy[dst], dX = G W_r^T (grouped), dx = sum over a source's segments;
// dW_r = X_g^T G over group r, X_g = x[src] of every (src, relation) row
// (a copy in source order, k_xg_scatter: a TMA gather4 K-row load of 32-bit
// MN-major tiles measured 2.5x slower than this copy + tile loads).
// Stage buffers (segment sums, Y, G, dX) round-trip HBM; DESIGN.md "RGCN".
#include <algorithm>
#include <numeric>
#include <random>

#include "plan.h"

namespace wg {

namespace {

constexpr int TILE_M = 128;

struct CsrExec {
  int64_t rows = 0, nnz = 0;
  int64_t* row_ptr = nullptr;
  int32_t* idx = nullptr;
  int32_t* key = nullptr;
  float* escale = nullptr;
  float* rscale = nullptr;
  ItemList items;
  int n_slots = 0;
};

struct RgcnPlan {
  int R = 1;
  int64_t n1v = 0, n1e = 0, n1T = 0; // Y rows, EDGE segment rows, transposed rows (each padded per relation)
  CsrExec f1, f3, b1, b3;
  int32_t* ysrc = nullptr;           // [n1v] source vertex of each Y row (0 in padding)
  int32_t* tile_type_v = nullptr;    // [n1v / 128]
  int32_t* tile_type_e = nullptr;    // [n1e / 128]
  int32_t* tile_typeT = nullptr;     // [n1T / 128]
  // X_g copy (k_xg_scatter): entry i writes x[xg_src[i]] (zeros for -1, the
  // per-relation padding) to X_g row xg_row[i]; entries in source order
  int32_t* xg_src = nullptr;
  int32_t* xg_row = nullptr;
  int64_t n_xg = 0, n_xg_src = 0;   // entries, distinct sources
  std::vector<int64_t> h_group_offT; // [R+1] transposed group row offsets
  TnUnits tn;                        // dW_r work units over the transposed groups
  // Y rows == transposed G rows (every gTask VERTEX, one partition): the
  // forward gathers X_g = x[src] once (saved), the Y GEMM streams it
  // contiguously, and the backward's dW_r GEMM reuses it
  bool share_xg = false;
};

template <typename T>
wg_status up(wg_plan_s* p, const std::vector<T>& h, T** d) {
  *d = nullptr;
  if (h.empty()) return WG_OK;
  void* q = nullptr;
  WG_CK(cudaMalloc(&q, sizeof(T) * h.size()));
  p->allocs.push_back(q);
  WG_CK(cudaMemcpy(q, h.data(), sizeof(T) * h.size(), cudaMemcpyHostToDevice));
  *d = static_cast<T*>(q);
  return WG_OK;
}

// Work items over a generic CSR: consecutive rows grouped until min(E_max,
// ITEM_EDGES) entries or ITEM_ROWS rows; rows with more than E_max entries
// become SPLIT chunks.  Stage rows are short (C3: ~1.4 edges per (dst,
// relation) row), so items span many rows: a CTA must stream thousands of
// edges to amortise its pipeline fill (128-row items ran at 29% of HBM).
wg_status build_exec(wg_plan_s* p, const std::vector<int64_t>& rp, const std::vector<int32_t>& idx,
                     const std::vector<float>* es, const std::vector<float>* rs, int64_t E_max, CsrExec* X) {
  X->rows = (int64_t)rp.size() - 1;
  X->nnz = rp.back();
  std::vector<int32_t> key(X->nnz);
  for (int64_t r = 0; r < X->rows; ++r)
    for (int64_t e = rp[r]; e < rp[r + 1]; ++e) key[e] = (int32_t)r;
  WG_TRY(up(p, rp, &X->row_ptr));
  WG_TRY(up(p, idx, &X->idx));
  WG_TRY(up(p, key, &X->key));
  if (es) WG_TRY(up(p, *es, &X->escale));
  if (rs) WG_TRY(up(p, *rs, &X->rscale));
  std::vector<std::pair<int64_t, WorkItem>> L;
  int slot = 0;
  ItemList& IL = X->items;
  // at least ~6 items per SM when the CSR is small (a few EDGE-plan gTasks)
  constexpr int64_t ITEM_ROWS = 4096, ITEM_EDGES = 4096;
  const int64_t item_edges = std::min(E_max, std::max<int64_t>(512, std::min(ITEM_EDGES, X->nnz / (148 * 6))));
  int64_t lo = 0;
  auto close = [&](int64_t hi) {
    if (hi <= lo) return;
    WorkItem w{};
    w.row_lo = (int32_t)lo; w.row_hi = (int32_t)hi; w.e_lo = rp[lo]; w.e_hi = rp[hi];
    w.split_slot = -1; w.task = -1;
    L.push_back({w.e_hi - w.e_lo, w});
    IL.n_edges += w.e_hi - w.e_lo;
    IL.n_rows += hi - lo;
  };
  for (int64_t r = 0; r < X->rows; ++r) {
    const int64_t deg = rp[r + 1] - rp[r];
    if (deg > E_max) {
      close(r);
      IL.hs.push_back(SplitRow{(int32_t)r, slot, 0, 0});
      for (int64_t c = rp[r]; c < rp[r + 1]; c += E_max) {
        WorkItem w{};
        w.row_lo = (int32_t)r; w.row_hi = (int32_t)r + 1; w.e_lo = c; w.e_hi = std::min(c + E_max, rp[r + 1]);
        w.split_slot = slot++; w.task = -1;
        L.push_back({INT64_MAX / 2 + (w.e_hi - w.e_lo), w});
        IL.hs.back().n_slots++;
        IL.n_edges += w.e_hi - w.e_lo;
      }
      lo = r + 1;
      continue;
    }
    if (rp[r + 1] - rp[lo] > item_edges || r - lo >= ITEM_ROWS) {
      close(r);
      lo = r;
    }
  }
  close(X->rows);
  std::stable_sort(L.begin(), L.end(), [](const auto& a, const auto& b) { return a.first > b.first; });
  for (auto& e : L) IL.h.push_back(e.second);
  IL.n = (int)IL.h.size();
  IL.n_split = (int)IL.hs.size();
  WG_TRY(up(p, IL.h, &IL.d));
  WG_TRY(up(p, IL.hs, &IL.split));
  X->n_slots = slot;
  return WG_OK;
}

template <typename T>
wg_status down(const T* d, int64_t n, std::vector<T>& h) {
  h.resize(n);
  if (n) WG_CK(cudaMemcpy(h.data(), d, sizeof(T) * n, cudaMemcpyDeviceToHost));
  return WG_OK;
}

// X_g = x[src] per transposed (source, relation) row, written in source
// order: consecutive entries read the same or adjacent x rows (L1 / L2 hits)
// and write whole scattered rows, so DRAM reads x about once instead of once
// per (source, relation) row (the row-order gather read 8 GB at C3 layer 1
// with 2.3 % L2 hits).  Persistent grid; a warp copies 32 / vpr entries per
// step (lane = one 16-byte vector), UNR steps of loads in flight.
constexpr int XG_UNR = 4;
__global__ void __launch_bounds__(256) k_xg_scatter(const int4* __restrict__ x, int64_t ldx16,
                                                    const int32_t* __restrict__ src, const int32_t* __restrict__ row,
                                                    int64_t n, int vpr, int4* out, int64_t ldo16) {
  const int lane = threadIdx.x & 31;
  const int lpe = min(vpr, 32);                   // lanes per entry
  const int per = 32 / lpe;                       // entries per warp step
  const int sub = lane / lpe, l = lane - sub * lpe;
  const bool act = sub < per;
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
  const int64_t w0 = blockIdx.x * (int64_t)(blockDim.x >> 5) + (threadIdx.x >> 5);
  for (int64_t base = w0 * per * XG_UNR; base < n; base += nw * per * XG_UNR) {
    for (int v = l; v < vpr; v += 32) {           // rows wider than 512 B: 32-vector chunks
      int4 val[XG_UNR];
      int32_t dr[XG_UNR];
#pragma unroll
      for (int k = 0; k < XG_UNR; ++k) {
        const int64_t i = base + (int64_t)k * per + sub;
        dr[k] = -1;
        val[k] = make_int4(0, 0, 0, 0);
        if (act && i < n) {
          const int32_t u = src[i];
          dr[k] = row[i];
          if (u >= 0) val[k] = __ldg(x + (int64_t)u * ldx16 + v);
        }
      }
#pragma unroll
      for (int k = 0; k < XG_UNR; ++k)
        if (dr[k] >= 0) out[(int64_t)dr[k] * ldo16 + v] = val[k];
    }
  }
}

wg_status xg_scatter(const RgcnPlan* rp, wg_dtype dt, const void* x, int64_t ldx, int f_in, void* xg, int64_t ldo,
                     cudaStream_t st) {
  if (rp->n_xg == 0) return WG_OK;
  const int s = dsize(dt);
  const int vpr = (int)cdiv((int64_t)f_in * s, 16);
  WG_REQ((ldx * s) % 16 == 0 && (ldo * s) % 16 == 0, WG_ERR_INVALID, "X_g copy: pitch not a 16-byte multiple");
  // algorithmic bytes: every X_g row written, each distinct source row read once, 8 B of ids per entry
  ProfScope ps(PK_AGG, st, (double)rp->n_xg * (vpr * 16 + 8.0) + (double)rp->n_xg_src * vpr * 16, 0.0);
  WG_LAUNCH(k_xg_scatter, 148 * 8, 256, 0, st, static_cast<const int4*>(x), ldx * s / 16, rp->xg_src, rp->xg_row,
            rp->n_xg, vpr, static_cast<int4*>(xg), ldo * s / 16);
  return WG_OK;
}

AggArgs exec_args(const CsrExec& X, int64_t E_max) {
  AggArgs a{};
  a.items = X.items.d;
  a.n_items = X.items.n;
  a.row_ptr = X.row_ptr;
  a.idx = X.idx;
  a.key = X.key;
  a.escale = X.escale;
  a.rscale = X.rscale;
  a.row_base = 0;
  a.self_coef = 1.f;
  a.E_max = E_max;
  a.n_edges = X.items.n_edges;
  a.n_rows = X.items.n_rows;
  return a;
}

CombineArgs comb(const AggArgs& a, const CsrExec& X) {
  CombineArgs b{};
  b.rows = X.items.split; b.n_rows = X.items.n_split;
  b.partial = a.partial; b.ld_part = a.ld_part;
  b.rscale = a.rscale; b.row_base = a.row_base;
  b.self_tab = a.self_tab; b.ld_self = a.ld_self; b.self_coef = a.self_coef;
  b.bias = a.bias; b.relu = a.relu; b.mask_ref = a.mask_ref; b.ld_mask = a.ld_mask;
  b.out = a.out; b.ld_out = a.ld_out;
  b.F = a.F; b.plan_filter = -1;
  return b;
}

wg_status run(wg_dtype dt, const AggArgs& a, const CsrExec& X, cudaStream_t s) {
  WG_TRY(launch_agg(dt, a, s));
  WG_TRY(launch_combine(dt, comb(a, X), s));
  return WG_OK;
}

}  // namespace

// -------------------------------------------------------------------- plan
wg_status rgcn_plan(wg_plan_s* p, cudaStream_t) {
  wg_graph_s* g = p->g;
  const wg_conv_desc& d = p->d;
  // 1-D partition: this rank owns rows [vb, ve); its forward
  // side holds their in-edges, its transposed side their out-edges; x / dT
  // tables are read with global row ids (replicated / all-gathered), outputs
  // are written for the owned rows only.
  // E = 0: no edge carries a type, but the R relation gradients still exist (all zero)
  const int R = (g->by_type || g->E_total == 0) ? g->R : 1;
  const int64_t E = g->fwd.E, Eb = g->bwd.E, V = g->V, vb = g->vb, nr = g->ve - g->vb;
  auto* rp = new RgcnPlan();
  rp->R = R;
  p->rg = rp;
  p->pi = pitch(d.f_in, d.dtype);
  p->po = pitch(d.f_out, d.dtype);
  p->bwd_path = 1;    // the backward exchange table is dT (f_out wide)
  // ---- host copies of the forward / transposed sorted edge arrays
  std::vector<int32_t> fk, fi_, ft, fperm, bk, bi, bt, bperm;
  WG_TRY(down(g->fwd.key, E, fk));
  WG_TRY(down(g->fwd.idx, E, fi_));
  WG_TRY(down(g->fwd.perm, E, fperm));
  WG_TRY(down(g->bwd.key, Eb, bk));
  WG_TRY(down(g->bwd.idx, Eb, bi));
  WG_TRY(down(g->bwd.perm, Eb, bperm));
  if (g->by_type) {
    WG_TRY(down(g->fwd.type, E, ft));
    WG_TRY(down(g->bwd.type, Eb, bt));
  } else {
    ft.assign(E, 0);
    bt.assign(Eb, 0);
  }
  // per-edge coefficient c_e (forward / transposed order): 1 or 1/|in_r(dst)|
  // (global counts, graph.cu rel_counts)
  std::vector<float> coef_f(E, 1.f), coef_b(Eb, 1.f);
  if (d.norm == WG_NORM_RIGHT) {
    std::vector<int32_t> cnt;
    if (g->by_type) {
      WG_TRY(down(g->rel_cnt, g->E_total, cnt));
    } else {   // one relation: |in_r(v)| = deg_in(v)
      std::vector<int32_t> din;
      WG_TRY(down(g->deg_in, V, din));
      cnt.resize(1);
      for (int64_t i = 0; i < E; ++i) coef_f[i] = 1.f / (float)std::max(1, din[fk[i]]);
      for (int64_t i = 0; i < Eb; ++i) coef_b[i] = 1.f / (float)std::max(1, din[bi[i]]);
    }
    if (g->by_type) {
      for (int64_t i = 0; i < E; ++i) coef_f[i] = 1.f / (float)cnt[fperm[i]];
      for (int64_t i = 0; i < Eb; ++i) coef_b[i] = 1.f / (float)cnt[bperm[i]];
    }
  }
  const auto& tasks = g->fwd.h_tasks;
  const int64_t nt = (int64_t)tasks.size();
  // ---- plan bits (a4)
  p->plan_bits.assign(nt, 0);
  {
    const int s = dsize(d.dtype);
    const int64_t A = rup((int64_t)d.f_in * s, 32), B = rup((int64_t)d.f_out * s, 32);
    std::mt19937_64 rng(d.policy_seed);
    // Y rows are unique per (source, relation) over ALL VERTEX gTasks of the
    // relation, so a gTask's share of the Y transform is amortised:
    // n_uniq_src(g) * U_r / S_r rows (U_r distinct sources of relation r,
    // S_r = sum of n_uniq_src over its gTasks)
    std::vector<int64_t> U(R, 0), S(R, 0);
    {
      std::vector<uint64_t> seen((size_t)cdiv((int64_t)R * V, 64), 0);
      for (int64_t i = 0; i < E; ++i) {
        const uint64_t bit = (uint64_t)ft[i] * (uint64_t)V + (uint64_t)fi_[i];
        uint64_t& w = seen[bit >> 6];
        const uint64_t m = 1ull << (bit & 63);
        if (!(w & m)) { w |= m; ++U[ft[i]]; }
      }
      for (int64_t t = 0; t < nt; ++t) S[tasks[t].type] += tasks[t].n_uniq_src;
    }
    for (int64_t t = 0; t < nt; ++t) {
      const wg_task& k = tasks[t];
      int64_t nseg = 0;
      for (int64_t i = k.e_begin; i < k.e_end; ++i) nseg += (i == k.e_begin || fk[i] != fk[i - 1]);
      const int64_t ne = k.e_end - k.e_begin, nu = k.n_uniq_src;
      // EDGE: gather f_in rows, then per (dst, relation) segment the S row
      // write + GEMM read, the T row write + stage-3 read
      const int64_t te = ne * (A + 4) + nseg * (2 * A + 2 * B + 4);
      // VERTEX: the amortised Y rows (gathered f_in row read + f_out row
      // write), then every edge reads its f_out-wide Y row
      const int64_t ny = S[k.type] > 0 ? nu * U[k.type] / S[k.type] : nu;
      const int64_t tv = ny * (A + B) + ne * (B + 8);
      uint8_t b = 0;
      if (d.policy == WG_PLAN_ALL_VERTEX) b = 1;
      else if (d.policy == WG_PLAN_RANDOM) b = (uint8_t)(rng() & 1);
      else if (d.policy == WG_PLAN_AUTO) b = tv < te ? 1 : 0;
      p->plan_bits[t] = b;
    }
    for (int64_t t = 1; t < nt; ++t)
      if ((tasks[t].flags & WG_TASK_SPLIT) && (tasks[t - 1].flags & WG_TASK_SPLIT) && tasks[t].d_lo == tasks[t - 1].d_lo &&
          tasks[t].type == tasks[t - 1].type)
        p->plan_bits[t] = p->plan_bits[t - 1];
    p->n_vert_tasks = std::count(p->plan_bits.begin(), p->plan_bits.end(), 1);
    p->n_edge_tasks = nt - p->n_vert_tasks;
  }
  // ---- forward rows: EDGE segment rows and VERTEX unique (src, relation) rows, grouped by relation
  struct Row1 { int64_t ent_b, ent_e; float rs; };
  std::vector<std::vector<Row1>> rows1(R);
  std::vector<std::vector<int32_t>> ents(R);                 // per-type EDGE stage-1 entries (source ids)
  std::vector<std::vector<int32_t>> uniq(R);                 // per-type VERTEX sources (sorted, unique)
  struct Contrib { int32_t dst; int32_t type; int64_t row; float c; bool vert; };
  std::vector<Contrib> contrib;
  contrib.reserve(E);
  // On one partition with >= 90% of the edges in VERTEX gTasks, the Y rows
  // cover every (source, relation) pair of the graph: the few extra rows
  // (sources reached only through EDGE gTasks) make the Y block identical to
  // the transposed G rows, so X_g is shared with the backward (share_xg)
  int64_t e_vert = 0;
  for (int64_t t = 0; t < nt; ++t)
    if (p->plan_bits[t] == 1) e_vert += tasks[t].e_end - tasks[t].e_begin;
  const bool y_all = nr == g->V && e_vert > 0 && e_vert * 10 >= E * 9;
  for (int64_t t = 0; t < nt; ++t)
    if (p->plan_bits[t] == 1 || y_all)
      for (int64_t i = tasks[t].e_begin; i < tasks[t].e_end; ++i) uniq[tasks[t].type].push_back(fi_[i]);
  for (int r = 0; r < R; ++r) {
    std::sort(uniq[r].begin(), uniq[r].end());
    uniq[r].erase(std::unique(uniq[r].begin(), uniq[r].end()), uniq[r].end());
  }
  int64_t open_seg_dst = -1, open_seg_type = -1;           // EDGE segment continuing across SPLIT tasks
  for (int64_t t = 0; t < nt; ++t) {
    const wg_task& k = tasks[t];
    const int r = k.type;
    if (p->plan_bits[t] == 0) {
      for (int64_t i = k.e_begin; i < k.e_end;) {
        int64_t j = i;
        while (j < k.e_end && fk[j] == fk[i]) ++j;
        const bool cont = (i == k.e_begin) && open_seg_dst == fk[i] && open_seg_type == r && (k.flags & WG_TASK_SPLIT);
        if (!cont) {
          const float rs = coef_f[i];   // segment (dst, r): every edge has the same c_e
          rows1[r].push_back(Row1{(int64_t)ents[r].size(), (int64_t)ents[r].size(), rs});
          contrib.push_back(Contrib{fk[i] - (int32_t)vb, r, (int64_t)rows1[r].size() - 1, 1.f, false});
        }
        for (int64_t q = i; q < j; ++q) ents[r].push_back(fi_[q]);
        rows1[r].back().ent_e = (int64_t)ents[r].size();
        open_seg_dst = fk[i];
        open_seg_type = r;
        i = j;
      }
    } else {
      open_seg_dst = -1;
      for (int64_t i = k.e_begin; i < k.e_end; ++i) {
        const int64_t m = std::lower_bound(uniq[r].begin(), uniq[r].end(), fi_[i]) - uniq[r].begin();
        contrib.push_back(Contrib{fk[i] - (int32_t)vb, r, m, coef_f[i], true});
      }
    }
  }
  // Y block: group r at base_v[r]; EDGE block: group r at base_e[r]; each padded to 128 rows
  std::vector<int64_t> base_v(R + 1, 0), base_e(R + 1, 0);
  for (int r = 0; r < R; ++r) {
    base_v[r + 1] = base_v[r] + rup((int64_t)uniq[r].size(), TILE_M);
    base_e[r + 1] = base_e[r] + rup((int64_t)rows1[r].size(), TILE_M);
  }
  rp->n1v = base_v[R];
  rp->n1e = base_e[R];
  {
    std::vector<int32_t> ys(rp->n1v, 0), tt(rp->n1v / TILE_M);
    for (int r = 0; r < R; ++r) {
      std::copy(uniq[r].begin(), uniq[r].end(), ys.begin() + base_v[r]);
      for (int64_t t = base_v[r] / TILE_M; t < base_v[r + 1] / TILE_M; ++t) tt[t] = r;
    }
    WG_TRY(up(p, ys, &rp->ysrc));
    WG_TRY(up(p, tt, &rp->tile_type_v));
  }
  {
    std::vector<int64_t> rpv(rp->n1e + 1, 0);
    std::vector<int32_t> idx;
    std::vector<float> rs(rp->n1e, 1.f);
    bool any_rs = false;
    int64_t row = 0;
    for (int r = 0; r < R; ++r) {
      for (const Row1& w : rows1[r]) {
        for (int64_t q = w.ent_b; q < w.ent_e; ++q) idx.push_back(ents[r][q]);
        rs[row] = w.rs;
        any_rs |= w.rs != 1.f;
        rpv[++row] = (int64_t)idx.size();
      }
      while (row < base_e[r + 1]) rpv[++row] = (int64_t)idx.size();
    }
    WG_TRY(build_exec(p, rpv, idx, nullptr, any_rs ? &rs : nullptr, g->E_max, &rp->f1));
    std::vector<int32_t> tt(rp->n1e / TILE_M);
    for (int r = 0; r < R; ++r)
      for (int64_t t = base_e[r] / TILE_M; t < base_e[r + 1] / TILE_M; ++t) tt[t] = r;
    WG_TRY(up(p, tt, &rp->tile_type_e));
  }
  // stage 3: contributions per destination row (sorted by dst, then stage row);
  // stage rows: [Y block | EDGE block]
  {
    for (auto& c : contrib) c.row += c.vert ? base_v[c.type] : rp->n1v + base_e[c.type];
    std::stable_sort(contrib.begin(), contrib.end(), [](const Contrib& a, const Contrib& b) {
      return a.dst != b.dst ? a.dst < b.dst : a.row < b.row;
    });
    std::vector<int64_t> rpv(nr + 1, 0);
    std::vector<int32_t> idx(contrib.size());
    std::vector<float> es(contrib.size());
    bool any = false;
    for (size_t i = 0; i < contrib.size(); ++i) {
      rpv[contrib[i].dst + 1]++;
      idx[i] = (int32_t)contrib[i].row;
      es[i] = contrib[i].c;
      any |= es[i] != 1.f;
    }
    for (int64_t v = 0; v < nr; ++v) rpv[v + 1] += rpv[v];
    WG_TRY(build_exec(p, rpv, idx, any ? &es : nullptr, nullptr, g->E_max, &rp->f3));
  }
  // ---- transposed: (src, relation) segments grouped by relation
  {
    std::vector<std::vector<std::pair<int64_t, int64_t>>> segs(R);   // [b, e) in transposed order
    std::vector<std::vector<int32_t>> seg_src(R);
    for (int64_t i = 0; i < Eb;) {
      int64_t j = i;
      while (j < Eb && bk[j] == bk[i] && bt[j] == bt[i]) ++j;
      segs[bt[i]].push_back({i, j});
      seg_src[bt[i]].push_back(bk[i]);
      i = j;
    }
    std::vector<int64_t> baseT(R + 1, 0);
    for (int r = 0; r < R; ++r) baseT[r + 1] = baseT[r] + rup((int64_t)segs[r].size(), TILE_M);
    rp->n1T = baseT[R];
    std::vector<int64_t> rpv(rp->n1T + 1, 0), rpg(rp->n1T + 1, 0);
    std::vector<int32_t> idx, gidx;
    std::vector<float> es;
    idx.reserve(Eb);
    es.reserve(Eb);
    bool any = false;
    struct SC { int32_t src; int64_t row; };
    std::vector<SC> sc;
    int64_t row = 0;
    for (int r = 0; r < R; ++r) {
      for (size_t s = 0; s < segs[r].size(); ++s) {
        for (int64_t q = segs[r][s].first; q < segs[r][s].second; ++q) {
          idx.push_back(bi[q]);
          const float c = coef_b[q];
          es.push_back(c);
          any |= c != 1.f;
        }
        gidx.push_back(seg_src[r][s]);
        sc.push_back(SC{seg_src[r][s], row});
        rpg[row + 1] = (int64_t)gidx.size();
        rpv[++row] = (int64_t)idx.size();
      }
      while (row < baseT[r + 1]) { rpg[row + 1] = (int64_t)gidx.size(); rpv[++row] = (int64_t)idx.size(); }
    }
    WG_TRY(build_exec(p, rpv, idx, any ? &es : nullptr, nullptr, g->E_max, &rp->b1));
    std::vector<int32_t> tt(rp->n1T / TILE_M);
    for (int r = 0; r < R; ++r)
      for (int64_t t = baseT[r] / TILE_M; t < baseT[r + 1] / TILE_M; ++t) tt[t] = r;
    WG_TRY(up(p, tt, &rp->tile_typeT));
    rp->h_group_offT = baseT;
    {
      std::vector<int4> units;
      std::vector<int32_t> uoff;
      const int64_t tiles = cdiv(d.f_in, 128) * cdiv(d.f_out, d.dtype == WG_F32 ? 128 : 256);
      make_tn_units(baseT, std::max<int64_t>(R, 4 * 148 / tiles), 128 / dsize(d.dtype), &units, &uoff);
      int4* du = nullptr;
      int32_t* duo = nullptr;
      WG_TRY(up(p, units, &du));
      WG_TRY(up(p, uoff, &duo));
      rp->tn.units = du; rp->tn.unit_off = duo;
      rp->tn.n_units = (int)units.size(); rp->tn.groups = R; rp->tn.align = TILE_M; rp->tn.k_total = baseT[R];
    }
    rp->share_xg = nr == g->V && rp->n1v == rp->n1T;
    for (int r = 0; r < R && rp->share_xg; ++r) rp->share_xg = uniq[r] == seg_src[r];
    std::stable_sort(sc.begin(), sc.end(), [](const SC& a, const SC& b) {
      return a.src != b.src ? a.src < b.src : a.row < b.row;
    });
    {
      std::vector<int32_t> xs, xr;
      xs.reserve(rp->n1T);
      xr.reserve(rp->n1T);
      for (size_t i = 0; i < sc.size(); ++i) {
        xs.push_back(sc[i].src);
        xr.push_back((int32_t)sc[i].row);
        rp->n_xg_src += i == 0 || sc[i].src != sc[i - 1].src;
      }
      for (int64_t r = 0; r < rp->n1T; ++r)
        if (rpg[r + 1] == rpg[r]) { xs.push_back(-1); xr.push_back((int32_t)r); }
      rp->n_xg = (int64_t)xs.size();
      WG_TRY(up(p, xs, &rp->xg_src));
      WG_TRY(up(p, xr, &rp->xg_row));
    }
    std::vector<int64_t> rp3(nr + 1, 0);
    std::vector<int32_t> idx3(sc.size());
    for (size_t i = 0; i < sc.size(); ++i) { rp3[sc[i].src - vb + 1]++; idx3[i] = (int32_t)sc[i].row; }
    for (int64_t v = 0; v < nr; ++v) rp3[v + 1] += rp3[v];
    WG_TRY(build_exec(p, rp3, idx3, nullptr, nullptr, g->E_max, &rp->b3));
  }
  // ---- buffers
  const int s = dsize(d.dtype);
  const int64_t rows_o = rup(d.f_out, 16), rows_i = rup(d.f_in, 16);
  const int64_t pl = rup(std::max(d.f_in, d.f_out), 8);
  Layout& S = p->saved;
  Layout& W = p->ws;
  S = Layout();
  W = Layout();
  S.add("none", 1);
  if (rp->share_xg) S.add("xg", (size_t)rp->n1T * p->pi * s);
  W.add("wt", (size_t)R * rows_o * p->pi * s);          // stacked W_r^T
  W.add("w", (size_t)R * rows_i * p->po * s);           // stacked W_r
  W.add("w0t", (size_t)rows_o * p->pi * s);
  W.add("w0", (size_t)rows_i * p->po * s);
  W.add("a1", (size_t)std::max<int64_t>(rp->n1e, 1) * p->pi * s);
  W.add("t1", (size_t)std::max<int64_t>(rp->n1v + rp->n1e, 1) * p->po * s);
  W.add("self", (size_t)nr * p->po * s);
  W.add("part", sizeof(float) * std::max({1, rp->f1.n_slots, rp->f3.n_slots, rp->b1.n_slots, rp->b3.n_slots}) * pl);
  W.add("xg", (size_t)rp->n1T * p->pi * s);
  W.add("dt", (size_t)nr * p->po * s);
  W.add("gt", (size_t)rp->n1T * p->po * s);
  W.add("dxt", (size_t)rp->n1T * p->pi * s);
  W.add("dxs", (size_t)nr * p->pi * s);
  W.add("colsum", bias_grad_scratch(nr, (int)p->po));
  W.add("tn", std::max(gemm_tn_scratch(nr, d.f_in, d.f_out), gemm_tn_grouped_scratch(rp->tn.n_units, d.f_in, d.f_out)));
  // the forward gTask work items are not used by RGCN (stage CSRs replace them)
  return WG_OK;
}

void rgcn_plan_free(wg_plan_s* p) {
  delete static_cast<RgcnPlan*>(p->rg);
  p->rg = nullptr;
}

// ----------------------------------------------------------------- forward
wg_status rgcn_forward(wg_plan_s* p, const wg_params* P, const wg_fwd_args* A, cudaStream_t st) {
  const wg_conv_desc& d = p->d;
  wg_graph_s* g = p->g;
  auto* rp = static_cast<RgcnPlan*>(p->rg);
  const wg_dtype dt = d.dtype;
  const int s = dsize(dt), R = rp->R;
  WG_REQ(P->W && A->x && A->y && A->workspace, WG_ERR_INVALID, "RGCN forward: null argument");
  WG_REQ(!d.self_loop || P->W_self, WG_ERR_INVALID, "self_loop needs W_self");
  // 1-D partition: x holds every row (the caller all-gathers it); nothing to
  // exchange before the forward, so PRE is a no-op and POST = ALL
  if (A->phase == WG_PHASE_PRE) return WG_OK;
  const Layout& L = p->ws;
  void* ws = A->workspace;
  const int64_t V = g->V, vb = g->vb, nr = g->ve - g->vb, rows_o = rup(d.f_out, 16),
                pl = rup(std::max(d.f_in, d.f_out), 8);
  ProfScope ps(PK_RGCN, st, 0.0, 0.0);
  void* wt = L.at<void>(ws, "wt");
  WG_TRY(prep_weight_batched(dt, P->W, R, d.f_in, d.f_out, 1, wt, p->pi, (int)rows_o, st));
  // stage 1 (EDGE gTasks): segment sums S = sum c_e x[src] into the EDGE block rows
  void* a1 = L.at<void>(ws, "a1");
  if (rp->n1e) {
    AggArgs a = exec_args(rp->f1, g->E_max);
    a.table = A->x; a.ld_tab = A->ldx;
    a.out = a1; a.ld_out = p->pi;
    a.partial = L.at<float>(ws, "part"); a.ld_part = pl;
    a.F = d.f_in;
    WG_TRY(run(dt, a, rp->f1, st));
  }
  // stage 2: grouped GEMMs  T1[Y block, group r] = x[ysrc] W_r (A rows gathered
  // from x) and T1[EDGE block, group r] = S W_r
  void* t1 = L.at<void>(ws, "t1");
  if (rp->n1v && rp->share_xg) {
    WG_REQ(A->saved, WG_ERR_INVALID, "RGCN forward: saved is NULL");
    void* xg = p->saved.at<void>(A->saved, "xg");
    WG_TRY(xg_scatter(rp, dt, A->x, A->ldx, d.f_in, xg, p->pi, st));
    GemmPart part{xg, p->pi, wt, p->pi, d.f_in, d.f_out};
    part.tile_group = rp->tile_type_v; part.group_rows = (int)rows_o; part.groups = R;
    GemmEpi e;
    e.D = t1; e.ldd = p->po;
    WG_TRY(gemm_nt(dt, rp->n1v, (int)rup(d.f_out, 16 / s), &part, 1, e, nullptr, 0, st));
  } else if (rp->n1v) {
    GemmPart part{A->x, A->ldx, wt, p->pi, d.f_in, d.f_out};
    part.tile_group = rp->tile_type_v; part.group_rows = (int)rows_o; part.groups = R;
    part.a_rows = rp->ysrc; part.a_table_rows = V;
    GemmEpi e;
    e.D = t1; e.ldd = p->po;
    WG_TRY(gemm_nt(dt, rp->n1v, (int)rup(d.f_out, 16 / s), &part, 1, e, nullptr, 0, st));
  }
  if (rp->n1e) {
    GemmPart part{a1, p->pi, wt, p->pi, d.f_in, d.f_out};
    part.tile_group = rp->tile_type_e; part.group_rows = (int)rows_o; part.groups = R;
    GemmEpi e;
    e.D = static_cast<char*>(t1) + (size_t)rp->n1v * p->po * s; e.ldd = p->po;
    WG_TRY(gemm_nt(dt, rp->n1e, (int)rup(d.f_out, 16 / s), &part, 1, e, nullptr, 0, st));
  }
  // self loop x W_0
  void* self = nullptr;
  if (d.self_loop) {
    void* w0t = L.at<void>(ws, "w0t");
    WG_TRY(prep_weight(dt, P->W_self, d.f_in, d.f_out, 1, w0t, p->pi, (int)rows_o, st));
    self = L.at<void>(ws, "self");
    const char* x_own = static_cast<const char*>(A->x) + (size_t)vb * A->ldx * s;
    GemmPart part{x_own, A->ldx, w0t, p->pi, d.f_in, (int)rows_o};
    GemmEpi e;
    e.D = self; e.ldd = p->po;
    WG_TRY(gemm_nt(dt, nr, (int)rup(d.f_out, 16 / s), &part, 1, e, nullptr, 0, st));
  }
  // stage 3: y[v] = sum of contributions (+ self + bias), ReLU
  {
    AggArgs a = exec_args(rp->f3, g->E_max);
    a.table = t1; a.ld_tab = p->po;
    a.self_tab = self; a.ld_self = p->po;
    a.bias = d.bias ? P->bias : nullptr;
    a.relu = d.fuse_relu;
    a.out = A->y; a.ld_out = A->ldy;
    a.partial = L.at<float>(ws, "part"); a.ld_part = pl;
    a.F = d.f_out;
    WG_TRY(run(dt, a, rp->f3, st));
  }
  return WG_OK;
}

// ---------------------------------------------------------------- backward
wg_status rgcn_backward(wg_plan_s* p, const wg_params* P, const wg_bwd_args* A, const wg_grads* G, cudaStream_t st,
                        const XHook* hk) {
  const wg_conv_desc& d = p->d;
  wg_graph_s* g = p->g;
  auto* rp = static_cast<RgcnPlan*>(p->rg);
  const wg_dtype dt = d.dtype;
  const int s = dsize(dt), R = rp->R;
  WG_REQ(P->W && A->dy && A->x && A->workspace, WG_ERR_INVALID, "RGCN backward: null argument");
  const bool mask_dy = d.fuse_relu && !A->dy_masked;
  WG_REQ(!mask_dy || A->y, WG_ERR_INVALID, "fuse_relu backward needs y");
  WG_REQ(!d.need_dx || A->dx, WG_ERR_INVALID, "need_dx but dx is NULL");
  const bool pre = A->phase != WG_PHASE_POST, post = A->phase != WG_PHASE_PRE;
  const Layout& L = p->ws;
  void* ws = A->workspace;
  const int64_t vb = g->vb, nr = g->ve - g->vb, rows_i = rup(d.f_in, 16), pl = rup(std::max(d.f_in, d.f_out), 8);
  const bool dist = nr != g->V;
  WG_REQ(!dist || A->xchg, WG_ERR_INVALID, "RGCN backward on a 1-D partition needs the dT exchange table");
  ProfScope ps(PK_RGCN, st, 0.0, 0.0);
  const char* x_own = static_cast<const char*>(A->x) + (size_t)vb * A->ldx * s;
  // dT = dy (masked by the fused ReLU): this rank's rows; the transposed
  // gather reads dT of every row -- the exchange table when distributed
  void* dt_own = nullptr;                       // written rows (nullptr: dT is dy itself)
  int64_t ld_own = p->po;
  if (A->xchg) { dt_own = static_cast<char*>(A->xchg) + (size_t)vb * A->ld_xchg * s; ld_own = A->ld_xchg; }
  else if (mask_dy) dt_own = L.at<void>(ws, "dt");
  const void* dT = dt_own ? dt_own : A->dy;     // own rows
  const int64_t lddT = dt_own ? ld_own : A->lddy;
  const void* dT_tab = A->xchg ? A->xchg : dT;  // every row (global ids)
  const int64_t ld_tab = A->xchg ? A->ld_xchg : lddT;
  void* dxs = d.self_loop ? L.at<void>(ws, "dxs") : nullptr;
  if (pre) {
    if (dt_own || (G && d.bias))
      WG_TRY(bias_grad_mask(dt, nr, d.f_out, A->dy, A->lddy, mask_dy ? A->y : nullptr, A->ldy, dt_own, ld_own,
                            (G && d.bias) ? G->bias : nullptr, L.at<float>(ws, "colsum"), st));
    if (d.self_loop && G && G->W_self)
      WG_TRY(gemm_tn(dt, nr, d.f_in, d.f_out, x_own, A->ldx, dT, lddT, G->W_self, L.at<void>(ws, "tn"), st));
    if (d.self_loop && d.need_dx) {   // dx self term dT W_0^T (own rows)
      void* w0 = L.at<void>(ws, "w0");
      WG_TRY(prep_weight(dt, P->W_self, d.f_in, d.f_out, 0, w0, p->po, (int)rows_i, st));
      GemmPart part{dT, lddT, w0, p->po, d.f_out, (int)rows_i};
      GemmEpi e;
      e.D = dxs; e.ldd = p->pi;
      WG_TRY(gemm_nt(dt, nr, (int)rup(d.f_in, 16 / s), &part, 1, e, nullptr, 0, st));
    }
  }
  if (!post) return WG_OK;
  if (hk) hk->wait(0, st);        // distributed: the dT table has arrived
  // stage 1T: G_(u,r) = sum_{e: src u, type r} c_e dT[dst_e]
  void* gt = L.at<void>(ws, "gt");
  {
    AggArgs a = exec_args(rp->b1, g->E_max);
    a.table = dT_tab; a.ld_tab = ld_tab;
    a.out = gt; a.ld_out = p->po;
    a.partial = L.at<float>(ws, "part"); a.ld_part = pl;
    a.F = d.f_out;
    WG_TRY(run(dt, a, rp->b1, st));
  }
  // dW_r = X_g[group r]^T G[group r]   (this rank's out-edges; the caller all-reduces)
  if (G && G->W) {
    void* xg = nullptr;
    if (rp->share_xg) {   // gathered by the forward
      WG_REQ(A->saved, WG_ERR_INVALID, "RGCN backward: saved is NULL");
      xg = p->saved.at<void>(A->saved, "xg");
    } else {
      xg = L.at<void>(ws, "xg");
      WG_TRY(xg_scatter(rp, dt, A->x, A->ldx, d.f_in, xg, p->pi, st));
    }
    WG_TRY(gemm_tn_grouped(dt, rp->tn, d.f_in, d.f_out, xg, p->pi, gt, p->po, G->W, L.at<void>(ws, "tn"), st));
  }
  if (!d.need_dx) return WG_OK;
  // stage 2T: dX_(u,r) = G_(u,r) W_r^T (grouped)
  void* w = L.at<void>(ws, "w");
  WG_TRY(prep_weight_batched(dt, P->W, R, d.f_in, d.f_out, 0, w, p->po, (int)rows_i, st));
  void* dxt = L.at<void>(ws, "dxt");
  {
    GemmPart part{gt, p->po, w, p->po, d.f_out, d.f_in};
    part.tile_group = rp->tile_typeT; part.group_rows = (int)rows_i; part.groups = R;
    GemmEpi e;
    e.D = dxt; e.ldd = p->pi;
    WG_TRY(gemm_nt(dt, rp->n1T, (int)rup(d.f_in, 16 / s), &part, 1, e, nullptr, 0, st));
  }
  // stage 3T: dx[u] = sum_r dX_(u,r) (+ dT W_0^T)
  {
    AggArgs a = exec_args(rp->b3, g->E_max);
    a.table = dxt; a.ld_tab = p->pi;
    a.self_tab = dxs; a.ld_self = p->pi;
    a.out = A->dx; a.ld_out = A->lddx;
    a.mask_ref = A->dx_mask; a.ld_mask = A->ld_dx_mask;
    a.partial = L.at<float>(ws, "part"); a.ld_part = pl;
    a.F = d.f_in;
    WG_TRY(run(dt, a, rp->b3, st));
  }
  return WG_OK;
}

}  // namespace wg
