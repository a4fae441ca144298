// Plan selection (a4) and execution structures.
//
// Cost model ("computation workload, memory access volume, and
// parallelism"; the paper gives no formula): integer
// HBM bytes per gTask and per layer, see choose_plans().  Both plans do the
// same GEMM FLOPs (one row transform per vertex: T1 unique extraction
// P:L1823-1843 + T2 indexing swapping P:L1845-1876 make the VERTEX plan
// transform each source row once), so on these HBM-bound shapes the bytes
// decide.  A / B are the 32-byte padded row bytes of f_in / f_out rows.
#include <algorithm>
#include <random>

#include "plan.h"

namespace wg {

namespace {

// Build work items from one side's gTask table (untyped graphs).
// plan: per task bit (nullptr => all EDGE).  out[0] EDGE items, out[1] VERTEX.
// b_empty: the list that takes rows of no gTask (edgeless tiles, rows beside
// a tile's SPLIT rows) -- one whose pass runs, so their epilogue is written.
void build_items(const wg_graph_s* g, const Side& S, const std::vector<uint8_t>* plan, ItemList* out0,
                 ItemList* out1, int* n_slots, int b_empty = 0) {
  const int64_t T = g->T, vb = g->vb, ve = g->ve;
  const int64_t t0 = vb / T, t1 = cdiv(ve, T);
  size_t ti = 0;
  int slot = 0;
  std::vector<std::pair<int64_t, WorkItem>> lists[2];
  for (int64_t tile = t0; tile < t1; ++tile) {
    const int32_t lo = (int32_t)(tile * T - vb), hi = (int32_t)(std::min<int64_t>((tile + 1) * T, ve) - vb);
    // tasks of this tile
    size_t tj = ti;
    while (tj < S.h_tasks.size() && S.h_tasks[tj].tile == tile) ++tj;
    int32_t cur_lo = lo;
    int64_t cur_task = -1;
    // emit the rows [cur_lo, end) as work items, cut around SPLIT rows
    // (deg > E_max: those rows are produced by their SPLIT chunks + combine)
    auto flush = [&](int32_t end) {
      const int b = cur_task >= 0 ? (plan ? (*plan)[cur_task] : 0) : b_empty;
      int32_t lo = cur_lo;
      for (int32_t r = cur_lo; r <= end; ++r) {
        const bool cut = (r == end) || (S.h_row_ptr[r + 1] - S.h_row_ptr[r] > g->E_max);
        if (!cut) continue;
        if (r > lo) {
          WorkItem w{};
          w.row_lo = lo; w.row_hi = r;
          w.e_lo = S.h_row_ptr[lo]; w.e_hi = S.h_row_ptr[r];
          w.split_slot = -1;
          w.task = (int32_t)cur_task;
          lists[b].push_back({w.e_hi - w.e_lo, w});
          (b ? out1 : out0)->n_edges += w.e_hi - w.e_lo;
          (b ? out1 : out0)->n_rows += r - lo;
        }
        lo = r + 1;
      }
    };
    bool first = true;
    int32_t split_row = -1;
    for (size_t k = ti; k < tj; ++k) {
      const wg_task& t = S.h_tasks[k];
      if (t.flags & WG_TASK_SPLIT) {
        int b = plan ? (*plan)[k] : 0;
        int32_t row = (int32_t)(t.d_lo - vb);
        ItemList* L = b ? out1 : out0;
        if (row != split_row) {
          L->hs.push_back(SplitRow{row, slot, 0, b});
          split_row = row;
        }
        L->hs.back().n_slots++;
        L->n_edges += t.e_end - t.e_begin;
        WorkItem w{};
        w.row_lo = row; w.row_hi = row + 1; w.e_lo = t.e_begin; w.e_hi = t.e_end;
        w.split_slot = slot++;
        w.task = (int32_t)k;
        // SPLIT chunks first (heaviest: overfill / frequent-value)
        lists[b].push_back({INT64_MAX / 2 + (t.e_end - t.e_begin), w});
        continue;
      }
      if (first) {
        cur_task = (int64_t)k;
        first = false;
      } else {
        flush((int32_t)(t.d_lo - vb));
        cur_lo = (int32_t)(t.d_lo - vb);
        cur_task = (int64_t)k;
      }
    }
    flush(hi);
    ti = tj;
  }
  ItemList* outs[2] = {out0, out1};
  // Underfill gTasks: a run of adjacent small work
  // items (each < UNDER edges) is merged into one item of <= CAP edges --
  // one CTA walks the run edge-wise across the gTask boundaries instead of
  // one mostly idle CTA per gTask; merged items are the smallest, so they
  // run last ("lower priority").  WG_UNDERFILL=0 disables.
  static int merge = -1;
  if (merge < 0) {
    const char* e = getenv("WG_UNDERFILL");
    merge = (e && e[0] == '0') ? 0 : 1;
  }
  constexpr int64_t UNDER = 256, CAP = 2048;
  for (int b = 0; b < 2; ++b) {
    auto& L = lists[b];
    if (merge) {
      std::vector<std::pair<int64_t, WorkItem>> m;
      for (auto& e : L) {
        const WorkItem& w = e.second;
        const int64_t ne = w.e_hi - w.e_lo;
        if (!m.empty() && w.split_slot < 0 && m.back().second.split_slot < 0 && ne < UNDER &&
            m.back().first < CAP && m.back().second.row_hi == w.row_lo && m.back().first + ne <= CAP &&
            (m.back().first < UNDER || m.back().second.task == -2)) {
          WorkItem& p = m.back().second;
          p.row_hi = w.row_hi;
          p.e_hi = w.e_hi;
          p.task = -2;                       // a merged run of gTasks
          m.back().first += ne;
          ++outs[b]->n_merged;
        } else {
          m.push_back(e);
        }
      }
      L.swap(m);
    }
    std::stable_sort(L.begin(), L.end(), [](const auto& x, const auto& y) { return x.first > y.first; });
    outs[b]->h.clear();
    outs[b]->n_split_items = 0;
    for (auto& e : L) {
      outs[b]->h.push_back(e.second);
      if (e.second.split_slot >= 0) ++outs[b]->n_split_items;
    }
  }
  *n_slots = slot;
}

}  // namespace

// Per gTask (HBM bytes, both plans' common terms dropped):
//   EDGE   t_e = n_e (A + 4) + n_rows 2A      (gather f_in rows, Agg round trip)
//   VERTEX t_v = n_e (B + 4)                  (gather f_out rows)
// plus per-layer terms: any VERTEX gTask needs Y = x W for every row,
// V (A + B); a mixed layer also writes / reads / zeroes Z, 3 B per row.
// sum = {all-EDGE, all-VERTEX, per-gTask minimum (mixed)}; the layer takes
// the cheapest (ties -> EDGE), i.e. the least-workload DFG.
// On a 1-D partition the ranks add their sums (wg_plan_create_dist) and take
// one uniform plan.
void lin_cost_sums(const wg_graph_s* g, const wg_conv_desc& d, int64_t sum[3], std::vector<uint8_t>* best) {
  const auto& tasks = g->fwd.h_tasks;
  const int64_t n = (int64_t)tasks.size();
  const int s = dsize(d.dtype);
  const int64_t A = rup((int64_t)d.f_in * s, 32), B = rup((int64_t)d.f_out * s, 32);
  const int64_t rows = g->ve - g->vb;
  sum[0] = 0; sum[1] = rows * (A + B); sum[2] = rows * (A + B) + rows * 3 * B;
  if (best) best->assign(n, 0);
  for (int64_t i = 0; i < n; ++i) {
    const wg_task& t = tasks[i];
    const int64_t ne = t.e_end - t.e_begin;
    const int64_t nrows = (int64_t)t.d_hi - t.d_lo + 1;
    const int64_t te = ne * (A + 4) + nrows * 2 * A, tv = ne * (B + 4);
    sum[0] += te;
    sum[1] += tv;
    sum[2] += std::min(te, tv);
    if (best) (*best)[i] = tv < te ? 1 : 0;
  }
}

// Exchange-table layouts.  Widths: forward Y (f_out) for
// GCN / SAGE / GIN VERTEX layers; backward dT (f_out) on the G path, dAgg
// (f_in) on the dAgg path, RGCN dT (f_out).  On a graph that owns a row block
// the GCN / SAGE tables are column-chunked into C <= 4 chunks of >= 256-byte
// rows (each chunk a whole number of 128-byte TMA store boxes), so the gather
// of chunk k overlaps the exchange of chunk k+1; GIN / RGCN tables stay
// row-major (C = 1).  WG_XCHG_CHUNK_BYTES overrides the 256-byte minimum
// (0 disables chunking).
int xchg_chunks(const wg_conv_desc& d, int64_t width) {
  if (!width || !(d.model == WG_GCN || d.model == WG_SAGE)) return 1;
  static int64_t min_chunk = -1;
  if (min_chunk < 0) {
    const char* e = getenv("WG_XCHG_CHUNK_BYTES");
    min_chunk = e ? atoll(e) : 256;
  }
  if (min_chunk <= 0) return 1;
  const int es = dsize(d.dtype);
  const int64_t pe = pitch(width, d.dtype), rho = pe * es;
  int C = (int)std::min<int64_t>(4, rho / min_chunk);
  while (C > 1 && (pe % C != 0 || (pe / C * es) % 128 != 0)) --C;
  return std::max(C, 1);
}

void xchg_layouts(wg_plan_s* p) {
  const wg_graph_s* g = p->g;
  const wg_conv_desc& d = p->d;
  p->xf = XLayout{};
  p->xb = XLayout{};
  const bool lin = d.model == WG_GCN || d.model == WG_SAGE || d.model == WG_GIN;
  const bool part = g->ve - g->vb != g->V;
  if (!part) return;                         // one partition: nothing is exchanged
  if (lin) {
    // forward: VERTEX layers exchange Y (a rank with no gTask follows the
    // layer's VERTEX policy); EDGE layers gather the caller's activation
    if (p->n_vert_tasks > 0 || (p->n_edge_tasks == 0 && d.policy == WG_PLAN_ALL_VERTEX)) p->xf.width = d.f_out;
    // backward: dT (G path) or dAgg (dAgg path, only when dx is needed)
    if (p->bwd_path == 1) p->xb.width = d.f_out;
    else if (d.need_dx) p->xb.width = d.f_in;
  } else if (d.model == WG_RGCN) {
    p->xb.width = d.f_out;
  }
  for (XLayout* X : {&p->xf, &p->xb}) {
    const int C = xchg_chunks(d, X->width);
    if (C > 1) { X->C = C; X->Fc = pitch(X->width, d.dtype) / C; }
  }
}

namespace {

// per-task plan bits for the untyped models (GCN / SAGE / GIN)
void choose_plans(wg_plan_s* p) {
  const wg_graph_s* g = p->g;
  const auto& tasks = g->fwd.h_tasks;
  const int64_t n = (int64_t)tasks.size();
  p->plan_bits.assign(n, 0);
  const wg_conv_desc& d = p->d;
  if (d.model == WG_SAGE_LSTM) {  // the LSTM aggregator is not linear: no T2 swap, EDGE only
    std::fill(p->plan_bits.begin(), p->plan_bits.end(), 0);
  } else if (d.model == WG_GAT) {  // GAT: transform-before-gather only
    std::fill(p->plan_bits.begin(), p->plan_bits.end(), 1);
  } else if (d.policy == WG_PLAN_ALL_VERTEX) {
    std::fill(p->plan_bits.begin(), p->plan_bits.end(), 1);
  } else if (d.policy == WG_PLAN_RANDOM) {
    std::mt19937_64 rng(d.policy_seed);
    for (int64_t i = 0; i < n; ++i) p->plan_bits[i] = (uint8_t)(rng() & 1);
  } else if (d.policy == WG_PLAN_AUTO) {
    int64_t sum[3];
    std::vector<uint8_t> best;
    lin_cost_sums(g, d, sum, &best);
    if (sum[0] <= sum[1] && sum[0] <= sum[2]) std::fill(p->plan_bits.begin(), p->plan_bits.end(), 0);
    else if (sum[1] <= sum[2]) std::fill(p->plan_bits.begin(), p->plan_bits.end(), 1);
    else p->plan_bits = best;
  }
  // all SPLIT chunks of one row take the plan of the row's first chunk
  for (int64_t i = 1; i < n; ++i)
    if ((tasks[i].flags & WG_TASK_SPLIT) && (tasks[i - 1].flags & WG_TASK_SPLIT) && tasks[i].d_lo == tasks[i - 1].d_lo &&
        tasks[i].type == tasks[i - 1].type)
      p->plan_bits[i] = p->plan_bits[i - 1];
  p->n_vert_tasks = std::count(p->plan_bits.begin(), p->plan_bits.end(), 1);
  p->n_edge_tasks = n - p->n_vert_tasks;
}

template <typename T>
wg_status upload(wg_plan_s* p, const std::vector<T>& h, T** d) {
  *d = nullptr;
  if (h.empty()) return WG_OK;
  void* q = nullptr;
  WG_CK(cudaMalloc(&q, sizeof(T) * h.size()));
  p->allocs.push_back(q);
  WG_CK(cudaMemcpy(q, h.data(), sizeof(T) * h.size(), cudaMemcpyHostToDevice));
  *d = static_cast<T*>(q);
  return WG_OK;
}

wg_status upload_list(wg_plan_s* p, ItemList& L) {
  L.n = (int)L.h.size();
  L.n_split = (int)L.hs.size();
  WG_TRY(upload(p, L.h, &L.d));
  WG_TRY(upload(p, L.hs, &L.split));
  return WG_OK;
}

}  // namespace

wg_status plan_create(wg_graph g, const wg_conv_desc* d, wg_plan* out) {
  WG_REQ(g && d && out, WG_ERR_INVALID, "wg_plan_create: null argument");
  WG_REQ(d->f_in >= 1 && d->f_out >= 1, WG_ERR_INVALID, "f_in / f_out must be >= 1");
  WG_REQ(d->dtype == WG_F32 || d->dtype == WG_BF16, WG_ERR_INVALID, "dtype");
  WG_REQ(d->model >= WG_GCN && d->model <= WG_SAGE_LSTM, WG_ERR_INVALID, "model");
  if (d->model != WG_RGCN)
    WG_REQ(!g->by_type, WG_ERR_UNSUPPORTED, "typed graph (num_types > 1) is only supported by RGCN");
  if (d->model == WG_GAT) WG_REQ(d->heads >= 1, WG_ERR_INVALID, "GAT needs heads >= 1");
  if (d->model == WG_GAT)
    WG_REQ(g->vb == 0 && g->ve == g->V, WG_ERR_UNSUPPORTED,
           "GAT layers need the full graph (the 1-D partition covers GCN / SAGE / GIN / RGCN)");
  WG_CK(cudaSetDevice(g->device));
  auto* p = new wg_plan_s();
  p->g = g;
  p->d = *d;
  if (p->d.heads < 1) p->d.heads = 1;
  if (d->model == WG_RGCN) {
    wg_status s = rgcn_plan(p, 0);
    if (s != WG_OK) { delete p; return s; }
  } else {
    choose_plans(p);
    // all-VERTEX layers run no EDGE pass; a layer with no gTask at all (E = 0) runs the EDGE one
    const int b_empty = (d->model != WG_GAT && p->n_edge_tasks == 0 && p->n_vert_tasks > 0) ? 1 : 0;
    build_items(g, g->fwd, &p->plan_bits, &p->fe, &p->fv, &p->n_slots_f, b_empty);
    ItemList dummy;
    build_items(g, g->bwd, nullptr, &p->bt, &dummy, &p->n_slots_t);
    wg_status s;
    if ((s = upload_list(p, p->fe)) != WG_OK || (s = upload_list(p, p->fv)) != WG_OK ||
        (s = upload_list(p, p->bt)) != WG_OK) {
      for (void* q : p->allocs) cudaFree(q);
      delete p;
      return s;
    }
    p->mixed = (p->n_edge_tasks > 0 && p->n_vert_tasks > 0) ? 1 : 0;
    // backward path: dAgg (needs Agg of every row, i.e. no VERTEX task) else G
    // (a VERTEX-policy plan without any gTask -- a rank owning no in-edge --
    // takes the G path too, so every rank exchanges the same table)
    p->bwd_path = (p->n_vert_tasks > 0 || (p->n_edge_tasks == 0 && d->policy == WG_PLAN_ALL_VERTEX)) ? 1 : 0;
    if (d->model == WG_SAGE_LSTM) {
      wg_status s2 = lstm_plan(p, 0);
      if (s2 != WG_OK) { lstm_plan_free(p); for (void* q : p->allocs) cudaFree(q); delete p; return s2; }
    } else if (d->model == WG_GAT) {
      gat_layout(p);
    } else {
      lin_layout(p);
    }
  }
  xchg_layouts(p);
  g->live_plans++;
  *out = p;
  return WG_OK;
}

}  // namespace wg

extern "C" {

wg_status wg_plan_create(wg_graph g, const wg_conv_desc* desc, wg_plan* out) {
  return wg::plan_create(g, desc, out);
}

wg_status wg_plan_sizes(wg_plan p, size_t* saved_bytes, size_t* workspace_bytes) {
  WG_REQ(p, WG_ERR_INVALID, "wg_plan_sizes: null plan");
  if (saved_bytes) *saved_bytes = p->saved.total;
  if (workspace_bytes) *workspace_bytes = p->ws.total;
  return WG_OK;
}

wg_status wg_plan_export(wg_plan p, uint8_t* per_task_plan, int64_t stats[8]) {
  WG_REQ(p, WG_ERR_INVALID, "wg_plan_export: null plan");
  if (per_task_plan) std::copy(p->plan_bits.begin(), p->plan_bits.end(), per_task_plan);
  if (stats) {
    stats[0] = p->n_edge_tasks;
    stats[1] = p->n_vert_tasks;
    stats[2] = p->bwd_path;
    stats[3] = p->xf.width;
    stats[4] = p->xb.width;
    stats[5] = p->fe.n + p->fv.n;
    stats[6] = p->bt.n;
    stats[7] = p->fe.n_split + p->fv.n_split;
  }
  return WG_OK;
}

wg_status wg_plan_buffer(wg_plan p, int which, const char* name, size_t* offset) {
  WG_REQ(p && name && offset, WG_ERR_INVALID, "wg_plan_buffer: null argument");
  const wg::Layout& L = which ? p->ws : p->saved;
  auto it = L.off.find(name);
  WG_REQ(it != L.off.end(), WG_ERR_INVALID, std::string("no buffer named ") + name);
  *offset = it->second;
  return WG_OK;
}

wg_status wg_plan_destroy(wg_plan p) {
  if (!p) return WG_OK;
  cudaSetDevice(p->g->device);
  cudaDeviceSynchronize();
  if (p->rg) wg::rgcn_plan_free(p);
  if (p->gat) wg::gat_plan_free(p);
  if (p->lstm) wg::lstm_plan_free(p);
  for (void* q : p->allocs) cudaFree(q);
  p->g->live_plans--;
  delete p;
  return WG_OK;
}

}  // extern "C"
