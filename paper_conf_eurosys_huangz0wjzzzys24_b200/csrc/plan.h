// Plan object: per-gTask operation plan (a4) plus the execution structures
// derived from the gTask tables (work items, split rows, buffer layout).
#pragma once
#include <map>
#include <string>

#include "wg_internal.cuh"

namespace wg {

// Named, 256-byte aligned sub-buffers of one caller-owned allocation.
struct Layout {
  std::map<std::string, size_t> off;
  size_t total = 0;
  void add(const std::string& name, size_t bytes) {
    off[name] = total;
    total += rup(std::max<size_t>(bytes, 1), 256);
  }
  bool has(const std::string& n) const { return off.count(n) != 0; }
  template <typename T> T* at(const void* base, const std::string& n) const {
    auto it = off.find(n);
    return it == off.end() ? nullptr : reinterpret_cast<T*>(const_cast<char*>(static_cast<const char*>(base)) + it->second);
  }
};

struct ItemList {
  WorkItem* d = nullptr;
  int n = 0;
  SplitRow* split = nullptr;
  int n_split = 0;
  std::vector<WorkItem> h;
  std::vector<SplitRow> hs;
  int64_t n_edges = 0, n_rows = 0;   // totals (algorithmic-byte accounting)
  int n_split_items = 0;             // leading items that are SPLIT chunks (heavy-first order)
  int n_merged = 0;                  // underfill items merged into their neighbours
};

// Column-chunked layout of an exchange table:
// C chunks of Fc columns, chunk k = [rows x Fc] row-major at k * rows * Fc
// elements, rows = the graph's global vertex count.  C = 1: one row-major
// [rows x ld] table (ld chosen by the caller).  Aggregation is
// column-separable, so the gather of chunk k can start as soon as chunk k of
// every rank has arrived, overlapping the exchange of chunk k+1.
struct XLayout {
  int C = 1;
  int64_t Fc = 0;          // columns per chunk (C > 1)
  int64_t width = 0;       // exchanged columns (f_out or f_in)
};

// Dependency hook for the POST gathers of a distributed call: before the
// gather of chunk k the compute stream waits for ev[k] (chunk k received).
struct XHook {
  const cudaEvent_t* ev = nullptr;
  int n = 0;
  void wait(int k, cudaStream_t s) const {
    if (ev && n > 0) cudaStreamWaitEvent(s, ev[k < n ? k : n - 1], 0);
  }
};

}  // namespace wg

struct wg_plan_s {
  wg_graph g = nullptr;
  wg_conv_desc d{};
  std::vector<uint8_t> plan_bits;    // per forward gTask: 0 EDGE, 1 VERTEX
  int64_t n_edge_tasks = 0, n_vert_tasks = 0;
  wg::ItemList fe, fv, bt;           // forward EDGE items, forward VERTEX items, transposed items
  int n_slots_f = 0, n_slots_t = 0;  // SPLIT partial slots
  int bwd_path = 0;                  // 0: dAgg path (Agg saved), 1: G path
  int mixed = 0;
  int64_t pi = 0, po = 0;            // row pitches (elements) of f_in / f_out wide tensors
  wg::Layout saved, ws;
  std::vector<void*> allocs;
  wg::XLayout xf, xb;                // exchange tables: forward (Y), backward (dT / dAgg)
  // model-specific structures (conv_rgcn.cu / conv_gat.cu)
  void* rg = nullptr;
  void* gat = nullptr;
  void* lstm = nullptr;
};

// The EDGE pass (aggregate, then the transform GEMM) runs when any gTask is
// EDGE, or when the layer has no gTask at all (E = 0: every row is the
// empty-neighbourhood epilogue, produced by that pass's items).
inline bool edge_path(const wg_plan_s* p) { return p->n_edge_tasks > 0 || p->n_vert_tasks == 0; }

namespace wg {
wg_status rgcn_plan(wg_plan_s* p, cudaStream_t s);
void rgcn_plan_free(wg_plan_s* p);
wg_status rgcn_forward(wg_plan_s* p, const wg_params* P, const wg_fwd_args* a, cudaStream_t s);
wg_status rgcn_backward(wg_plan_s* p, const wg_params* P, const wg_bwd_args* a, const wg_grads* G, cudaStream_t s,
                        const XHook* hk = nullptr);
wg_status gat_forward(wg_plan_s* p, const wg_params* P, const wg_fwd_args* a, cudaStream_t s);
wg_status gat_backward(wg_plan_s* p, const wg_params* P, const wg_bwd_args* a, const wg_grads* G, cudaStream_t s);
wg_status lin_forward(wg_plan_s* p, const wg_params* P, const wg_fwd_args* a, cudaStream_t s,
                      const XHook* hk = nullptr);
wg_status lin_backward(wg_plan_s* p, const wg_params* P, const wg_bwd_args* a, const wg_grads* G, cudaStream_t s,
                       const XHook* hk = nullptr);
// exchange layouts of a plan (set by plan_create for graphs owning a row block)
void xchg_layouts(wg_plan_s* p);
// column chunks of a GCN / SAGE exchange table of `width` columns (1: row-major)
int xchg_chunks(const wg_conv_desc& d, int64_t width);
// a4 layer cost sums {all-EDGE, all-VERTEX, mixed} of the untyped models
void lin_cost_sums(const wg_graph_s* g, const wg_conv_desc& d, int64_t sum[3], std::vector<uint8_t>* best);
wg_status plan_create(wg_graph g, const wg_conv_desc* d, wg_plan* out);
wg_status graph_create(const wg_graph_desc* d, int device, cudaStream_t st, wg_graph* out);
void gat_layout(wg_plan_s* p);
wg_status lstm_plan(wg_plan_s* p, cudaStream_t s);
void lstm_plan_free(wg_plan_s* p);
wg_status lstm_forward(wg_plan_s* p, const wg_params* P, const wg_fwd_args* a, cudaStream_t s);
wg_status lstm_backward(wg_plan_s* p, const wg_params* P, const wg_bwd_args* a, const wg_grads* G, cudaStream_t s);
void gat_plan_free(wg_plan_s* p);
void lin_layout(wg_plan_s* p);
}  // namespace wg
