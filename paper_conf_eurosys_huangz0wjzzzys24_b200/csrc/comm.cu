// Multi-GPU gTask layer (SURVEY §8(e), §8(b) "multi-GPU" entry points).
//
// The paper's data-parallel scheme (Fig 11): every GPU owns a
// block of destination vertices and the gTasks of those rows; before a layer
// the embeddings its gathers read are exchanged.  Here:
//   * 1-D partition: T-aligned vertex blocks balanced on in- plus out-edges
//     (the forward gathers a rank's in-edges, the backward its out-edges);
//   * one exchange per layer and direction, over NCCL on a dedicated
//     high-priority communication stream: the activation itself for EDGE
//     layers, Y = h W for VERTEX layers (transform before communicate,
//     P:L2279-2289, Fig 11c), dT / dAgg in the backward.  Blocks of unequal
//     size are exchanged as an all-gather-v (grouped ncclBroadcast, one root
//     per rank), equal blocks by ncclAllGather;
//   * overlap: GCN / SAGE exchange tables are column-chunked (plan.h XLayout,
//     aggregation is column-separable), chunk k is exchanged while the POST
//     gather of chunk k-1 runs; the weight-gradient all-reduce is left running
//     on the communication stream under the next layer's backward
//     (wg_comm_wait joins it).
// NCCL is resolved at run time from the library the process already loaded
// (torch's), so one NCCL instance serves the process; without NCCL the
// multi-GPU calls return WG_ERR_UNSUPPORTED (no fallback).
//
// Emulated communicator (wg_comm_init_emulated): one process, one GPU, one
// rank of a P-way partition (bench.py --rank-slice).  Each exchange is a copy
// kernel on the communication stream that reads and rewrites every non-owned
// row of the table with WG_EMU_CTAS CTAs (default 40: about the 0.7 TB/s an
// NVLink 5 all-gather delivers), so the overlap of exchange and gathers can be timed on one
// GPU.  It moves no data between ranks: a timing device, not a result.
#include <dlfcn.h>

#include <algorithm>
#include <cstring>

#include "plan.h"

namespace wg {
namespace {

// ----------------------------------------------------------- NCCL (dlopen)
// The stable C ABI of nccl.h: opaque comm, 128-byte unique id, int enums.
typedef struct ncclComm* ncclComm_t;
struct NcclUid { char internal[128]; };
typedef int nccl_res;
constexpr int N_INT8 = 0, N_INT64 = 4, N_FLOAT32 = 7, N_SUM = 0;

struct NcclApi {
  bool ok = false;
  std::string why;
  nccl_res (*GetUniqueId)(NcclUid*) = nullptr;
  nccl_res (*CommInitRank)(ncclComm_t*, int, NcclUid, int) = nullptr;
  nccl_res (*CommDestroy)(ncclComm_t) = nullptr;
  nccl_res (*Broadcast)(const void*, void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
  nccl_res (*AllGather)(const void*, void*, size_t, int, ncclComm_t, cudaStream_t) = nullptr;
  nccl_res (*AllReduce)(const void*, void*, size_t, int, int, ncclComm_t, cudaStream_t) = nullptr;
  nccl_res (*GroupStart)() = nullptr;
  nccl_res (*GroupEnd)() = nullptr;
  const char* (*GetErrorString)(nccl_res) = nullptr;
};

NcclApi load_nccl() {
  NcclApi a;
  void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_NOLOAD);   // the process's NCCL (torch)
  if (!h) {
    const char* e = getenv("WG_NCCL_LIB");
    h = dlopen(e && e[0] ? e : "libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
  }
  if (!h) { a.why = std::string("cannot load libnccl.so.2: ") + dlerror(); return a; }
#define WG_SYM(f)                                                          \
  a.f = reinterpret_cast<decltype(a.f)>(dlsym(h, "nccl" #f));               \
  if (!a.f) { a.why = "libnccl.so.2 lacks nccl" #f; return a; }
  WG_SYM(GetUniqueId) WG_SYM(CommInitRank) WG_SYM(CommDestroy) WG_SYM(Broadcast) WG_SYM(AllGather)
  WG_SYM(AllReduce) WG_SYM(GroupStart) WG_SYM(GroupEnd) WG_SYM(GetErrorString)
#undef WG_SYM
  a.ok = true;
  return a;
}

NcclApi& nccl() {
  static NcclApi a = load_nccl();
  return a;
}

#define WG_NCCL(call)                                                                  \
  do {                                                                                 \
    nccl_res r_ = (call);                                                              \
    if (r_ != 0) {                                                                     \
      ::wg::set_error(std::string(#call) + ": " + nccl().GetErrorString(r_));          \
      return WG_ERR_CUDA;                                                              \
    }                                                                                  \
  } while (0)

// emulated exchange: re-read and re-write the non-owned rows in place
__global__ void k_emu_xchg(int4* base, int64_t lo, int64_t hi, int64_t n) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x, own = hi - lo;
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n - own; j += stride) {
    const int64_t i = j < lo ? j : j + own;     // skip this rank's rows
    int4 v = __ldcg(base + i);
    __stcg(base + i, v);
  }
}

}  // namespace
}  // namespace wg

struct wg_comm_s {
  int rank = 0, world = 1, device = 0, emulated = 0;
  wg::ncclComm_t comm = nullptr;
  cudaStream_t cs = nullptr;                     // communication stream
  cudaEvent_t fork = nullptr, join = nullptr;
  cudaEvent_t ev[8] = {};                        // per-chunk arrival
  int emu_ctas = 40;   // ~0.7 TB/s of rewritten rows (calibrated on B200: 16 CTAs -> 0.28 TB/s)
};

namespace wg {
namespace {

wg_status comm_streams(wg_comm_s* c) {
  int lo = 0, hi = 0;
  WG_CK(cudaDeviceGetStreamPriorityRange(&lo, &hi));
  WG_CK(cudaStreamCreateWithPriority(&c->cs, cudaStreamNonBlocking, hi));
  WG_CK(cudaEventCreateWithFlags(&c->fork, cudaEventDisableTiming));
  WG_CK(cudaEventCreateWithFlags(&c->join, cudaEventDisableTiming));
  for (auto& e : c->ev) WG_CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  return WG_OK;
}

// the communication stream continues after the work queued so far on s
wg_status fork_to_comm(wg_comm_s* c, cudaStream_t s) {
  WG_CK(cudaEventRecord(c->fork, s));
  WG_CK(cudaStreamWaitEvent(c->cs, c->fork, 0));
  return WG_OK;
}

// All-gather-v of the row blocks [bounds[q], bounds[q+1]) of one table (rows
// of ld_bytes), in place, on the communication stream.
wg_status exchange_rows(wg_comm_s* c, void* base, int64_t ld_bytes, const std::vector<int64_t>& b) {
  if (c->world <= 1) return WG_OK;
  char* p = static_cast<char*>(base);
  if (c->emulated == 2) return WG_OK;          // compute-only emulation: no exchange at all
  if (c->emulated) {
    const int64_t n = b.back() * ld_bytes / 16;
    WG_LAUNCH(k_emu_xchg, c->emu_ctas, 512, 0, c->cs, reinterpret_cast<int4*>(p), b[c->rank] * ld_bytes / 16,
              b[c->rank + 1] * ld_bytes / 16, n);
    return WG_OK;
  }
  bool equal = true;
  for (int q = 0; q < c->world; ++q) equal = equal && (b[q + 1] - b[q] == b[1] - b[0]);
  if (equal) {
    const size_t cnt = (size_t)(b[1] - b[0]) * ld_bytes;
    WG_NCCL(nccl().AllGather(p + (size_t)b[c->rank] * ld_bytes, p, cnt, N_INT8, c->comm, c->cs));
    return WG_OK;
  }
  WG_NCCL(nccl().GroupStart());
  for (int q = 0; q < c->world; ++q) {
    char* blk = p + (size_t)b[q] * ld_bytes;
    const size_t cnt = (size_t)(b[q + 1] - b[q]) * ld_bytes;
    if (cnt) WG_NCCL(nccl().Broadcast(blk, blk, cnt, N_INT8, q, c->comm, c->cs));
  }
  WG_NCCL(nccl().GroupEnd());
  return WG_OK;
}

// Exchange an exchange table of layout X (C chunks) on the comm stream after
// the work queued on s; ev[k] marks chunk k received.  ld: pitch (elements)
// of a C = 1 table.
wg_status exchange_table(wg_comm_s* c, cudaStream_t s, void* tab, const XLayout& X, int64_t ld, int es,
                         const std::vector<int64_t>& b, XHook* hk) {
  WG_TRY(fork_to_comm(c, s));
  const int C = std::max(1, X.C);
  const int64_t V = b.back();
  for (int k = 0; k < C; ++k) {
    char* base = static_cast<char*>(tab) + (C > 1 ? (size_t)k * V * X.Fc * es : 0);
    WG_TRY(exchange_rows(c, base, (C > 1 ? X.Fc : ld) * es, b));
    WG_CK(cudaEventRecord(c->ev[k], c->cs));
  }
  hk->ev = c->ev;
  hk->n = C;
  return WG_OK;
}

wg_status join_comm(wg_comm_s* c, cudaStream_t s) {
  WG_CK(cudaEventRecord(c->join, c->cs));
  WG_CK(cudaStreamWaitEvent(s, c->join, 0));
  return WG_OK;
}

bool lin_model(const wg_conv_desc& d) { return d.model == WG_GCN || d.model == WG_SAGE || d.model == WG_GIN; }

// VERTEX layer of a uniform distributed plan (a rank with no gTask follows the policy)
bool vertex_layer(const wg_plan_s* p) {
  return p->n_vert_tasks > 0 || (p->n_edge_tasks == 0 && p->d.policy == WG_PLAN_ALL_VERTEX);
}

wg_status check_dist(wg_comm_s* c, wg_plan_s* p) {
  WG_REQ(c && p, WG_ERR_INVALID, "null comm / plan");
  WG_REQ((int64_t)p->g->bounds.size() == c->world + 1, WG_ERR_STATE,
         "distributed calls need a graph made by wg_graph_create_dist with this communicator");
  WG_REQ(p->d.model != WG_GAT || c->world == 1, WG_ERR_UNSUPPORTED,
         "the 1-D partition covers GCN / SAGE / GIN / RGCN");
  WG_CK(cudaSetDevice(p->g->device));
  WG_CK(cudaGetLastError());
  return WG_OK;
}

// element counts of the gradient buffers (wg_grads order)
void grad_counts(const wg_plan_s* p, int64_t n[7]) {
  const wg_conv_desc& d = p->d;
  const int64_t fi = d.f_in, fo = d.f_out, H = std::max(1, d.heads);
  for (int i = 0; i < 7; ++i) n[i] = 0;
  if (d.model == WG_RGCN) n[0] = (int64_t)p->g->R * fi * fo;
  else if (d.model == WG_GAT) n[0] = fi * H * fo;
  else n[0] = fi * fo;
  n[1] = fi * fo;
  n[2] = (d.model == WG_GAT && d.concat_heads) ? H * fo : fo;
  n[3] = n[4] = H * fo;
  n[5] = fo * fo;
  n[6] = fo;
}

}  // namespace
}  // namespace wg

extern "C" {

wg_status wg_comm_unique_id(void* id) {
  using namespace wg;
  WG_REQ(id, WG_ERR_INVALID, "wg_comm_unique_id: null");
  WG_REQ(nccl().ok, WG_ERR_UNSUPPORTED, nccl().why);
  NcclUid u;
  WG_NCCL(nccl().GetUniqueId(&u));
  memcpy(id, &u, sizeof(u));
  return WG_OK;
}

wg_status wg_comm_init(const void* id, int rank, int world, int device, wg_comm* out) {
  using namespace wg;
  WG_REQ(id && out && world >= 1 && rank >= 0 && rank < world, WG_ERR_INVALID, "wg_comm_init: bad argument");
  WG_REQ(nccl().ok, WG_ERR_UNSUPPORTED, nccl().why);
  WG_CK(cudaSetDevice(device));
  auto* c = new wg_comm_s();
  c->rank = rank; c->world = world; c->device = device;
  NcclUid u;
  memcpy(&u, id, sizeof(u));
  wg_status st = comm_streams(c);
  if (st == WG_OK) {
    nccl_res r = nccl().CommInitRank(&c->comm, world, u, rank);
    if (r != 0) { set_error(std::string("ncclCommInitRank: ") + nccl().GetErrorString(r)); st = WG_ERR_CUDA; }
  }
  if (st != WG_OK) { wg_comm_destroy(c); return st; }
  *out = c;
  return WG_OK;
}

wg_status wg_comm_init_emulated(int rank, int world, int device, int copy, wg_comm* out) {
  using namespace wg;
  WG_REQ(out && world >= 1 && rank >= 0 && rank < world, WG_ERR_INVALID, "wg_comm_init_emulated: bad argument");
  WG_CK(cudaSetDevice(device));
  auto* c = new wg_comm_s();
  c->rank = rank; c->world = world; c->device = device; c->emulated = copy ? 1 : 2;
  const char* e = getenv("WG_EMU_CTAS");
  if (e && atoi(e) > 0) c->emu_ctas = atoi(e);
  wg_status st = comm_streams(c);
  if (st != WG_OK) { wg_comm_destroy(c); return st; }
  *out = c;
  return WG_OK;
}

wg_status wg_comm_info(wg_comm c, int32_t info[4]) {
  WG_REQ(c && info, WG_ERR_INVALID, "wg_comm_info: null");
  info[0] = c->rank; info[1] = c->world; info[2] = c->device; info[3] = c->emulated;
  return WG_OK;
}

wg_status wg_comm_wait(wg_comm c, wg_stream stream) {
  WG_REQ(c, WG_ERR_INVALID, "wg_comm_wait: null");
  WG_CK(cudaSetDevice(c->device));
  return wg::join_comm(c, (cudaStream_t)stream);
}

wg_status wg_comm_destroy(wg_comm c) {
  if (!c) return WG_OK;
  cudaSetDevice(c->device);
  if (c->cs) cudaStreamSynchronize(c->cs);
  if (c->comm && wg::nccl().ok) wg::nccl().CommDestroy(c->comm);
  for (auto& e : c->ev) if (e) cudaEventDestroy(e);
  if (c->fork) cudaEventDestroy(c->fork);
  if (c->join) cudaEventDestroy(c->join);
  if (c->cs) cudaStreamDestroy(c->cs);
  delete c;
  return WG_OK;
}

// --------------------------------------------------------- 1-D partition
wg_status wg_partition_1d(const wg_graph_desc* d, int world, int64_t* bounds) {
  using namespace wg;
  WG_REQ(d && bounds && world >= 1, WG_ERR_INVALID, "wg_partition_1d: bad argument");
  const int64_t V = d->num_vertices, E = d->num_edges;
  const int64_t T = d->tile_rows > 0 ? d->tile_rows : 128;
  WG_REQ(V >= 1 && E >= 0 && (E == 0 || d->src), WG_ERR_INVALID, "wg_partition_1d: bad sizes");
  WG_REQ(d->indptr || d->dst || E == 0, WG_ERR_INVALID, "wg_partition_1d: need indptr or dst");
  const int64_t nt = cdiv(V, T);
  WG_REQ(nt >= world, WG_ERR_INVALID, "wg_partition_1d: fewer T-row tiles than ranks");
  // host copies (pointers may be host or device)
  auto fetch = [](const void* ptr, size_t bytes, std::vector<char>& buf) -> const void* {
    cudaPointerAttributes a;
    bool dev = false;
    if (cudaPointerGetAttributes(&a, ptr) == cudaSuccess)
      dev = a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
    else
      cudaGetLastError();
    if (!dev) return ptr;
    buf.resize(bytes);
    if (cudaMemcpy(buf.data(), ptr, bytes, cudaMemcpyDeviceToHost) != cudaSuccess) return nullptr;
    return buf.data();
  };
  std::vector<int64_t> w(nt, 0);   // per tile: in-edges + out-edges + rows
  for (int64_t v = 0; v < V; ++v) w[v / T] += 1;
  std::vector<char> b1, b2;
  if (E > 0) {
    const int32_t* src = static_cast<const int32_t*>(fetch(d->src, sizeof(int32_t) * E, b1));
    WG_REQ(src, WG_ERR_CUDA, "wg_partition_1d: copy of src failed");
    for (int64_t e = 0; e < E; ++e) {
      WG_REQ(src[e] >= 0 && src[e] < V, WG_ERR_RANGE, "wg_partition_1d: src out of range");
      w[src[e] / T] += 1;
    }
    if (d->indptr) {
      const int64_t* ip = static_cast<const int64_t*>(fetch(d->indptr, sizeof(int64_t) * (V + 1), b2));
      WG_REQ(ip, WG_ERR_CUDA, "wg_partition_1d: copy of indptr failed");
      for (int64_t v = 0; v < V; ++v) w[v / T] += ip[v + 1] - ip[v];
    } else {
      const int32_t* dst = static_cast<const int32_t*>(fetch(d->dst, sizeof(int32_t) * E, b2));
      WG_REQ(dst, WG_ERR_CUDA, "wg_partition_1d: copy of dst failed");
      for (int64_t e = 0; e < E; ++e) {
        WG_REQ(dst[e] >= 0 && dst[e] < V, WG_ERR_RANGE, "wg_partition_1d: dst out of range");
        w[dst[e] / T] += 1;
      }
    }
  }
  std::vector<int64_t> S(nt + 1, 0);   // S[t] = load of tiles [0, t)
  for (int64_t t = 0; t < nt; ++t) S[t + 1] = S[t] + w[t];
  const int64_t total = S[nt];
  bounds[0] = 0;
  int64_t prev = 0;
  for (int q = 1; q < world; ++q) {
    // the tile boundary whose prefix load is nearest to q/world of the total,
    // leaving at least one tile to every rank
    const long double target = (long double)total * q / world;
    int64_t t = std::lower_bound(S.begin(), S.end(), (int64_t)target) - S.begin();
    if (t > 0 && (long double)S[t] - target > target - (long double)S[t - 1]) --t;
    t = std::max(t, prev + 1);
    t = std::min(t, nt - (world - q));
    bounds[q] = t * T;
    prev = t;
  }
  bounds[world] = V;
  return WG_OK;
}

wg_status wg_graph_create_dist(wg_comm c, const wg_graph_desc* global, const int64_t* bounds_in, int device,
                               wg_stream stream, wg_graph* out, int64_t* v_begin, int64_t* v_end) {
  using namespace wg;
  WG_REQ(c && global && out, WG_ERR_INVALID, "wg_graph_create_dist: null argument");
  WG_REQ(device == c->device, WG_ERR_INVALID, "wg_graph_create_dist: device differs from the communicator's");
  std::vector<int64_t> b(c->world + 1);
  const int64_t T = global->tile_rows > 0 ? global->tile_rows : 128;
  if (bounds_in) {
    std::copy(bounds_in, bounds_in + c->world + 1, b.begin());
    WG_REQ(b[0] == 0 && b[c->world] == global->num_vertices, WG_ERR_INVALID, "bounds must cover [0, V)");
    for (int q = 0; q < c->world; ++q)
      WG_REQ(b[q] < b[q + 1] && b[q] % T == 0, WG_ERR_INVALID, "bounds must be increasing multiples of T");
  } else {
    WG_TRY(wg_partition_1d(global, c->world, b.data()));
  }
  wg_graph_desc d = *global;
  if (c->world > 1) { d.v_begin = b[c->rank]; d.v_end = b[c->rank + 1]; }
  else { d.v_begin = 0; d.v_end = 0; }
  WG_TRY(graph_create(&d, device, (cudaStream_t)stream, out));
  (*out)->bounds = b;
  if (v_begin) *v_begin = b[c->rank];
  if (v_end) *v_end = b[c->rank + 1];
  return WG_OK;
}

wg_status wg_graph_bounds(wg_graph g, int64_t* bounds, int32_t* n_ranks) {
  WG_REQ(g, WG_ERR_INVALID, "wg_graph_bounds: null");
  if (n_ranks) *n_ranks = g->bounds.empty() ? 0 : (int32_t)g->bounds.size() - 1;
  if (bounds) std::copy(g->bounds.begin(), g->bounds.end(), bounds);
  return WG_OK;
}

wg_status wg_plan_create_dist(wg_comm c, wg_graph g, const wg_conv_desc* desc, wg_plan* out) {
  using namespace wg;
  WG_REQ(c && g && desc && out, WG_ERR_INVALID, "wg_plan_create_dist: null argument");
  WG_REQ((int64_t)g->bounds.size() == c->world + 1, WG_ERR_STATE, "graph not made by wg_graph_create_dist");
  wg_conv_desc d = *desc;
  if (lin_model(d) && c->world > 1) {
    // one uniform plan per layer on every rank: the ranks exchange one table
    WG_REQ(d.policy != WG_PLAN_RANDOM, WG_ERR_UNSUPPORTED, "mixed (random) plans are single-partition only");
    if (d.policy == WG_PLAN_AUTO) {
      // Operation placement by data volume (Fig 11): the a4
      // HBM cost of each uniform plan plus the exchange it implies on this
      // rank, pipelined over the table's column chunks.  EDGE exchanges the
      // activation (unless replicated) and, for dx, dAgg (f_in wide);
      // VERTEX exchanges Y = x W and dT (f_out wide).  Per-rank times are
      // summed over the ranks (an all-reduce) and the smaller plan is taken.
      int64_t sum[3];
      lin_cost_sums(g, d, sum, nullptr);
      const int es = dsize(d.dtype);
      const int64_t remote = g->V - (g->ve - g->vb);
      const int64_t rin = pitch(d.f_in, d.dtype) * es, rout = pitch(d.f_out, d.dtype) * es;
      auto pipe = [](int64_t gather, int64_t link, int C) {   // C-chunk pipeline (milli-fs)
        return link / C + (C - 1) * std::max(gather, link) / C + gather / C;
      };
      // forward gather ~ half of the layer's a4 bytes, backward the other half
      const int64_t ge = sum[0] * K_MEM / 2, gv = sum[1] * K_MEM / 2;
      const int64_t le_f = d.x_replicated ? 0 : remote * rin * K_LINK, le_b = d.need_dx ? remote * rin * K_LINK : 0;
      const int64_t lv = remote * rout * K_LINK;
      const int ci = xchg_chunks(d, d.f_in), co = xchg_chunks(d, d.f_out);
      int64_t t[2] = {pipe(ge, le_f, 1) + pipe(ge, le_b, ci), pipe(gv, lv, co) + pipe(gv, lv, co)};
      if (!c->emulated) {   // add the ranks' layer costs (all-EDGE, all-VERTEX)
        WG_CK(cudaSetDevice(g->device));
        int64_t* dsum = nullptr;
        WG_CK(cudaMalloc(&dsum, 2 * sizeof(int64_t)));
        cudaMemcpy(dsum, t, 2 * sizeof(int64_t), cudaMemcpyHostToDevice);
        nccl_res r = nccl().AllReduce(dsum, dsum, 2, N_INT64, N_SUM, c->comm, c->cs);
        cudaStreamSynchronize(c->cs);
        cudaMemcpy(t, dsum, 2 * sizeof(int64_t), cudaMemcpyDeviceToHost);
        cudaFree(dsum);
        if (r != 0) { set_error(std::string("ncclAllReduce: ") + nccl().GetErrorString(r)); return WG_ERR_CUDA; }
      }
      d.policy = t[1] < t[0] ? WG_PLAN_ALL_VERTEX : WG_PLAN_ALL_EDGE;
    }
  }
  return plan_create(g, &d, out);
}

wg_status wg_plan_xchg(wg_plan p, int dir, int64_t info[4]) {
  using namespace wg;
  WG_REQ(p && info && (dir == 0 || dir == 1), WG_ERR_INVALID, "wg_plan_xchg: bad argument");
  const XLayout& X = dir == 0 ? p->xf : p->xb;
  const int es = dsize(p->d.dtype);
  const int64_t cols = X.C > 1 ? X.Fc : pitch(std::max<int64_t>(X.width, 1), p->d.dtype);
  info[0] = p->g->V;                          // rows
  info[1] = cols;                             // row pitch of one chunk (elements)
  info[2] = std::max(1, X.C);                 // chunks
  info[3] = X.width ? (int64_t)info[0] * cols * info[2] * es : 0;   // bytes (0: no table)
  return WG_OK;
}

wg_status wg_conv_forward_dist(wg_comm c, wg_plan p, const wg_params* P, const wg_fwd_args* a, int x_gathered,
                               wg_stream stream) {
  using namespace wg;
  WG_TRY(check_dist(c, p));
  WG_REQ(P && a && a->phase == WG_PHASE_ALL, WG_ERR_INVALID, "wg_conv_forward_dist: phase must be WG_PHASE_ALL");
  cudaStream_t s = (cudaStream_t)stream;
  const wg_conv_desc& d = p->d;
  const int es = dsize(d.dtype);
  const auto& b = p->g->bounds;
  const bool lin = lin_model(d);
  const bool vx = lin && vertex_layer(p);
  // layers that gather raw rows of x read rows other ranks own: all-gather x in place
  if (c->world > 1 && !x_gathered && (d.model == WG_RGCN || (lin && !vx))) {
    XHook hk;
    WG_TRY(exchange_table(c, s, const_cast<void*>(a->x), XLayout{}, a->ldx, es, b, &hk));
    hk.wait(0, s);
  }
  if (!vx || c->world == 1) {
    switch (d.model) {
      case WG_GCN: case WG_SAGE: case WG_GIN: return lin_forward(p, P, a, s);
      case WG_RGCN: return rgcn_forward(p, P, a, s);
      default: return gat_forward(p, P, a, s);
    }
  }
  WG_REQ(a->xchg, WG_ERR_INVALID, "wg_conv_forward_dist: a VERTEX layer needs the exchange table (wg_plan_xchg)");
  wg_fwd_args A = *a;
  A.phase = WG_PHASE_PRE;
  WG_TRY(lin_forward(p, P, &A, s));
  XHook hk;
  WG_TRY(exchange_table(c, s, A.xchg, p->xf, A.ld_xchg, es, b, &hk));
  A.phase = WG_PHASE_POST;
  WG_TRY(lin_forward(p, P, &A, s, &hk));
  return join_comm(c, s);
}

wg_status wg_conv_backward_dist(wg_comm c, wg_plan p, const wg_params* P, const wg_bwd_args* a, const wg_grads* G,
                                wg_stream stream) {
  using namespace wg;
  WG_TRY(check_dist(c, p));
  WG_REQ(P && a && a->phase == WG_PHASE_ALL, WG_ERR_INVALID, "wg_conv_backward_dist: phase must be WG_PHASE_ALL");
  cudaStream_t s = (cudaStream_t)stream;
  const wg_conv_desc& d = p->d;
  const int es = dsize(d.dtype);
  const bool lin = lin_model(d);
  const bool xchg = c->world > 1 && (d.model == WG_RGCN || (lin && (p->bwd_path == 1 || d.need_dx)));
  if (!xchg) {
    switch (d.model) {
      case WG_GCN: case WG_SAGE: case WG_GIN: WG_TRY(lin_backward(p, P, a, G, s)); break;
      case WG_RGCN: WG_TRY(rgcn_backward(p, P, a, G, s)); break;
      default: WG_TRY(gat_backward(p, P, a, G, s)); break;
    }
  } else {
    WG_REQ(a->xchg, WG_ERR_INVALID, "wg_conv_backward_dist: the exchange table is required (wg_plan_xchg)");
    wg_bwd_args A = *a;
    A.phase = WG_PHASE_PRE;
    WG_TRY(lin ? lin_backward(p, P, &A, G, s) : rgcn_backward(p, P, &A, G, s));
    XHook hk;
    WG_TRY(exchange_table(c, s, A.xchg, p->xb, A.ld_xchg, es, p->g->bounds, &hk));
    A.phase = WG_PHASE_POST;
    WG_TRY(lin ? lin_backward(p, P, &A, G, s, &hk) : rgcn_backward(p, P, &A, G, s, &hk));
    WG_TRY(join_comm(c, s));
  }
  // weight gradients: all-reduce (sum) on the communication stream, left
  // running under the caller's next work; wg_comm_wait joins it
  if (G && c->world > 1 && !c->emulated) {
    int64_t n[7];
    grad_counts(p, n);
    float* g[7] = {G->W, G->W_self, G->bias, G->attn_l, G->attn_r, G->W2, G->b2};
    WG_TRY(fork_to_comm(c, s));
    WG_NCCL(nccl().GroupStart());
    for (int i = 0; i < 7; ++i)
      if (g[i] && n[i]) WG_NCCL(nccl().AllReduce(g[i], g[i], (size_t)n[i], N_FLOAT32, N_SUM, c->comm, c->cs));
    WG_NCCL(nccl().GroupEnd());
  }
  return WG_OK;
}

}  // extern "C"
