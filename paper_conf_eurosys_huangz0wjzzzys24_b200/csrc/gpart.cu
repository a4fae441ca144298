// General restriction engine and an executor for the
// non-destination-exclusive gTasks it produces.
//
// The graph partition table of §4.2: per edge attribute a
// restriction uniq(a) = k (at most k distinct values of a in a gTask) or
// uniq(a) = min (gTasks with fewer distinct values preferred), over dst-id,
// src-id, edge type, dst-degree (an inherent attribute) and
// edge-id; Fig 7 and Fig 9's source-based RGCN gTasks
// are instances.  The greedy of P:L1431-1451: sort by the
// restricted attributes, scan in order, add the edge if every restriction
// still holds, else start a new gTask.  Sort-key reading Q25:
// uniq = 1 attributes, then min attributes, then uniq = k > 1 attributes
// (edge-id excluded), then dst-id if absent, then edge-id.
//
// GPU steps: LSD multi-pass stable radix sort of the edge ids (one CUB pass
// per key attribute, least significant first); groups = runs of equal
// uniq = 1 attributes; one warp per group scans it in order (the greedy is
// sequential by definition), tracking each k > 1 attribute's distinct values
// in shared memory (a warp-wide ballot search; a run of equal values hits a
// last-value fast path) and flagging gTask starts; compaction and per-gTask
// statistics (d_lo / d_hi / n_uniq_src by a (task, src) key sort).
//
// Executor: gTasks here may share destinations, so the aggregation
// Agg[v] = sum_{e in in(v)} c_e x[src_e] (the Index / Index-add pair of
// P:L520-536) accumulates fp32 partial rows with vector atomics
// (red.global.add.v4.f32) -- one atomic per run of equal destinations in a
// warp's edge chunk -- and a finishing pass applies the destination scale
// and the RNE cast.  The atomic order varies run to run (results are equal up
// to fp32 rounding); the destination-exclusive tile engine (graph.cu /
// agg.cu) stays the deterministic production path.
#include <cub/cub.cuh>

#include <algorithm>

#include "wg_internal.cuh"

struct wg_gpart_s {
  int device = 0;
  int64_t V = 0, E = 0;
  int32_t* perm = nullptr;     // [E] edge ids in sorted order
  int32_t* src_s = nullptr;    // [E] src in sorted order
  int32_t* dst_s = nullptr;    // [E] dst in sorted order
  float* rs_out = nullptr;     // [V] deg_out^-1/2
  float* rs_in = nullptr;      // [V] deg_in^-1/2
  float* inv_in = nullptr;     // [V] 1/deg_in
  wg_task* tasks = nullptr;
  int64_t n_tasks = 0;
  std::vector<wg_task> h_tasks;
  std::vector<void*> allocs;
};

namespace wg {
namespace {

constexpr int MAX_SET = 2048;      // distinct values tracked per warp (sum over k > 1 attributes)

struct GTmp {
  void* p = nullptr;
  cudaStream_t s;
  explicit GTmp(cudaStream_t st) : s(st) {}
  ~GTmp() { if (p) cudaFreeAsync(p, s); }
  wg_status get(size_t bytes) {
    if (p) cudaFreeAsync(p, s);
    p = nullptr;
    if (cudaMallocAsync(&p, std::max<size_t>(bytes, 256), s) != cudaSuccess) {
      set_error("cudaMallocAsync(tmp) failed");
      return WG_ERR_NOMEM;
    }
    return WG_OK;
  }
  template <typename T> T* as() { return static_cast<T*>(p); }
};

template <typename T>
wg_status galloc(wg_gpart_s* g, T** p, size_t n, cudaStream_t s) {
  void* q = nullptr;
  if (cudaMallocAsync(&q, std::max<size_t>(n * sizeof(T), 256), s) != cudaSuccess) {
    set_error("cudaMallocAsync failed");
    return WG_ERR_NOMEM;
  }
  g->allocs.push_back(q);
  *p = static_cast<T*>(q);
  return WG_OK;
}

struct AttrSrc {
  const int32_t *src, *dst, *type;
  const int32_t* deg;
};

__device__ __forceinline__ uint32_t attr_val(const AttrSrc& a, int attr, int32_t e) {
  switch (attr) {
    case 0: return (uint32_t)a.dst[e];
    case 1: return (uint32_t)a.src[e];
    case 2: return a.type ? (uint32_t)a.type[e] : 0u;
    case 3: return (uint32_t)a.deg[a.dst[e]];
    default: return (uint32_t)e;
  }
}

__global__ void k_iota(int32_t* p, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    p[i] = (int32_t)i;
}

__global__ void k_keys(AttrSrc a, int attr, const int32_t* perm, uint32_t* key, int64_t n) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    key[i] = attr_val(a, attr, perm[i]);
}

__global__ void k_deg(const int32_t* idx, int64_t E, int32_t* deg) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < E; i += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(deg + idx[i], 1);
}

__global__ void k_scales(const int32_t* din, const int32_t* dout, int64_t V, float* rs_in, float* rs_out, float* inv) {
  for (int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; v < V; v += (int64_t)gridDim.x * blockDim.x) {
    const float di = (float)max(din[v], 1), dO = (float)max(dout[v], 1);
    rs_in[v] = rsqrtf(di); rs_out[v] = rsqrtf(dO); inv[v] = 1.f / di;
  }
}

// group start flags: a uniq = 1 attribute changes (position 0 always starts)
struct Spec {
  int n;                 // restrictions
  int attr[5], k[5];
};

__global__ void k_group_flags(AttrSrc a, Spec sp, const int32_t* perm, int64_t n, uint8_t* f) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    bool st = i == 0;
    for (int r = 0; r < sp.n && !st; ++r)
      if (sp.k[r] == 1 && attr_val(a, sp.attr[r], perm[i]) != attr_val(a, sp.attr[r], perm[i - 1])) st = true;
    f[i] = st ? 1 : 0;
  }
}

// One warp per group: the greedy scan of P:L1431-1451.  Writes start[i] = 1
// at the first edge of every gTask (the group's first edge included).
__global__ void __launch_bounds__(128) k_greedy(AttrSrc a, Spec sp, const int32_t* perm, const int64_t* gstart,
                                                int64_t ngroups, int64_t E, uint8_t* start) {
  extern __shared__ uint32_t gset[];                       // [4 warps][MAX_SET]
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t g = (int64_t)blockIdx.x * 4 + warp;
  if (g >= ngroups) return;
  uint32_t* set = gset + warp * MAX_SET;
  // restrictions that can break a gTask inside a group: k > 1
  int off[5], cnt[5], kk[5], at[5], nr = 0;
  uint32_t last[5];
  int o = 0;
  for (int r = 0; r < sp.n; ++r)
    if (sp.k[r] > 1) { at[nr] = sp.attr[r]; kk[nr] = sp.k[r]; off[nr] = o; o += (sp.attr[r] == 4 ? 0 : sp.k[r]); ++nr; }
  const int64_t b = gstart[g], e = gstart[g + 1];
  for (int r = 0; r < nr; ++r) cnt[r] = 0;
  for (int64_t i = b; i < e; ++i) {
    const int32_t eid = perm[i];
    bool fits = true, isnew[5];
    uint32_t v[5];
    for (int r = 0; r < nr; ++r) {
      v[r] = attr_val(a, at[r], eid);
      bool nw;
      if (at[r] == 4) nw = true;                               // edge ids are all distinct
      else if (cnt[r] > 0 && v[r] == last[r]) nw = false;      // run of equal values
      else {
        bool found = false;
        for (int j0 = 0; j0 < cnt[r] && !found; j0 += 32) {
          const int j = j0 + lane;
          found = __any_sync(0xffffffffu, j < cnt[r] && set[off[r] + j] == v[r]);
        }
        nw = !found;
      }
      isnew[r] = nw;
      if (nw && cnt[r] == kk[r]) fits = false;
    }
    if (!fits || i == b) {
      if (lane == 0) start[i] = 1;
      for (int r = 0; r < nr; ++r) { cnt[r] = 0; isnew[r] = true; }
    }
    for (int r = 0; r < nr; ++r) {
      if (isnew[r]) {
        if (at[r] != 4 && lane == 0) set[off[r] + cnt[r]] = v[r];
        ++cnt[r];
      }
      last[r] = v[r];
    }
    __syncwarp();
  }
}

__global__ void k_task_of(const uint8_t* start, int64_t n, int32_t* mark) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    mark[i] = start[i];
}

__global__ void k_gather_sorted(const int32_t* perm, const int32_t* src, const int32_t* dst, int64_t n, int32_t* ss,
                                int32_t* ds) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    ss[i] = src[perm[i]];
    ds[i] = dst[perm[i]];
  }
}

// per task: bounds, type of the first edge, d_lo / d_hi (warp reductions)
__global__ void k_task_rec(const int64_t* starts, int64_t nt, int64_t E, const int32_t* perm, const int32_t* ds,
                           const int32_t* type, wg_task* t) {
  const int lane = threadIdx.x & 31;
  const int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (w >= nt) return;
  const int64_t b = starts[w], e = w + 1 < nt ? starts[w + 1] : E;
  int32_t lo = INT32_MAX, hi = INT32_MIN;
  for (int64_t i = b + lane; i < e; i += 32) { lo = min(lo, ds[i]); hi = max(hi, ds[i]); }
  for (int o = 16; o; o >>= 1) {
    lo = min(lo, __shfl_xor_sync(0xffffffffu, lo, o));
    hi = max(hi, __shfl_xor_sync(0xffffffffu, hi, o));
  }
  if (lane == 0) {
    wg_task r;
    r.tile = -1;
    r.type = type ? type[perm[b]] : 0;
    r.e_begin = b; r.e_end = e;
    r.d_lo = lo; r.d_hi = hi;
    r.flags = 0;
    r.n_uniq_src = 0;
    t[w] = r;
  }
}

__global__ void k_uniq_keys(const int32_t* task_of, const int32_t* ss, int64_t n, uint64_t* k) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    k[i] = ((uint64_t)(uint32_t)task_of[i] << 32) | (uint32_t)ss[i];
}

__global__ void k_uniq_count(const uint64_t* k, int64_t n, wg_task* t) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    if (i == 0 || k[i] != k[i - 1]) atomicAdd(&t[k[i] >> 32].n_uniq_src, 1);
}

// ---------------------------------------------------------------- executor
template <typename T> __device__ __forceinline__ void load4(const T* p, float* f);
template <> __device__ __forceinline__ void load4<float>(const float* p, float* f) {
  const float4 v = __ldg(reinterpret_cast<const float4*>(p));
  f[0] = v.x; f[1] = v.y; f[2] = v.z; f[3] = v.w;
}
template <> __device__ __forceinline__ void load4<__nv_bfloat16>(const __nv_bfloat16* p, float* f) {
  const uint2 v = __ldg(reinterpret_cast<const uint2*>(p));
  f[0] = __uint_as_float(v.x << 16); f[1] = __uint_as_float(v.x & 0xffff0000u);
  f[2] = __uint_as_float(v.y << 16); f[3] = __uint_as_float(v.y & 0xffff0000u);
}

__device__ __forceinline__ void red4(float* p, const float* f) {
  asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(f[0]), "f"(f[1]), "f"(f[2]), "f"(f[3])
               : "memory");
}

// One warp per chunk of CH sorted edges (chunks never straddle gTasks);
// each lane owns 4 columns per 128-column slice; a run of equal destinations
// is reduced in registers and flushed with one vector atomic per lane.
template <typename T>
__global__ void __launch_bounds__(256) k_gagg(const int4* chunks, int64_t nchunks, const int32_t* ss,
                                              const int32_t* ds, const float* gs, const T* x, int64_t ldx, int F,
                                              float* acc, int64_t lda) {
  const int lane = threadIdx.x & 31;
  const int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (w >= nchunks) return;
  const int4 ch = chunks[w];
  const int64_t b = ((int64_t)ch.y << 32) | (uint32_t)ch.x, e = b + ch.z;
  for (int c0 = 0; c0 < F; c0 += 128) {
    const int c = c0 + lane * 4;
    const bool on = c < F;
    float a[4] = {0.f, 0.f, 0.f, 0.f};
    int32_t cur = ds[b];
    for (int64_t i = b; i < e; ++i) {
      const int32_t d = ds[i];
      if (d != cur) {
        if (on) red4(acc + (int64_t)cur * lda + c, a);
        a[0] = a[1] = a[2] = a[3] = 0.f;
        cur = d;
      }
      const int32_t s = ss[i];
      if (on) {
        float f[4];
        load4<T>(x + (int64_t)s * ldx + c, f);
        const float sc = gs ? gs[s] : 1.f;
#pragma unroll
        for (int j = 0; j < 4; ++j) a[j] += sc * f[j];
      }
    }
    if (on) red4(acc + (int64_t)cur * lda + c, a);
  }
}

template <typename T>
__global__ void k_gfinish(const float* acc, int64_t lda, int64_t V, int F, const float* rs, T* out, int64_t ldo) {
  const int64_t n = V * (int64_t)ldo;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t v = t / ldo;
    const int c = (int)(t % ldo);
    const float val = c < F ? acc[v * lda + c] * (rs ? rs[v] : 1.f) : 0.f;
    out[t] = (T)val;   // RNE for bf16 (Q23)
  }
}

int64_t gacc_ld(int F) { return rup(F, 128); }

}  // namespace
}  // namespace wg

extern "C" {

wg_status wg_gpart_create(const wg_graph_desc* d, const wg_restriction* r, int32_t n_r, int device, wg_stream stream,
                          wg_gpart* out) {
  using namespace wg;
  WG_REQ(d && out && (n_r == 0 || r) && n_r >= 0 && n_r <= 5, WG_ERR_INVALID, "wg_gpart_create: bad argument");
  const int64_t V = d->num_vertices, E = d->num_edges;
  WG_REQ(V >= 1 && V < (1ll << 31) && E >= 0 && E < (1ll << 31), WG_ERR_INVALID, "wg_gpart_create: sizes");
  WG_REQ(E == 0 || (d->src && (d->dst || d->indptr)), WG_ERR_INVALID, "wg_gpart_create: src / dst");
  Spec sp{};
  sp.n = n_r;
  int set_total = 0;
  bool used[5] = {false, false, false, false, false};
  for (int i = 0; i < n_r; ++i) {
    WG_REQ(r[i].attr >= 0 && r[i].attr <= 4 && !used[r[i].attr], WG_ERR_INVALID,
           "wg_gpart_create: attributes 0..4, each at most once");
    WG_REQ(r[i].k >= 1 || r[i].k == WG_UNIQ_MIN, WG_ERR_INVALID, "wg_gpart_create: k >= 1 or WG_UNIQ_MIN");
    used[r[i].attr] = true;
    sp.attr[i] = r[i].attr;
    sp.k[i] = r[i].k;
    if (r[i].k > 1 && r[i].attr != 4) set_total += r[i].k;
  }
  WG_REQ(set_total <= MAX_SET, WG_ERR_UNSUPPORTED, "wg_gpart_create: sum of k over k > 1 attributes > 2048");
  WG_CK(cudaSetDevice(device));
  cudaStream_t s = (cudaStream_t)stream;
  auto* g = new wg_gpart_s();
  g->device = device; g->V = V; g->E = E;
  auto fail = [&](wg_status st) { for (void* q : g->allocs) cudaFreeAsync(q, s); delete g; return st; };
  // device copies of the edge attributes (inputs may be host or device)
  auto dev_copy = [&](const void* p, size_t bytes, void** o) -> wg_status {
    cudaPointerAttributes at;
    bool dev = false;
    if (cudaPointerGetAttributes(&at, p) == cudaSuccess)
      dev = at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged;
    else
      cudaGetLastError();
    if (cudaMallocAsync(o, std::max<size_t>(bytes, 256), s) != cudaSuccess) return WG_ERR_NOMEM;
    g->allocs.push_back(*o);
    if (bytes && cudaMemcpyAsync(*o, p, bytes, dev ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice, s) !=
                     cudaSuccess)
      return WG_ERR_CUDA;
    return WG_OK;
  };
  int32_t *src = nullptr, *dst = nullptr, *type = nullptr;
  wg_status st;
  if (E > 0) {
    if ((st = dev_copy(d->src, 4 * E, (void**)&src)) != WG_OK) return fail(st);
    if (d->indptr) {
      std::vector<int64_t> ip(V + 1);
      cudaPointerAttributes at;
      bool dev = cudaPointerGetAttributes(&at, d->indptr) == cudaSuccess &&
                 (at.type == cudaMemoryTypeDevice || at.type == cudaMemoryTypeManaged);
      cudaGetLastError();
      if (cudaMemcpy(ip.data(), d->indptr, 8 * (V + 1), dev ? cudaMemcpyDeviceToHost : cudaMemcpyHostToHost) !=
          cudaSuccess)
        return fail(WG_ERR_CUDA);
      std::vector<int32_t> hd(E);
      for (int64_t v = 0; v < V; ++v) for (int64_t e = ip[v]; e < ip[v + 1]; ++e) hd[e] = (int32_t)v;
      if ((st = dev_copy(hd.data(), 4 * E, (void**)&dst)) != WG_OK) return fail(st);
      if (cudaStreamSynchronize(s) != cudaSuccess) return fail(WG_ERR_CUDA);
    } else if ((st = dev_copy(d->dst, 4 * E, (void**)&dst)) != WG_OK) {
      return fail(st);
    }
    if (d->etype && (st = dev_copy(d->etype, 4 * E, (void**)&type)) != WG_OK) return fail(st);
  }
  int32_t *din = nullptr, *dout = nullptr;
  if ((st = galloc(g, &din, V, s)) != WG_OK || (st = galloc(g, &dout, V, s)) != WG_OK ||
      (st = galloc(g, &g->rs_in, V, s)) != WG_OK || (st = galloc(g, &g->rs_out, V, s)) != WG_OK ||
      (st = galloc(g, &g->inv_in, V, s)) != WG_OK || (st = galloc(g, &g->perm, E, s)) != WG_OK ||
      (st = galloc(g, &g->src_s, E, s)) != WG_OK || (st = galloc(g, &g->dst_s, E, s)) != WG_OK)
    return fail(st);
  WG_CK(cudaMemsetAsync(din, 0, 4 * V, s));
  WG_CK(cudaMemsetAsync(dout, 0, 4 * V, s));
  const unsigned G = 148 * 8;
  if (E > 0) {
    WG_LAUNCH(k_deg, G, 256, 0, s, dst, E, din);
    WG_LAUNCH(k_deg, G, 256, 0, s, src, E, dout);
  }
  WG_LAUNCH(k_scales, G, 256, 0, s, din, dout, V, g->rs_in, g->rs_out, g->inv_in);
  if (E == 0) {
    WG_CK(cudaStreamSynchronize(s));
    *out = g;
    return WG_OK;
  }
  AttrSrc a{src, dst, type, din};
  // sort key (Q25), most significant first
  int key[8], nk = 0;
  bool in_key[5] = {false, false, false, false, false};
  for (int pass = 0; pass < 3; ++pass)
    for (int i = 0; i < n_r; ++i) {
      const bool take = pass == 0 ? sp.k[i] == 1 : pass == 1 ? sp.k[i] == WG_UNIQ_MIN : (sp.k[i] > 1 && sp.attr[i] != 4);
      if (take && !in_key[sp.attr[i]]) { key[nk++] = sp.attr[i]; in_key[sp.attr[i]] = true; }
    }
  if (!in_key[0]) key[nk++] = 0;
  // LSD: edge-id order first (iota), then stable sorts from the least significant attribute
  GTmp kbuf(s), kbuf2(s), pbuf(s), temp(s);
  if ((st = kbuf.get(4 * E)) != WG_OK || (st = kbuf2.get(4 * E)) != WG_OK || (st = pbuf.get(4 * E)) != WG_OK)
    return fail(st);
  WG_LAUNCH(k_iota, G, 256, 0, s, g->perm, E);
  for (int i = nk - 1; i >= 0; --i) {
    WG_LAUNCH(k_keys, G, 256, 0, s, a, key[i], g->perm, kbuf.as<uint32_t>(), E);
    size_t tb = 0;
    WG_CK(cub::DeviceRadixSort::SortPairs(nullptr, tb, kbuf.as<uint32_t>(), kbuf2.as<uint32_t>(), g->perm,
                                          pbuf.as<int32_t>(), E, 0, 32, s));
    if ((st = temp.get(tb)) != WG_OK) return fail(st);
    WG_CK(cub::DeviceRadixSort::SortPairs(temp.p, tb, kbuf.as<uint32_t>(), kbuf2.as<uint32_t>(), g->perm,
                                          pbuf.as<int32_t>(), E, 0, 32, s));
    ++launch_counter();
    WG_CK(cudaMemcpyAsync(g->perm, pbuf.p, 4 * E, cudaMemcpyDeviceToDevice, s));
  }
  // groups (runs of equal uniq = 1 attributes) and the greedy scan
  GTmp flags(s), gst(s), iota64(s), nsel(s), start(s);
  if ((st = flags.get(E)) != WG_OK || (st = gst.get(8 * (E + 1))) != WG_OK || (st = iota64.get(8 * E)) != WG_OK ||
      (st = nsel.get(8)) != WG_OK || (st = start.get(E)) != WG_OK)
    return fail(st);
  WG_LAUNCH(k_group_flags, G, 256, 0, s, a, sp, g->perm, E, flags.as<uint8_t>());
  {
    cub::CountingInputIterator<int64_t> it(0);
    size_t tb = 0;
    WG_CK(cub::DeviceSelect::Flagged(nullptr, tb, it, flags.as<uint8_t>(), gst.as<int64_t>(), nsel.as<int64_t>(), E,
                                     s));
    if ((st = temp.get(tb)) != WG_OK) return fail(st);
    WG_CK(cub::DeviceSelect::Flagged(temp.p, tb, it, flags.as<uint8_t>(), gst.as<int64_t>(), nsel.as<int64_t>(), E,
                                     s));
    ++launch_counter();
  }
  int64_t ngroups = 0;
  WG_CK(cudaMemcpyAsync(&ngroups, nsel.p, 8, cudaMemcpyDeviceToHost, s));
  WG_CK(cudaStreamSynchronize(s));
  WG_CK(cudaMemcpyAsync(gst.as<int64_t>() + ngroups, &E, 8, cudaMemcpyHostToDevice, s));
  WG_CK(cudaMemsetAsync(start.p, 0, E, s));
  const size_t smem = 4 * MAX_SET * sizeof(uint32_t);
  static bool attr_set = false;
  if (!attr_set) {
    cudaFuncSetAttribute(k_greedy, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    attr_set = true;
  }
  WG_LAUNCH(k_greedy, (unsigned)cdiv(ngroups, 4), 128, smem, s, a, sp, g->perm, gst.as<int64_t>(), ngroups, E,
            start.as<uint8_t>());
  // task starts -> task table
  GTmp tstart(s);
  if ((st = tstart.get(8 * E)) != WG_OK) return fail(st);
  {
    cub::CountingInputIterator<int64_t> it(0);
    size_t tb = 0;
    WG_CK(cub::DeviceSelect::Flagged(nullptr, tb, it, start.as<uint8_t>(), tstart.as<int64_t>(), nsel.as<int64_t>(),
                                     E, s));
    if ((st = temp.get(tb)) != WG_OK) return fail(st);
    WG_CK(cub::DeviceSelect::Flagged(temp.p, tb, it, start.as<uint8_t>(), tstart.as<int64_t>(), nsel.as<int64_t>(),
                                     E, s));
    ++launch_counter();
  }
  int64_t nt = 0;
  WG_CK(cudaMemcpyAsync(&nt, nsel.p, 8, cudaMemcpyDeviceToHost, s));
  WG_CK(cudaStreamSynchronize(s));
  g->n_tasks = nt;
  if ((st = galloc(g, &g->tasks, nt, s)) != WG_OK) return fail(st);
  WG_LAUNCH(k_gather_sorted, G, 256, 0, s, g->perm, src, dst, E, g->src_s, g->dst_s);
  WG_LAUNCH(k_task_rec, (unsigned)cdiv(nt * 32, 256), 256, 0, s, tstart.as<int64_t>(), nt, E, g->perm, g->dst_s, type,
            g->tasks);
  // n_uniq_src: (task, src) keys sorted, heads counted per task
  GTmp tof(s), mark(s), uk(s), uk2(s);
  if ((st = mark.get(4 * E)) != WG_OK || (st = tof.get(4 * E)) != WG_OK || (st = uk.get(8 * E)) != WG_OK ||
      (st = uk2.get(8 * E)) != WG_OK)
    return fail(st);
  WG_LAUNCH(k_task_of, G, 256, 0, s, start.as<uint8_t>(), E, mark.as<int32_t>());
  {
    size_t tb = 0;
    WG_CK(cub::DeviceScan::InclusiveSum(nullptr, tb, mark.as<int32_t>(), tof.as<int32_t>(), E, s));
    if ((st = temp.get(tb)) != WG_OK) return fail(st);
    WG_CK(cub::DeviceScan::InclusiveSum(temp.p, tb, mark.as<int32_t>(), tof.as<int32_t>(), E, s));
    ++launch_counter();
  }
  // task ids are 1-based after the inclusive sum: shift inside the key
  WG_LAUNCH(k_uniq_keys, G, 256, 0, s, tof.as<int32_t>(), g->src_s, E, uk.as<uint64_t>());
  {
    size_t tb = 0;
    WG_CK(cub::DeviceRadixSort::SortKeys(nullptr, tb, uk.as<uint64_t>(), uk2.as<uint64_t>(), E, 0, 64, s));
    if ((st = temp.get(tb)) != WG_OK) return fail(st);
    WG_CK(cub::DeviceRadixSort::SortKeys(temp.p, tb, uk.as<uint64_t>(), uk2.as<uint64_t>(), E, 0, 64, s));
    ++launch_counter();
  }
  WG_LAUNCH(k_uniq_count, G, 256, 0, s, uk2.as<uint64_t>(), E, g->tasks - 1);
  g->h_tasks.resize(nt);
  WG_CK(cudaMemcpyAsync(g->h_tasks.data(), g->tasks, sizeof(wg_task) * nt, cudaMemcpyDeviceToHost, s));
  WG_CK(cudaStreamSynchronize(s));
  WG_CK(cudaGetLastError());
  *out = g;
  return WG_OK;
}

wg_status wg_gpart_info(wg_gpart g, int64_t info[3]) {
  WG_REQ(g && info, WG_ERR_INVALID, "wg_gpart_info: null");
  info[0] = g->V; info[1] = g->E; info[2] = g->n_tasks;
  return WG_OK;
}

wg_status wg_gpart_export(wg_gpart g, int64_t* perm, wg_task* tasks) {
  WG_REQ(g, WG_ERR_INVALID, "wg_gpart_export: null");
  WG_CK(cudaSetDevice(g->device));
  if (perm && g->E) {
    std::vector<int32_t> p(g->E);
    WG_CK(cudaMemcpy(p.data(), g->perm, 4 * g->E, cudaMemcpyDeviceToHost));
    for (int64_t i = 0; i < g->E; ++i) perm[i] = p[i];
  }
  if (tasks) std::copy(g->h_tasks.begin(), g->h_tasks.end(), tasks);
  return WG_OK;
}

size_t wg_gpart_workspace(wg_gpart g, int32_t F) {
  if (!g || F < 1) return 0;
  const int64_t nch = (int64_t)g->n_tasks + wg::cdiv(g->E, 64) + 1;
  return (size_t)g->V * wg::gacc_ld(F) * sizeof(float) + 256 + sizeof(int4) * nch;
}

wg_status wg_gpart_aggregate(wg_gpart g, wg_dtype dt, int32_t F, wg_norm norm, const void* x, int64_t ldx, void* out,
                             int64_t ldo, void* workspace, wg_stream stream) {
  using namespace wg;
  WG_REQ(g && x && out && workspace && F >= 1, WG_ERR_INVALID, "wg_gpart_aggregate: null argument");
  const int es = dsize(dt);
  WG_REQ(F % 4 == 0 && (ldx * es) % 16 == 0 && ldx >= F && ldo >= F && (ldo * es) % 16 == 0, WG_ERR_UNSUPPORTED,
         "wg_gpart_aggregate: F a multiple of 4, 16-byte row pitches");
  WG_CK(cudaSetDevice(g->device));
  cudaStream_t s = (cudaStream_t)stream;
  const int64_t lda = gacc_ld(F);
  float* acc = static_cast<float*>(workspace);
  int4* chunks = reinterpret_cast<int4*>(static_cast<char*>(workspace) + rup((int64_t)g->V * lda * 4, 256));
  // chunks of <= 64 edges that never straddle a gTask (host table, built per call)
  std::vector<int4> h;
  for (const wg_task& t : g->h_tasks)
    for (int64_t b = t.e_begin; b < t.e_end; b += 64) {
      const int64_t n = std::min<int64_t>(64, t.e_end - b);
      h.push_back(make_int4((int32_t)(b & 0xffffffff), (int32_t)(b >> 32), (int32_t)n, 0));
    }
  WG_CK(cudaMemsetAsync(acc, 0, sizeof(float) * g->V * lda, s));
  if (!h.empty()) WG_CK(cudaMemcpyAsync(chunks, h.data(), sizeof(int4) * h.size(), cudaMemcpyHostToDevice, s));
  const float* gs = norm == WG_NORM_BOTH ? g->rs_out : nullptr;
  const float* rs = norm == WG_NORM_BOTH ? g->rs_in : norm == WG_NORM_RIGHT ? g->inv_in : nullptr;
  ProfScope ps(PK_AGG, s, (double)g->E * (4.0 + F * es) + (double)g->V * F * (4.0 + es), 2.0 * g->E * F);
  const int64_t nch = (int64_t)h.size();
  if (nch) {
    if (dt == WG_BF16)
      WG_LAUNCH(k_gagg<__nv_bfloat16>, (unsigned)cdiv(nch * 32, 256), 256, 0, s, chunks, nch, g->src_s, g->dst_s, gs,
                static_cast<const __nv_bfloat16*>(x), ldx, F, acc, lda);
    else
      WG_LAUNCH(k_gagg<float>, (unsigned)cdiv(nch * 32, 256), 256, 0, s, chunks, nch, g->src_s, g->dst_s, gs,
                static_cast<const float*>(x), ldx, F, acc, lda);
  }
  const unsigned G = (unsigned)std::min<int64_t>(cdiv(g->V * ldo, 256), 148 * 16);
  if (dt == WG_BF16)
    WG_LAUNCH(k_gfinish<__nv_bfloat16>, G, 256, 0, s, acc, lda, g->V, F, rs, static_cast<__nv_bfloat16*>(out), ldo);
  else
    WG_LAUNCH(k_gfinish<float>, G, 256, 0, s, acc, lda, g->V, F, rs, static_cast<float*>(out), ldo);
  return WG_OK;
}

wg_status wg_gpart_destroy(wg_gpart g) {
  if (!g) return WG_OK;
  cudaSetDevice(g->device);
  cudaDeviceSynchronize();
  for (void* q : g->allocs) cudaFree(q);
  delete g;
  return WG_OK;
}

}  // extern "C"
