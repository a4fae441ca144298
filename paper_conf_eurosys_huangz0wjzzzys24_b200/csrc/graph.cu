// Graph ingest (a1) and GPU gTask partitioner (a2, a3).
//
// The partition is the paper's greedy restriction scan for the
// restriction instance uniq(dst-range of T rows) = 1 [& uniq(type) = 1] &
// uniq(edge-id) <= E_max (Fig 7(c)(d); degree-aware splitting of
// frequent-value / overfill destinations).  It runs on the GPU
// ("WiseGraph processes graph data in parallel using GPU"):
//   1. composite key (tile, type, row-in-tile), stable radix sort of edge ids
//      (CUB; stable => ties broken by edge id, so perm is unique);
//   2. segment / group boundaries by flag + select;
//   3. one thread per (tile, type) group replays the greedy scan over its
//      segments (count pass, scan, write pass);
//   4. n_uniq_src per task by a (task, src) key sort.
// The result must equal the oracle bit for bit (tests/test_gpu_partition.py).
#include <cub/cub.cuh>

#include <algorithm>
#include <numeric>

#include "wg_internal.cuh"

namespace wg {

namespace {

template <typename T>
wg_status dalloc(wg_graph_s* g, T** p, size_t n, cudaStream_t s) {
  void* q = nullptr;
  size_t bytes = std::max<size_t>(n * sizeof(T), 256);
  cudaError_t e = cudaMallocAsync(&q, bytes, s);
  if (e != cudaSuccess) {
    set_error(std::string("cudaMallocAsync: ") + cudaGetErrorString(e));
    return WG_ERR_NOMEM;
  }
  g->allocs.push_back(q);
  *p = static_cast<T*>(q);
  return WG_OK;
}

// scoped temporary device buffer (stream-ordered)
struct Tmp {
  void* p = nullptr;
  cudaStream_t s;
  explicit Tmp(cudaStream_t st) : s(st) {}
  ~Tmp() { if (p) cudaFreeAsync(p, s); }
  wg_status get(size_t bytes) {
    if (p) cudaFreeAsync(p, s);
    p = nullptr;
    cudaError_t e = cudaMallocAsync(&p, std::max<size_t>(bytes, 256), s);
    if (e != cudaSuccess) { set_error("cudaMallocAsync(tmp) failed"); return WG_ERR_NOMEM; }
    return WG_OK;
  }
  template <typename T> T* as() { return static_cast<T*>(p); }
};

__global__ void k_coo_from_csr(const int64_t* indptr, int64_t V, int32_t* dst) {
  int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (v >= V) return;
  for (int64_t e = indptr[v]; e < indptr[v + 1]; ++e) dst[e] = (int32_t)v;
}

__global__ void k_validate(const int32_t* src, const int32_t* dst, const int32_t* et, int64_t E,
                           int64_t V, int32_t R, int32_t* bad) {
  int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (e >= E) return;
  bool ok = src[e] >= 0 && src[e] < V && dst[e] >= 0 && dst[e] < V;
  if (et) ok = ok && et[e] >= 0 && et[e] < R;
  if (!ok) atomicExch(bad, 1);
}

__global__ void k_degrees(const int32_t* src, const int32_t* dst, int64_t E, int32_t* din, int32_t* dout) {
  int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (e >= E) return;
  atomicAdd(&din[dst[e]], 1);
  atomicAdd(&dout[src[e]], 1);
}

__global__ void k_scales(const int32_t* din, const int32_t* dout, int64_t V, float* rs_in, float* rs_out,
                         float* inv_in) {
  int64_t v = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (v >= V) return;
  float a = (float)max(din[v], 1), b = (float)max(dout[v], 1);
  rs_in[v] = 1.0f / sqrtf(a);
  rs_out[v] = 1.0f / sqrtf(b);
  inv_in[v] = 1.0f / a;
}

__global__ void k_make_keys(const int32_t* kv, const int32_t* et, int64_t E, int32_t T, int32_t Rk,
                            uint64_t* keys, int32_t* vals) {
  int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (e >= E) return;
  uint64_t v = (uint64_t)kv[e];
  uint64_t t = et ? (uint64_t)et[e] : 0;
  keys[e] = ((v / T) * (uint64_t)Rk + t) * (uint64_t)T + (v % T);
  vals[e] = (int32_t)e;
}

// first position whose key >= thr (keys sorted ascending)
__global__ void k_lower_bound(const uint64_t* keys, int64_t n, uint64_t thr, int64_t* out) {
  int64_t lo = 0, hi = n;
  while (lo < hi) {
    int64_t mid = (lo + hi) / 2;
    if (keys[mid] < thr) lo = mid + 1; else hi = mid;
  }
  *out = lo;
}

__global__ void k_gather_side(const int32_t* perm, int64_t n, const int32_t* kv, const int32_t* ov,
                              const int32_t* et, int32_t* key, int32_t* idx, int32_t* type) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  int32_t e = perm[i];
  key[i] = kv[e];
  idx[i] = ov[e];
  if (type) type[i] = et ? et[e] : 0;
}

// flags: segment start (new key vertex or new type), group start (new tile or type)
__global__ void k_flags(const uint64_t* keys, int64_t n, int32_t T, uint8_t* seg, uint8_t* grp) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= n) return;
  bool s = (i == 0) || keys[i] != keys[i - 1];
  bool g = (i == 0) || (keys[i] / T) != (keys[i - 1] / T);
  seg[i] = s;
  grp[i] = g;
}

__global__ void k_iota64(int64_t* p, int64_t n) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i < n) p[i] = i;
}

// group g's first segment index: flag segments whose start is a group start
__global__ void k_seg_is_grp(const int64_t* seg_off, int64_t nseg, const uint8_t* grp, uint8_t* f) {
  int64_t s = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (s < nseg) f[s] = grp[seg_off[s]];
}

// Greedy pack of one (tile, type) group's segments.
// mode 0: count tasks; mode 1: write tasks at out[base]
__global__ void k_pack(const int64_t* seg_off /*nseg+1*/, const int64_t* grp_first /*ngrp+1*/, int64_t ngrp,
                       const uint64_t* keys, const int32_t* key_vertex, int32_t T, int32_t Rk,
                       int64_t E_max, int mode, int64_t* counts, const int64_t* offsets, wg_task* out) {
  int64_t g = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (g >= ngrp) return;
  int64_t s0 = grp_first[g], s1 = grp_first[g + 1];
  uint64_t k0 = keys[seg_off[s0]] / T;     // (tile * Rk + type)
  int32_t tile = (int32_t)(k0 / Rk), type = (int32_t)(k0 % Rk);
  int64_t n = 0;
  wg_task* o = mode ? out + offsets[g] : nullptr;
  auto emit = [&](int64_t b, int64_t e, int32_t flags) {
    if (mode) {
      wg_task t;
      t.tile = tile; t.type = type; t.e_begin = b; t.e_end = e;
      t.d_lo = key_vertex[b]; t.d_hi = key_vertex[e - 1];
      t.flags = flags; t.n_uniq_src = 0;
      o[n] = t;
    }
    ++n;
  };
  int64_t open_b = -1;
  for (int64_t s = s0; s < s1; ++s) {
    int64_t b = seg_off[s], e = seg_off[s + 1], len = e - b;
    if (len > E_max) {
      if (open_b >= 0) emit(open_b, b, 0);
      open_b = -1;
      for (int64_t c = b; c < e; c += E_max) emit(c, min(c + E_max, e), WG_TASK_SPLIT);
    } else if (open_b < 0) {
      open_b = b;
    } else if ((b - open_b) + len > E_max) {
      emit(open_b, b, 0);
      open_b = b;
    }
  }
  if (open_b >= 0) emit(open_b, seg_off[s1], 0);
  if (!mode) counts[g] = n;
}

__global__ void k_task_starts(const wg_task* tasks, int64_t nt, int32_t* mark) {
  int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (t < nt) mark[tasks[t].e_begin] = (int32_t)t;
}

__global__ void k_uniq_keys(const int32_t* task_of, const int32_t* idx, int64_t n, uint64_t* k) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i < n) k[i] = ((uint64_t)(uint32_t)task_of[i] << 32) | (uint32_t)idx[i];
}

// n_uniq_src per task: sorted (task, src) keys, one count per first-of-run
// key.  Warp-aggregated: the lanes holding one task add their flags with a
// single atomic (a gTask's keys are contiguous, so per-lane atomics on one
// counter serialised: 17 ms per side at C4).
__global__ void k_uniq_count(const uint64_t* k, int64_t n, int32_t* cnt) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const bool in = i < n;
  const bool first = in && (i == 0 || k[i] != k[i - 1]);
  const unsigned task = in ? (unsigned)(k[i] >> 32) : 0xffffffffu;
  const unsigned peers = __match_any_sync(0xffffffffu, task);
  const unsigned flags = __ballot_sync(0xffffffffu, first) & peers;
  if (in && (int)(threadIdx.x & 31) == __ffs(peers) - 1 && flags) atomicAdd(&cnt[task], __popc(flags));
}

__global__ void k_set_uniq(wg_task* t, const int32_t* cnt, int64_t nt) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i < nt) t[i].n_uniq_src = cnt[i];
}

__global__ void k_row_hist(const int32_t* key, int64_t n, int64_t vb, int64_t* cnt) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i < n) atomicAdd((unsigned long long*)&cnt[key[i] - vb + 1], 1ULL);
}

__global__ void k_inv_perm(const int32_t* perm, int64_t n, int64_t* inv) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i < n) inv[perm[i]] = i;
}

__global__ void k_fwdpos(const int32_t* permT, int64_t n, const int64_t* inv, int64_t* out) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i < n) out[i] = inv[permT[i]];
}

inline unsigned nblk(int64_t n, int b = 256) { return (unsigned)std::max<int64_t>(1, cdiv(n, b)); }

int bits_for(uint64_t maxval) {
  int b = 1;
  while (b < 64 && (maxval >> b) != 0) ++b;
  return b;
}

// Partition one side.  kv = key vertex per edge (dst fwd / src transposed),
// ov = other endpoint.  Owned key rows [vb, ve).
// |in_r(dst_e)| per global edge id (RGCN NORM_RIGHT, Q2: c_e = 1/|N_v^r|):
// sort the (dst, type) keys of ALL edges, count each edge's key by two binary
// searches -- global, so a rank of a 1-D partition also has the coefficient
// of out-edges whose destination another rank owns
__global__ void k_rel_keys(const int32_t* dst, const int32_t* et, int64_t E, int32_t R, uint64_t* k) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < E; e += (int64_t)gridDim.x * blockDim.x)
    k[e] = (uint64_t)dst[e] * (uint64_t)R + (uint64_t)et[e];
}
__global__ void k_rel_count(const uint64_t* keys, const uint64_t* sorted, int64_t E, int32_t* cnt) {
  for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < E; e += (int64_t)gridDim.x * blockDim.x) {
    const uint64_t k = keys[e];
    int64_t lo = 0, hi = E;
    while (lo < hi) { const int64_t m = (lo + hi) >> 1; if (sorted[m] < k) lo = m + 1; else hi = m; }
    int64_t lo2 = lo, hi2 = E;
    while (lo2 < hi2) { const int64_t m = (lo2 + hi2) >> 1; if (sorted[m] <= k) lo2 = m + 1; else hi2 = m; }
    cnt[e] = (int32_t)(lo2 - lo);
  }
}

wg_status rel_counts(wg_graph_s* g, const int32_t* dst, const int32_t* et, cudaStream_t st) {
  const int64_t E = g->E_total;
  WG_TRY(dalloc(g, &g->rel_cnt, std::max<int64_t>(E, 1), st));
  if (E == 0) return WG_OK;
  Tmp k(st), ks(st), temp(st);
  WG_TRY(k.get(sizeof(uint64_t) * E));
  WG_TRY(ks.get(sizeof(uint64_t) * E));
  const unsigned nb = (unsigned)std::min<int64_t>(nblk(E), 148 * 16);
  WG_LAUNCH(k_rel_keys, nb, 256, 0, st, dst, et, E, g->R, k.as<uint64_t>());
  const int nbits = bits_for((uint64_t)(g->V - 1) * g->R + (g->R - 1));
  size_t tb = 0;
  WG_CK(cub::DeviceRadixSort::SortKeys(nullptr, tb, k.as<uint64_t>(), ks.as<uint64_t>(), E, 0, nbits, st));
  WG_TRY(temp.get(tb));
  WG_CK(cub::DeviceRadixSort::SortKeys(temp.p, tb, k.as<uint64_t>(), ks.as<uint64_t>(), E, 0, nbits, st));
  ++launch_counter();
  WG_LAUNCH(k_rel_count, nb, 256, 0, st, k.as<uint64_t>(), ks.as<uint64_t>(), E, g->rel_cnt);
  return WG_OK;
}

wg_status build_side(wg_graph_s* g, Side& S, const int32_t* kv, const int32_t* ov, const int32_t* et,
                     cudaStream_t st) {
  const int64_t E = g->E_total, T = g->T;
  const int32_t Rk = g->by_type ? g->R : 1;
  const int32_t* etk = g->by_type ? et : nullptr;
  S.n_rows = g->ve - g->vb;

  Tmp keys_in(st), keys_out(st), vals_in(st), vals_out(st), temp(st);
  WG_TRY(keys_in.get(sizeof(uint64_t) * std::max<int64_t>(E, 1)));
  WG_TRY(keys_out.get(sizeof(uint64_t) * std::max<int64_t>(E, 1)));
  WG_TRY(vals_in.get(sizeof(int32_t) * std::max<int64_t>(E, 1)));
  WG_TRY(vals_out.get(sizeof(int32_t) * std::max<int64_t>(E, 1)));
  if (E > 0) {
    WG_LAUNCH(k_make_keys, nblk(E), 256, 0, st, kv, etk, E, (int32_t)T, Rk, keys_in.as<uint64_t>(),
              vals_in.as<int32_t>());
    uint64_t maxkey = (((uint64_t)(g->V - 1) / T) * Rk + (Rk - 1)) * T + (T - 1);
    int nbits = bits_for(maxkey);
    size_t tb = 0;
    WG_CK(cub::DeviceRadixSort::SortPairs(nullptr, tb, keys_in.as<uint64_t>(), keys_out.as<uint64_t>(),
                                          vals_in.as<int32_t>(), vals_out.as<int32_t>(), E, 0, nbits, st));
    WG_TRY(temp.get(tb));
    WG_CK(cub::DeviceRadixSort::SortPairs(temp.p, tb, keys_in.as<uint64_t>(), keys_out.as<uint64_t>(),
                                          vals_in.as<int32_t>(), vals_out.as<int32_t>(), E, 0, nbits, st));
    ++launch_counter();
  }
  // local slice [off, off + n) of the sorted edges (owned key rows)
  int64_t off = 0, endp = E;
  if (E > 0 && (g->vb > 0 || g->ve < g->V)) {
    Tmp lb(st);
    WG_TRY(lb.get(2 * sizeof(int64_t)));
    uint64_t thr0 = ((uint64_t)(g->vb / T) * Rk) * T;
    uint64_t thr1 = g->ve >= g->V ? ~0ULL : ((uint64_t)(g->ve / T) * Rk) * T;
    WG_LAUNCH(k_lower_bound, 1, 1, 0, st, keys_out.as<uint64_t>(), E, thr0, lb.as<int64_t>());
    if (g->ve < g->V) WG_LAUNCH(k_lower_bound, 1, 1, 0, st, keys_out.as<uint64_t>(), E, thr1, lb.as<int64_t>() + 1);
    int64_t h[2] = {0, E};
    WG_CK(cudaMemcpyAsync(h, lb.p, (g->ve < g->V ? 2 : 1) * sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    WG_CK(cudaStreamSynchronize(st));
    off = h[0];
    endp = g->ve < g->V ? h[1] : E;
  }
  const int64_t n = endp - off;
  S.E = n;
  WG_TRY(dalloc(g, &S.perm, n, st));
  WG_TRY(dalloc(g, &S.idx, n, st));
  WG_TRY(dalloc(g, &S.key, n, st));
  if (g->by_type) WG_TRY(dalloc(g, &S.type, n, st));
  if (n > 0) {
    WG_CK(cudaMemcpyAsync(S.perm, vals_out.as<int32_t>() + off, n * sizeof(int32_t), cudaMemcpyDeviceToDevice, st));
    WG_LAUNCH(k_gather_side, nblk(n), 256, 0, st, S.perm, n, kv, ov, et, S.key, S.idx, S.type);
  }
  const uint64_t* keys = keys_out.as<uint64_t>() + off;

  // segments and groups
  int64_t nseg = 0, ngrp = 0;
  Tmp segf(st), grpf(st), iota(st), seg_off(st), sgf(st), grp_first(st), nsel(st);
  if (n > 0) {
    WG_TRY(segf.get(n));
    WG_TRY(grpf.get(n));
    WG_TRY(iota.get(sizeof(int64_t) * n));
    WG_TRY(seg_off.get(sizeof(int64_t) * (n + 1)));
    WG_TRY(nsel.get(sizeof(int64_t) * 2));
    WG_LAUNCH(k_flags, nblk(n), 256, 0, st, keys, n, (int32_t)T, segf.as<uint8_t>(), grpf.as<uint8_t>());
    WG_LAUNCH(k_iota64, nblk(n), 256, 0, st, iota.as<int64_t>(), n);
    size_t tb = 0;
    WG_CK(cub::DeviceSelect::Flagged(nullptr, tb, iota.as<int64_t>(), segf.as<uint8_t>(), seg_off.as<int64_t>(),
                                     nsel.as<int64_t>(), n, st));
    WG_TRY(temp.get(tb));
    WG_CK(cub::DeviceSelect::Flagged(temp.p, tb, iota.as<int64_t>(), segf.as<uint8_t>(), seg_off.as<int64_t>(),
                                     nsel.as<int64_t>(), n, st));
    ++launch_counter();
    WG_CK(cudaMemcpyAsync(&nseg, nsel.p, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    WG_CK(cudaStreamSynchronize(st));
    WG_CK(cudaMemcpyAsync(seg_off.as<int64_t>() + nseg, &n, sizeof(int64_t), cudaMemcpyHostToDevice, st));
    WG_TRY(sgf.get(nseg));
    WG_TRY(grp_first.get(sizeof(int64_t) * (nseg + 1)));
    WG_LAUNCH(k_seg_is_grp, nblk(nseg), 256, 0, st, seg_off.as<int64_t>(), nseg, grpf.as<uint8_t>(), sgf.as<uint8_t>());
    WG_LAUNCH(k_iota64, nblk(nseg), 256, 0, st, iota.as<int64_t>(), nseg);
    tb = 0;
    WG_CK(cub::DeviceSelect::Flagged(nullptr, tb, iota.as<int64_t>(), sgf.as<uint8_t>(), grp_first.as<int64_t>(),
                                     nsel.as<int64_t>(), nseg, st));
    WG_TRY(temp.get(tb));
    WG_CK(cub::DeviceSelect::Flagged(temp.p, tb, iota.as<int64_t>(), sgf.as<uint8_t>(), grp_first.as<int64_t>(),
                                     nsel.as<int64_t>(), nseg, st));
    ++launch_counter();
    WG_CK(cudaMemcpyAsync(&ngrp, nsel.p, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    WG_CK(cudaStreamSynchronize(st));
    WG_CK(cudaMemcpyAsync(grp_first.as<int64_t>() + ngrp, &nseg, sizeof(int64_t), cudaMemcpyHostToDevice, st));
  }
  // greedy pack: count, scan, write
  S.n_tasks = 0;
  if (ngrp > 0) {
    Tmp counts(st), offs(st);
    WG_TRY(counts.get(sizeof(int64_t) * ngrp));
    WG_TRY(offs.get(sizeof(int64_t) * (ngrp + 1)));
    WG_LAUNCH(k_pack, nblk(ngrp, 128), 128, 0, st, seg_off.as<int64_t>(), grp_first.as<int64_t>(), ngrp, keys,
              S.key, (int32_t)T, Rk, g->E_max, 0, counts.as<int64_t>(), (const int64_t*)nullptr, (wg_task*)nullptr);
    size_t tb = 0;
    WG_CK(cub::DeviceScan::ExclusiveSum(nullptr, tb, counts.as<int64_t>(), offs.as<int64_t>(), ngrp + 1, st));
    // ExclusiveSum over ngrp+1 reads counts[ngrp]: make it a valid zero
    Tmp counts2(st);
    WG_TRY(counts2.get(sizeof(int64_t) * (ngrp + 1)));
    WG_CK(cudaMemsetAsync(counts2.p, 0, sizeof(int64_t) * (ngrp + 1), st));
    WG_CK(cudaMemcpyAsync(counts2.p, counts.p, sizeof(int64_t) * ngrp, cudaMemcpyDeviceToDevice, st));
    WG_TRY(temp.get(tb));
    WG_CK(cub::DeviceScan::ExclusiveSum(temp.p, tb, counts2.as<int64_t>(), offs.as<int64_t>(), ngrp + 1, st));
    ++launch_counter();
    WG_CK(cudaMemcpyAsync(&S.n_tasks, offs.as<int64_t>() + ngrp, sizeof(int64_t), cudaMemcpyDeviceToHost, st));
    WG_CK(cudaStreamSynchronize(st));
    WG_TRY(dalloc(g, &S.tasks, S.n_tasks, st));
    WG_LAUNCH(k_pack, nblk(ngrp, 128), 128, 0, st, seg_off.as<int64_t>(), grp_first.as<int64_t>(), ngrp, keys,
              S.key, (int32_t)T, Rk, g->E_max, 1, (int64_t*)nullptr, offs.as<int64_t>(), S.tasks);
    // n_uniq_src: task id per position (max-scan of task starts), sort (task, idx), count distinct
    Tmp mark(st), taskof(st), uk(st), uk2(st), cnt(st);
    WG_TRY(mark.get(sizeof(int32_t) * n));
    WG_TRY(taskof.get(sizeof(int32_t) * n));
    WG_CK(cudaMemsetAsync(mark.p, 0, sizeof(int32_t) * n, st));
    WG_LAUNCH(k_task_starts, nblk(S.n_tasks), 256, 0, st, S.tasks, S.n_tasks, mark.as<int32_t>());
    tb = 0;
    WG_CK(cub::DeviceScan::InclusiveScan(nullptr, tb, mark.as<int32_t>(), taskof.as<int32_t>(), cub::Max(), n, st));
    WG_TRY(temp.get(tb));
    WG_CK(cub::DeviceScan::InclusiveScan(temp.p, tb, mark.as<int32_t>(), taskof.as<int32_t>(), cub::Max(), n, st));
    ++launch_counter();
    WG_TRY(uk.get(sizeof(uint64_t) * n));
    WG_TRY(uk2.get(sizeof(uint64_t) * n));
    WG_LAUNCH(k_uniq_keys, nblk(n), 256, 0, st, taskof.as<int32_t>(), S.idx, n, uk.as<uint64_t>());
    tb = 0;
    WG_CK(cub::DeviceRadixSort::SortKeys(nullptr, tb, uk.as<uint64_t>(), uk2.as<uint64_t>(), n, 0, 64, st));
    WG_TRY(temp.get(tb));
    WG_CK(cub::DeviceRadixSort::SortKeys(temp.p, tb, uk.as<uint64_t>(), uk2.as<uint64_t>(), n, 0, 64, st));
    ++launch_counter();
    WG_TRY(cnt.get(sizeof(int32_t) * S.n_tasks));
    WG_CK(cudaMemsetAsync(cnt.p, 0, sizeof(int32_t) * S.n_tasks, st));
    WG_LAUNCH(k_uniq_count, nblk(n), 256, 0, st, uk2.as<uint64_t>(), n, cnt.as<int32_t>());
    WG_LAUNCH(k_set_uniq, nblk(S.n_tasks), 256, 0, st, S.tasks, cnt.as<int32_t>(), S.n_tasks);
  } else {
    WG_TRY(dalloc(g, &S.tasks, 1, st));
  }
  S.h_tasks.resize(S.n_tasks);
  if (S.n_tasks) WG_CK(cudaMemcpyAsync(S.h_tasks.data(), S.tasks, S.n_tasks * sizeof(wg_task), cudaMemcpyDeviceToHost, st));
  // local CSR over key rows (untyped graphs: key order = vertex order)
  WG_TRY(dalloc(g, &S.row_ptr, S.n_rows + 1, st));
  WG_CK(cudaMemsetAsync(S.row_ptr, 0, sizeof(int64_t) * (S.n_rows + 1), st));
  if (!g->by_type && n > 0) {
    Tmp hist(st);
    WG_TRY(hist.get(sizeof(int64_t) * (S.n_rows + 1)));
    WG_CK(cudaMemsetAsync(hist.p, 0, sizeof(int64_t) * (S.n_rows + 1), st));
    WG_LAUNCH(k_row_hist, nblk(n), 256, 0, st, S.key, n, g->vb, hist.as<int64_t>());
    size_t tb = 0;
    WG_CK(cub::DeviceScan::InclusiveSum(nullptr, tb, hist.as<int64_t>(), S.row_ptr, S.n_rows + 1, st));
    WG_TRY(temp.get(tb));
    WG_CK(cub::DeviceScan::InclusiveSum(temp.p, tb, hist.as<int64_t>(), S.row_ptr, S.n_rows + 1, st));
    ++launch_counter();
  }
  S.h_row_ptr.resize(S.n_rows + 1);
  WG_CK(cudaMemcpyAsync(S.h_row_ptr.data(), S.row_ptr, sizeof(int64_t) * (S.n_rows + 1), cudaMemcpyDeviceToHost, st));
  WG_CK(cudaStreamSynchronize(st));
  return WG_OK;
}

bool is_device_ptr(const void* p) {
  if (!p) return false;
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) { cudaGetLastError(); return false; }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

template <typename T>
wg_status to_device(wg_graph_s* g, const T* p, int64_t n, cudaStream_t s, T** out, std::vector<void*>& tmp) {
  if (!p) { *out = nullptr; return WG_OK; }
  if (is_device_ptr(p)) { *out = const_cast<T*>(p); return WG_OK; }
  void* q = nullptr;
  WG_CK(cudaMallocAsync(&q, std::max<size_t>(sizeof(T) * n, 256), s));
  tmp.push_back(q);
  WG_CK(cudaMemcpyAsync(q, p, sizeof(T) * n, cudaMemcpyHostToDevice, s));
  *out = static_cast<T*>(q);
  return WG_OK;
}

}  // namespace

wg_status graph_create(const wg_graph_desc* d, int device, cudaStream_t st, wg_graph* out) {
  WG_REQ(d && out, WG_ERR_INVALID, "wg_graph_create: null argument");
  WG_REQ(d->num_vertices >= 1 && d->num_vertices < (1LL << 31), WG_ERR_INVALID, "num_vertices out of [1, 2^31)");
  WG_REQ(d->num_edges >= 0 && d->num_edges < (1LL << 31), WG_ERR_INVALID, "num_edges out of [0, 2^31)");
  WG_REQ(d->src != nullptr || d->num_edges == 0, WG_ERR_INVALID, "src is NULL");
  WG_REQ(d->indptr != nullptr || d->dst != nullptr || d->num_edges == 0, WG_ERR_INVALID, "dst and indptr are NULL");
  WG_REQ(d->num_types >= 1, WG_ERR_INVALID, "num_types < 1");
  WG_CK(cudaSetDevice(device));
  auto* g = new wg_graph_s();
  g->device = device;
  g->V = d->num_vertices;
  g->E_total = d->num_edges;
  g->T = d->tile_rows > 0 ? d->tile_rows : 128;
  g->R = d->num_types;
  g->by_type = (d->etype != nullptr && d->num_types > 1) ? 1 : 0;
  g->vb = d->v_begin;
  g->ve = (d->v_begin == 0 && d->v_end == 0) ? g->V : d->v_end;
  auto fail = [&](wg_status s) { wg_graph_destroy(g); return s; };
  if (!(g->vb >= 0 && g->vb < g->ve && g->ve <= g->V && g->vb % g->T == 0 && (g->ve % g->T == 0 || g->ve == g->V))) {
    set_error("v_begin/v_end must be T-aligned and within [0, V]");
    return fail(WG_ERR_INVALID);
  }
  if (d->max_task_edges > 0) {
    g->E_max = d->max_task_edges;
  } else {  // Q13: clamp(pow2ceil(4 T ceil(E/V)), 1024, 65536)
    int64_t avg = std::max<int64_t>(1, cdiv(g->E_total, g->V));
    int64_t x = 4 * (int64_t)g->T * avg, p = 1;
    while (p < x) p <<= 1;
    g->E_max = std::min<int64_t>(std::max<int64_t>(p, 1024), 65536);
  }
  const int64_t E = g->E_total;
  std::vector<void*> tmp;
  auto free_tmp = [&]() { for (void* q : tmp) cudaFreeAsync(q, st); tmp.clear(); };
  wg_status s = WG_OK;
  const int32_t *src = nullptr, *dst = nullptr, *et = nullptr;
  const int64_t* indptr = nullptr;
  if ((s = to_device(g, d->src, E, st, const_cast<int32_t**>(&src), tmp)) != WG_OK) { free_tmp(); return fail(s); }
  if (d->etype && (s = to_device(g, d->etype, E, st, const_cast<int32_t**>(&et), tmp)) != WG_OK) { free_tmp(); return fail(s); }
  if (d->indptr) {
    if ((s = to_device(g, d->indptr, g->V + 1, st, const_cast<int64_t**>(&indptr), tmp)) != WG_OK) { free_tmp(); return fail(s); }
    int32_t* dd = nullptr;
    if (cudaMallocAsync((void**)&dd, std::max<size_t>(4 * E, 256), st) != cudaSuccess) { free_tmp(); return fail(WG_ERR_NOMEM); }
    tmp.push_back(dd);
    k_coo_from_csr<<<nblk(g->V), 256, 0, st>>>(indptr, g->V, dd);
    ++launch_counter();
    dst = dd;
  } else if ((s = to_device(g, d->dst, E, st, const_cast<int32_t**>(&dst), tmp)) != WG_OK) {
    free_tmp(); return fail(s);
  }
  // validation
  {
    int32_t* bad = nullptr;
    cudaMallocAsync((void**)&bad, 256, st);
    tmp.push_back(bad);
    cudaMemsetAsync(bad, 0, 4, st);
    if (E > 0) { k_validate<<<nblk(E), 256, 0, st>>>(src, dst, g->by_type ? et : nullptr, E, g->V, g->R, bad); ++launch_counter(); }
    int32_t hb = 0;
    cudaMemcpyAsync(&hb, bad, 4, cudaMemcpyDeviceToHost, st);
    if (cudaStreamSynchronize(st) != cudaSuccess) { set_error("CUDA error during validation"); free_tmp(); return fail(WG_ERR_CUDA); }
    if (hb) { set_error("vertex id or edge type out of range"); free_tmp(); return fail(WG_ERR_RANGE); }
  }
  // degrees and normalisation scales (global)
  if ((s = dalloc(g, &g->deg_in, g->V, st)) || (s = dalloc(g, &g->deg_out, g->V, st)) ||
      (s = dalloc(g, &g->rs_in, g->V, st)) || (s = dalloc(g, &g->rs_out, g->V, st)) ||
      (s = dalloc(g, &g->inv_in, g->V, st))) { free_tmp(); return fail(s); }
  cudaMemsetAsync(g->deg_in, 0, 4 * g->V, st);
  cudaMemsetAsync(g->deg_out, 0, 4 * g->V, st);
  if (E > 0) { k_degrees<<<nblk(E), 256, 0, st>>>(src, dst, E, g->deg_in, g->deg_out); ++launch_counter(); }
  k_scales<<<nblk(g->V), 256, 0, st>>>(g->deg_in, g->deg_out, g->V, g->rs_in, g->rs_out, g->inv_in);
  ++launch_counter();
  {
    std::vector<int32_t> h(g->V);
    cudaMemcpyAsync(h.data(), g->deg_in, 4 * g->V, cudaMemcpyDeviceToHost, st);
    cudaStreamSynchronize(st);
    g->max_in_deg = *std::max_element(h.begin(), h.end());
  }
  if (g->by_type) {
    if ((s = dalloc(g, &g->etype_all, E, st)) != WG_OK) { free_tmp(); return fail(s); }
    cudaMemcpyAsync(g->etype_all, et, 4 * E, cudaMemcpyDeviceToDevice, st);
    if ((s = rel_counts(g, dst, et, st)) != WG_OK) { free_tmp(); return fail(s); }
  }
  if ((s = build_side(g, g->fwd, dst, src, et, st)) != WG_OK) { free_tmp(); return fail(s); }
  if ((s = build_side(g, g->bwd, src, dst, et, st)) != WG_OK) { free_tmp(); return fail(s); }
  if (g->vb == 0 && g->ve == g->V && E > 0) {
    int64_t* inv = nullptr;
    if (cudaMallocAsync((void**)&inv, 8 * E, st) != cudaSuccess) { free_tmp(); return fail(WG_ERR_NOMEM); }
    tmp.push_back(inv);
    if ((s = dalloc(g, &g->fwdpos, E, st)) != WG_OK) { free_tmp(); return fail(s); }
    k_inv_perm<<<nblk(E), 256, 0, st>>>(g->fwd.perm, E, inv);
    k_fwdpos<<<nblk(E), 256, 0, st>>>(g->bwd.perm, E, inv, g->fwdpos);
    launch_counter() += 2;
  }
  free_tmp();
  cudaError_t e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) { set_error(std::string("graph_create: ") + cudaGetErrorString(e)); return fail(WG_ERR_CUDA); }
  *out = g;
  return WG_OK;
}

}  // namespace wg

extern "C" {

wg_status wg_graph_create(const wg_graph_desc* desc, int device, wg_stream stream, wg_graph* out) {
  return wg::graph_create(desc, device, (cudaStream_t)stream, out);
}

wg_status wg_graph_info(wg_graph g, int64_t info[10]) {
  WG_REQ(g && info, WG_ERR_INVALID, "wg_graph_info: null argument");
  info[0] = g->V; info[1] = g->ve - g->vb; info[2] = g->fwd.E; info[3] = g->bwd.E;
  info[4] = g->fwd.n_tasks; info[5] = g->bwd.n_tasks; info[6] = g->T; info[7] = g->E_max;
  info[8] = g->by_type; info[9] = g->max_in_deg;
  return WG_OK;
}

wg_status wg_graph_export(wg_graph g, int transposed, int64_t* perm, wg_task* tasks, int64_t* fwdpos) {
  WG_REQ(g, WG_ERR_INVALID, "wg_graph_export: null graph");
  WG_CK(cudaSetDevice(g->device));
  const wg::Side& S = transposed ? g->bwd : g->fwd;
  if (perm && S.E) {
    std::vector<int32_t> p(S.E);
    WG_CK(cudaMemcpy(p.data(), S.perm, 4 * S.E, cudaMemcpyDeviceToHost));
    for (int64_t i = 0; i < S.E; ++i) perm[i] = p[i];
  }
  if (tasks && S.n_tasks) std::copy(S.h_tasks.begin(), S.h_tasks.end(), tasks);
  if (fwdpos && transposed) {
    WG_REQ(g->fwdpos != nullptr || S.E == 0, WG_ERR_STATE, "fwdpos needs a graph that owns all rows");
    if (S.E) WG_CK(cudaMemcpy(fwdpos, g->fwdpos, 8 * S.E, cudaMemcpyDeviceToHost));
  }
  return WG_OK;
}

wg_status wg_graph_destroy(wg_graph g) {
  if (!g) return WG_OK;
  WG_REQ(g->live_plans == 0, WG_ERR_STATE, "wg_graph_destroy: plans still alive");
  cudaSetDevice(g->device);
  cudaDeviceSynchronize();
  for (void* p : g->allocs) cudaFree(p);
  delete g;
  return WG_OK;
}

}  // extern "C"
