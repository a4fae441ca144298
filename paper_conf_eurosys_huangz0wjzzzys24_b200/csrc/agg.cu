// Gather + segment-reduce over gTask work items (SURVEY §8(a) a6 forward,
// a10 backward on the transposed partition) and the SPLIT-row combine (a8).
//
// Indexing ops of the paper: Index (h[src-id]) then Index-add (h[dst-id] +=)
// (Fig 2b); "indexing dominates" tensor-centric execution
// (P:L821-831).  One CTA executes one work item (the rows of one gTask, or one
// SPLIT chunk of an over-long row).  Inside a gTask the edges are sorted by
// destination, so the reduction is a warp-segmented scan over a flat edge
// range -- no global atomics:
//   * the item's edge range is cut into 8*G equal chunks, one per "worker"
//     (a group of LPE lanes; G = 32/LPE workers per warp), so every worker
//     streams the same number of rows of the table regardless of the degree
//     mix (overfill rows are shared by all workers);
//   * a worker keeps U row loads (16 B per lane) in flight across row
//     boundaries and flushes a destination row (epilogue + one 16-byte store
//     per lane) as soon as it is complete;
//   * a row cut by a chunk boundary leaves fp32 partials in shared memory; the
//     worker where the row starts sums them in worker order and stores it.
// Every reduction has a fixed order, so results are run-to-run deterministic.
//
//   out[r] = epi( rscale[r] * sum_{j in seg(r)} gscale[idx_j] * table[idx_j]
//                 + self_coef * self[r] )
//   epi(v) = mask( relu( v + bias ) )
#include <cooperative_groups.h>

#include "wg_internal.cuh"

namespace wg {

namespace {

constexpr int WARPS = 8;

template <typename T> struct VT;
template <> struct VT<float> {
  static constexpr int EPV = 4;
  __device__ static void add(float* acc, const int4& v, float s) {
    acc[0] += s * __int_as_float(v.x); acc[1] += s * __int_as_float(v.y);
    acc[2] += s * __int_as_float(v.z); acc[3] += s * __int_as_float(v.w);
  }
  __device__ static void unpack(const int4& v, float* f) {
    f[0] = __int_as_float(v.x); f[1] = __int_as_float(v.y); f[2] = __int_as_float(v.z); f[3] = __int_as_float(v.w);
  }
  __device__ static int4 pack(const float* f) {
    return make_int4(__float_as_int(f[0]), __float_as_int(f[1]), __float_as_int(f[2]), __float_as_int(f[3]));
  }
};
template <> struct VT<__nv_bfloat16> {
  static constexpr int EPV = 8;
  __device__ static void add(float* acc, const int4& v, float s) {
    const uint32_t w[4] = {(uint32_t)v.x, (uint32_t)v.y, (uint32_t)v.z, (uint32_t)v.w};
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      acc[2 * i] += s * __uint_as_float(w[i] << 16);
      acc[2 * i + 1] += s * __uint_as_float(w[i] & 0xffff0000u);
    }
  }
  __device__ static void unpack(const int4& v, float* f) {
    const uint32_t w[4] = {(uint32_t)v.x, (uint32_t)v.y, (uint32_t)v.z, (uint32_t)v.w};
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      f[2 * i] = __uint_as_float(w[i] << 16);
      f[2 * i + 1] = __uint_as_float(w[i] & 0xffff0000u);
    }
  }
  __device__ static int4 pack(const float* f) {
    uint32_t w[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      __nv_bfloat162 h = __floats2bfloat162_rn(f[2 * i], f[2 * i + 1]);  // RNE (Q23)
      w[i] = *reinterpret_cast<uint32_t*>(&h);
    }
    return make_int4((int)w[0], (int)w[1], (int)w[2], (int)w[3]);
  }
};

__device__ __forceinline__ int4 ldg16(const void* p) { return __ldg(reinterpret_cast<const int4*>(p)); }

// epilogue on one 16-byte output vector (EPV columns starting at column c0) of local row r
template <typename T>
__device__ __forceinline__ void epilogue_store(const float* acc_in, int r, int c0, float rs, const void* self_tab,
                                               int64_t ld_self, float self_coef, const float* bias, int relu,
                                               const void* mask_ref, int64_t ld_mask, void* out, int64_t ld_out,
                                               int F) {
  constexpr int EPV = VT<T>::EPV;
  float v[EPV];
#pragma unroll
  for (int i = 0; i < EPV; ++i) v[i] = rs * acc_in[i];
  if (self_tab) {
    float sf[EPV];
    VT<T>::unpack(ldg16(static_cast<const T*>(self_tab) + (int64_t)r * ld_self + c0), sf);
#pragma unroll
    for (int i = 0; i < EPV; ++i) v[i] += self_coef * sf[i];
  }
  if (bias) {
#pragma unroll
    for (int i = 0; i < EPV; ++i) v[i] += (c0 + i < F) ? bias[c0 + i] : 0.f;
  }
  if (relu) {
#pragma unroll
    for (int i = 0; i < EPV; ++i) v[i] = fmaxf(v[i], 0.f);
  }
  if (mask_ref) {
    float m[EPV];
    VT<T>::unpack(ldg16(static_cast<const T*>(mask_ref) + (int64_t)r * ld_mask + c0), m);
#pragma unroll
    for (int i = 0; i < EPV; ++i) v[i] = m[i] > 0.f ? v[i] : 0.f;
  }
#pragma unroll
  for (int i = 0; i < EPV; ++i) if (c0 + i >= F) v[i] = 0.f;
  *reinterpret_cast<int4*>(static_cast<T*>(out) + (int64_t)r * ld_out + c0) = VT<T>::pack(v);
}

// write a finished row: epilogue store, or (SPLIT chunk) raw fp32 partial
template <typename T>
__device__ __forceinline__ void finish_vec(const AggArgs& a, const float* acc, int r, int c0, int slot) {
  constexpr int EPV = VT<T>::EPV;
  if (slot >= 0) {
    float* pp = a.partial + (int64_t)slot * a.ld_part + c0;
#pragma unroll
    for (int i = 0; i < EPV; ++i) pp[i] = acc[i];
    return;
  }
  const float rs = a.rscale ? a.rscale[a.row_base + r] : 1.f;
  epilogue_store<T>(acc, r, c0, rs, a.self_tab, a.ld_self, a.self_coef, a.bias, a.relu, a.mask_ref, a.ld_mask, a.out,
                    a.ld_out, a.F);
}

// Rows of a regular item without in-edges get the epilogue of a zero sum
// (bias / self term), and the optional second output is zeroed.  The test is
// one thread per row (all rows' row_ptr loads in parallel, coalesced): a
// per-warp row loop put a dependent global load per row on the CTA's tail
// (4096-row RGCN stage items: ~500 serial loads per warp).
template <typename T>
__device__ __forceinline__ void empty_rows(const AggArgs& a, const WorkItem& it, int VPR) {
  constexpr int EPV = VT<T>::EPV;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int r0 = it.row_lo; r0 < it.row_hi; r0 += WARPS * 32) {
    const int r = r0 + (int)threadIdx.x;
    const bool empty = r < it.row_hi && a.row_ptr[r + 1] == a.row_ptr[r];
    unsigned m = __ballot_sync(0xffffffffu, empty);
    while (m) {
      const int rr = r0 + warp * 32 + __ffs(m) - 1;
      m &= m - 1;
      const float zero[EPV] = {};
      for (int vi = lane; vi < VPR; vi += 32) finish_vec<T>(a, zero, rr, vi * EPV, -1);
    }
  }
  if (a.zero_out) {
    for (int r = it.row_lo + warp; r < it.row_hi; r += WARPS) {
      T* p = static_cast<T*>(a.zero_out) + (int64_t)r * a.ld_zero;
      for (int c = lane * EPV; c < a.zero_cols; c += 32 * EPV) *reinterpret_cast<int4*>(p + c) = make_int4(0, 0, 0, 0);
    }
  }
}

// Warp-segmented gather-reduce.  Template: LPE lanes per edge row chunk, NV
// 16-byte vectors per lane (chunk width CW = LPE*NV vectors), U edges in flight.
template <typename T, int LPE, int NV, int U>
__global__ void __launch_bounds__(WARPS * 32, 3) k_agg(AggArgs a, int VPR) {
  constexpr int EPV = VT<T>::EPV;
  constexpr int G = 32 / LPE;
  constexpr int W = WARPS * G;                 // workers per CTA
  constexpr int CW = LPE * NV;                 // vectors per column chunk
  constexpr int SLOTF = CW * EPV;              // floats per partial slot
  extern __shared__ float part_smem[];         // [W][2][SLOTF]
  __shared__ int slot_row[W][2];               // local row of slot 0 (continuation) / slot 1 (owner), -1 none

  const WorkItem it = a.items[blockIdx.x];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int grp = lane / LPE, l = lane % LPE, worker = warp * G + grp;
  const unsigned gmask = LPE == 32 ? 0xffffffffu : (((1u << LPE) - 1u) << (grp * LPE));
  const bool split = it.split_slot >= 0;
  const int64_t eb = split ? it.e_lo : a.row_ptr[it.row_lo];
  const int64_t ee = split ? it.e_hi : a.row_ptr[it.row_hi];
  const int64_t len = ee - eb;
  const int64_t cb = eb + len * worker / W, ce = eb + len * (worker + 1) / W;
  const T* tab = static_cast<const T*>(a.table);
  const int64_t rb = a.row_base;
  const int* key = a.key;

  for (int cv0 = 0; cv0 < VPR; cv0 += CW) {
    const int nvec = min(CW, VPR - cv0);
    if (l == 0) { slot_row[worker][0] = -1; slot_row[worker][1] = -1; }
    if (cb < ce) {
      float acc[NV][EPV];
#pragma unroll
      for (int q = 0; q < NV; ++q)
#pragma unroll
        for (int i = 0; i < EPV; ++i) acc[q][i] = 0.f;
      int cur = split ? it.row_lo : (int)(key[cb] - rb);
      bool first = true;
      // first row starts before this chunk -> its partial is a continuation
      const bool first_cont = split ? (cb > eb) : (a.row_ptr[cur] < cb);
      int64_t pos = cb;
      int my_idx = 0, my_key = 0;
      float my_sc = 1.f;
      if (pos + l < ce) {
        my_idx = a.idx[pos + l];
        my_key = split ? it.row_lo : (int)(key[pos + l] - rb);
        if (a.gscale) my_sc = a.gscale[my_idx];
        else if (a.escale) my_sc = a.escale[pos + l];
      }
      auto flush = [&](int row, bool as_cont, bool as_owner) {
        // as_cont: continuation partial (slot 0); as_owner: owner partial (slot 1); else final
        if (as_cont || as_owner) {
          const int s = as_cont ? 0 : 1;
          float* sp = part_smem + ((size_t)worker * 2 + s) * SLOTF;
#pragma unroll
          for (int q = 0; q < NV; ++q)
#pragma unroll
            for (int i = 0; i < EPV; ++i) sp[(l + q * LPE) * EPV + i] = acc[q][i];
          if (l == 0) slot_row[worker][s] = row;
        } else {
#pragma unroll
          for (int q = 0; q < NV; ++q) {
            const int vi = l + q * LPE;
            if (vi < nvec) finish_vec<T>(a, acc[q], row, (cv0 + vi) * EPV, split ? it.split_slot : -1);
          }
        }
      };
      while (pos < ce) {
        const int n = (int)min((int64_t)LPE, ce - pos);
        // prefetch the next round of indices
        int nx_idx = 0, nx_key = 0;
        float nx_sc = 1.f;
        const int64_t np = pos + LPE + l;
        if (np < ce) {
          nx_idx = a.idx[np];
          nx_key = split ? it.row_lo : (int)(key[np] - rb);
          if (a.gscale) nx_sc = a.gscale[nx_idx];
          else if (a.escale) nx_sc = a.escale[np];
        }
        for (int j = 0; j < n; j += U) {
          int4 v[U][NV];
          float sc[U];
          int rk[U];
#pragma unroll
          for (int u = 0; u < U; ++u) {
            const int k = j + u;
            const bool ok = k < n;
            const int s = __shfl_sync(gmask, my_idx, ok ? k : 0, LPE);
            sc[u] = __shfl_sync(gmask, my_sc, ok ? k : 0, LPE);
            rk[u] = __shfl_sync(gmask, my_key, ok ? k : 0, LPE);
            if (!ok) rk[u] = -1;
            const T* row = tab + (int64_t)s * a.ld_tab + (int64_t)cv0 * EPV;
#pragma unroll
            for (int q = 0; q < NV; ++q) {
              const int vi = l + q * LPE;
              v[u][q] = (ok && vi < nvec) ? ldg16(row + vi * EPV) : make_int4(0, 0, 0, 0);
            }
          }
#pragma unroll
          for (int u = 0; u < U; ++u) {
            if (rk[u] < 0) break;
            if (rk[u] != cur) {
              flush(cur, first && first_cont, false);
              first = false;
              cur = rk[u];
#pragma unroll
              for (int q = 0; q < NV; ++q)
#pragma unroll
                for (int i = 0; i < EPV; ++i) acc[q][i] = 0.f;
            }
#pragma unroll
            for (int q = 0; q < NV; ++q) VT<T>::add(acc[q], v[u][q], sc[u]);
          }
        }
        my_idx = nx_idx;
        my_key = nx_key;
        my_sc = nx_sc;
        pos += LPE;
      }
      // last row of the chunk: does it continue past the chunk end?
      const bool last_open = split ? (ce < ee) : (a.row_ptr[cur + 1] > ce);
      if (first && first_cont) flush(cur, true, false);       // whole chunk inside one cut row
      else flush(cur, false, last_open);
    }
    __syncthreads();
    // owners merge the continuation partials of the following workers, in order
    if (cb < ce && slot_row[worker][1] >= 0) {
      const int r = slot_row[worker][1];
      for (int q = 0; q < NV; ++q) {
        const int vi = l + q * LPE;
        if (vi >= nvec) continue;
        float s[EPV];
        const float* sp = part_smem + ((size_t)worker * 2 + 1) * SLOTF + vi * EPV;
#pragma unroll
        for (int i = 0; i < EPV; ++i) s[i] = sp[i];
        for (int w2 = worker + 1; w2 < W; ++w2) {
          if (len * w2 / W == len * (w2 + 1) / W) continue;   // empty chunk (items shorter than W edges)
          if (slot_row[w2][0] != r) break;
          const float* sq = part_smem + ((size_t)w2 * 2 + 0) * SLOTF + vi * EPV;
#pragma unroll
          for (int i = 0; i < EPV; ++i) s[i] += sq[i];
        }
        finish_vec<T>(a, s, r, (cv0 + vi) * EPV, split ? it.split_slot : -1);
      }
    }
    __syncthreads();
  }
  if (split) return;
  empty_rows<T>(a, it, VPR);
}

// ---------------------------------------------------------------------------
// k_agg_cp: the same warp-segmented reduction, with the gathered rows staged
// through a per-lane shared-memory ring filled by cp.async (LDGSTS): lane l of
// a worker copies and later reads only its own 16-byte slices, so no barrier
// is needed between copy and use, and no register is held per in-flight row.
// D = NR*RS edges per worker are in flight (NR rounds of RS edges); per SM
// that is 2 CTAs x 256 lanes x D x 16 B ~ 190 KB, enough to cover HBM latency
// at full bandwidth (Little's law: 6.5 TB/s x ~2 us / 148 SMs ~ 90 KB).
// Edge metadata (destination row, source scale) rides in a per-worker ring.
// Gathered rows: random accesses, whose DRAM cost is set by the L2 fill
// granularity -- measured (scripts/gran_probe.cu, profiles/r02/gran_probe.md):
// a random 32-128 B row fetches a whole 128-byte line by default; with the
// .L2::64B prefetch-size hint only the 64-byte halves it touches (a 64-B row
// 64 B instead of 128, a 96-B row 128 instead of 192 on average).  Random
// row accesses are capped near 35 G/s either way (DRAM activations), so the
// hint cuts bytes, not accesses.
__device__ __forceinline__ void cp_async16(void* smem, const void* gmem, bool pred) {
  const uint32_t s = static_cast<uint32_t>(__cvta_generic_to_shared(smem));
  const int n = pred ? 16 : 0;
  asm volatile("cp.async.cg.shared.global.L2::64B [%0], [%1], 16, %2;" ::"r"(s), "l"(gmem), "r"(n) : "memory");
}
__device__ __forceinline__ void cp_async4(void* smem, const void* gmem, bool pred) {
  const uint32_t s = static_cast<uint32_t>(__cvta_generic_to_shared(smem));
  const int n = pred ? 4 : 0;
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(s), "l"(gmem), "r"(n) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

template <typename T, int LPE, int NV, int RS, int NR, int MINB = 2>
__global__ void __launch_bounds__(WARPS * 32, MINB) k_agg_cp(AggArgs a, int VPR) {
  constexpr int EPV = VT<T>::EPV;
  constexpr int G = 32 / LPE;
  constexpr int W = WARPS * G;
  constexpr int CW = LPE * NV;
  constexpr int SLOTF = CW * EPV;
  constexpr int D = NR * RS;                   // ring depth (edges) per worker
  static_assert(RS <= LPE, "a round is issued by RS lanes of the worker");
  extern __shared__ __align__(16) uint8_t smem_cp[];
  int4* ring = reinterpret_cast<int4*>(smem_cp);                                   // [D][NV][256]
  float* part_smem = reinterpret_cast<float*>(ring + (size_t)D * NV * WARPS * 32);  // [W][2][SLOTF]
  int* key_ring = reinterpret_cast<int*>(part_smem + (size_t)W * 2 * SLOTF);       // [W][D]
  float* sc_ring = reinterpret_cast<float*>(key_ring + W * D);                      // [W][D]
  int* idx_ring = reinterpret_cast<int*>(sc_ring + W * D);                          // [NR+1][256]
  __shared__ int slot_row[W][2];

  const WorkItem it = a.items[blockIdx.x];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int grp = lane / LPE, l = lane % LPE, worker = warp * G + grp;
  const unsigned gmask = LPE == 32 ? 0xffffffffu : (((1u << LPE) - 1u) << (grp * LPE));
  const bool split = it.split_slot >= 0;
  const int64_t eb = split ? it.e_lo : a.row_ptr[it.row_lo];
  const int64_t ee = split ? it.e_hi : a.row_ptr[it.row_hi];
  const int64_t len = ee - eb;
  const int64_t cb = eb + len * worker / W, ce = eb + len * (worker + 1) / W;
  const T* tab = static_cast<const T*>(a.table);
  const int64_t rb = a.row_base;
  int* kr = key_ring + worker * D;
  float* sr = sc_ring + worker * D;

  // Every worker of the CTA runs the same number of rounds (chunk lengths
  // differ by at most one edge): control flow is warp-uniform, so all warp
  // primitives use the full mask, and ring slots advance by wrap-around
  // counters (no divisions in the loop).
  const int64_t maxlen = (len + W - 1) / W;
  const int nrounds = (int)((maxlen + RS - 1) / RS);
  const int irb = (int)rb;
  const int lbase = grp * LPE;
  constexpr int TPB = WARPS * 32;
  constexpr int RSTRIDE = NV * TPB;            // int4 per ring slot (one edge)
  int4* my_ring = ring + threadIdx.x;
  int* my_iring = idx_ring + threadIdx.x;
  const bool scaled = a.gscale || a.escale;
  (void)gmask;

  for (int cv0 = 0; cv0 < VPR; cv0 += CW) {
    const int nvec = min(CW, VPR - cv0);
    if (l == 0) { slot_row[worker][0] = -1; slot_row[worker][1] = -1; }
    if (nrounds > 0) {
      // Source ids ride the same cp.async pipeline NR rounds ahead of the row
      // copies (per-lane ring of NR+1 rounds; rounds are RS-aligned from cb).
      auto iload = [&](int round, int islot) {
        const int64_t e = cb + (int64_t)round * RS + l;
        const bool ok = l < RS && e < ce;
        cp_async4(my_iring + islot * TPB, a.idx + (ok ? e : eb), ok);
      };
#pragma unroll 1
      for (int r = 0; r < NR; ++r) iload(r, r);
      cp_async_commit();
      cp_async_wait<0>();
      int islot_w = NR, islot_r = 0, pslot = 0, issued = 0;
      int64_t prod = cb;
      auto issue = [&]() {
        const int n = (int)max((int64_t)0, min((int64_t)RS, ce - prod));
        const int pidx = my_iring[islot_r * TPB];
#pragma unroll
        for (int u = 0; u < RS; ++u) {
          const int s = __shfl_sync(0xffffffffu, pidx, lbase + u);
          const T* row = tab + (int64_t)s * a.ld_tab + (int64_t)cv0 * EPV;
#pragma unroll
          for (int q = 0; q < NV; ++q) {
            const int vi = l + q * LPE;
            // lanes past the row's last vector point at its first one (no extra 64-B block)
            cp_async16(my_ring + (pslot + u) * RSTRIDE + q * TPB, row + (vi < nvec ? vi : 0) * EPV, u < n && vi < nvec);
          }
        }
        if (l < RS) {
          const bool ok = l < n;
          if (split) { if (ok) kr[pslot + l] = (int)(it.row_lo + rb); }
          else cp_async4(kr + pslot + l, a.key + (ok ? prod + l : eb), ok);
          if (a.gscale) cp_async4(sr + pslot + l, a.gscale + pidx, ok);
          else if (a.escale) cp_async4(sr + pslot + l, a.escale + (ok ? prod + l : eb), ok);
        }
        iload(issued + NR, islot_w);
        cp_async_commit();
        islot_w = islot_w == NR ? 0 : islot_w + 1;
        islot_r = islot_r == NR ? 0 : islot_r + 1;
        pslot = pslot + RS == D ? 0 : pslot + RS;
        prod += RS;
        ++issued;
      };
#pragma unroll 1
      for (int r = 0; r < NR; ++r) issue();
      float acc[NV][EPV];
#pragma unroll
      for (int q = 0; q < NV; ++q)
#pragma unroll
        for (int i = 0; i < EPV; ++i) acc[q][i] = 0.f;
      int cur = cb < ce ? (split ? it.row_lo : (int)(a.key[cb] - rb)) : -1;
      bool first = true;
      const bool first_cont = cb < ce && (split ? (cb > eb) : (a.row_ptr[cur] < cb));
      auto flush = [&](int row, bool as_cont, bool as_owner) {
        if (as_cont || as_owner) {
          const int s = as_cont ? 0 : 1;
          float* sp = part_smem + ((size_t)worker * 2 + s) * SLOTF;
#pragma unroll
          for (int q = 0; q < NV; ++q)
#pragma unroll
            for (int i = 0; i < EPV; ++i) sp[(l + q * LPE) * EPV + i] = acc[q][i];
          if (l == 0) slot_row[worker][s] = row;
        } else {
#pragma unroll
          for (int q = 0; q < NV; ++q) {
            const int vi = l + q * LPE;
            if (vi < nvec) finish_vec<T>(a, acc[q], row, (cv0 + vi) * EPV, split ? it.split_slot : -1);
          }
        }
      };
      int cslot = 0;
#pragma unroll 1
      for (int r = 0; r < nrounds; ++r) {
        cp_async_wait<NR - 1>();
        __syncwarp();
        const int n = (int)max((int64_t)0, min((int64_t)RS, ce - (cb + (int64_t)r * RS)));
        // fast path: a full round inside the current row (edges are sorted by
        // row, so first == last == cur implies all) -> branch-free accumulate
        if (n == RS && (split || (kr[cslot] - irb == cur && kr[cslot + RS - 1] - irb == cur))) {
#pragma unroll
          for (int u = 0; u < RS; ++u) {
            const float sc = scaled ? sr[cslot + u] : 1.f;
#pragma unroll
            for (int q = 0; q < NV; ++q) VT<T>::add(acc[q], my_ring[(cslot + u) * RSTRIDE + q * TPB], sc);
          }
        } else {
#pragma unroll
        for (int u = 0; u < RS; ++u) {
          if (u < n) {
            const int rk = split ? it.row_lo : kr[cslot + u] - irb;
            const float sc = scaled ? sr[cslot + u] : 1.f;
            if (rk != cur) {
              flush(cur, first && first_cont, false);
              first = false;
              cur = rk;
#pragma unroll
              for (int q = 0; q < NV; ++q)
#pragma unroll
                for (int i = 0; i < EPV; ++i) acc[q][i] = 0.f;
            }
#pragma unroll
            for (int q = 0; q < NV; ++q) VT<T>::add(acc[q], my_ring[(cslot + u) * RSTRIDE + q * TPB], sc);
          }
        }
        }
        cslot = cslot + RS == D ? 0 : cslot + RS;
        __syncwarp();
        issue();
      }
      cp_async_wait<0>();
      if (cb < ce) {
        const bool last_open = split ? (ce < ee) : (a.row_ptr[cur + 1] > ce);
        if (first && first_cont) flush(cur, true, false);
        else flush(cur, false, last_open);
      }
    }
    __syncthreads();
    if (cb < ce && slot_row[worker][1] >= 0) {
      const int r = slot_row[worker][1];
      for (int q = 0; q < NV; ++q) {
        const int vi = l + q * LPE;
        if (vi >= nvec) continue;
        float s[EPV];
        const float* sp = part_smem + ((size_t)worker * 2 + 1) * SLOTF + vi * EPV;
#pragma unroll
        for (int i = 0; i < EPV; ++i) s[i] = sp[i];
        for (int w2 = worker + 1; w2 < W; ++w2) {
          if (len * w2 / W == len * (w2 + 1) / W) continue;
          if (slot_row[w2][0] != r) break;
          const float* sq = part_smem + ((size_t)w2 * 2 + 0) * SLOTF + vi * EPV;
#pragma unroll
          for (int i = 0; i < EPV; ++i) s[i] += sq[i];
        }
        finish_vec<T>(a, s, r, (cv0 + vi) * EPV, split ? it.split_slot : -1);
      }
    }
    __syncthreads();
  }
  if (split) return;
  empty_rows<T>(a, it, VPR);
}

template <typename T>
__global__ void k_combine(CombineArgs a, int VPR) {
  constexpr int EPV = VT<T>::EPV;
  const SplitRow sr = a.rows[blockIdx.x];
  if (a.plan_filter >= 0 && sr.plan != a.plan_filter) return;
  const float rs = a.rscale ? a.rscale[a.row_base + sr.row] : 1.f;
  for (int vi = threadIdx.x; vi < VPR; vi += blockDim.x) {
    const int c0 = vi * EPV;
    float s[EPV];
#pragma unroll
    for (int i = 0; i < EPV; ++i) s[i] = 0.f;
    for (int k = 0; k < sr.n_slots; ++k) {
      const float* pp = a.partial + (int64_t)(sr.first_slot + k) * a.ld_part + c0;
#pragma unroll
      for (int i = 0; i < EPV; ++i) s[i] += pp[i];
    }
    epilogue_store<T>(s, sr.row, c0, rs, a.self_tab, a.ld_self, a.self_coef, a.bias, a.relu, a.mask_ref, a.ld_mask,
                      a.out, a.ld_out, a.F);
  }
  if (a.zero_out) {
    T* p = static_cast<T*>(a.zero_out) + (int64_t)sr.row * a.ld_zero;
    for (int c = threadIdx.x * EPV; c < a.zero_cols; c += blockDim.x * EPV)
      *reinterpret_cast<int4*>(p + c) = make_int4(0, 0, 0, 0);
  }
}

// ---------------------------------------------------------------------------
// Overfill gTasks ("a separate GPU kernel that
// increases thread blocks and shared memory size", run with higher
// priority): every destination row longer than E_max (its SPLIT chunks) is
// reduced by one thread-block CLUSTER of HC CTAs.  Each CTA sums an equal
// share of the row's edges (8 warps, fixed order) into shared memory; after a
// cluster barrier the leader CTA adds the HC partial rows through distributed
// shared memory in rank order and applies the epilogue -- no global fp32
// scratch, no combine launch, deterministic.
constexpr int HC = 16;                     // CTAs per heavy row (non-portable cluster size, opted in)
template <typename T>
__global__ void __launch_bounds__(WARPS * 32) k_agg_heavy(AggArgs a, const SplitRow* rows, int VPR) {
  namespace cg = cooperative_groups;
  cg::cluster_group cl = cg::this_cluster();
  constexpr int EPV = VT<T>::EPV;
  extern __shared__ __align__(16) float hsm[];            // [WARPS][VPR*EPV] then [VPR*EPV] (CTA total)
  const int rank = (int)cl.block_rank();
  const SplitRow sr = rows[blockIdx.x / HC];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int Fp = VPR * EPV;
  float* cta = hsm + WARPS * Fp;
  const int64_t eb = a.row_ptr[sr.row], ee = a.row_ptr[sr.row + 1], len = ee - eb;
  // this CTA's share, then this warp's share of it (fixed partition of the row)
  const int64_t cb = eb + len * rank / HC, ce = eb + len * (rank + 1) / HC;
  const int64_t wb = cb + (ce - cb) * warp / WARPS, we = cb + (ce - cb) * (warp + 1) / WARPS;
  const T* tab = static_cast<const T*>(a.table);
  for (int v0 = 0; v0 < VPR; v0 += 32) {
    const int vi = v0 + lane;
    float acc[EPV];
#pragma unroll
    for (int i = 0; i < EPV; ++i) acc[i] = 0.f;
    int64_t e = wb;
    constexpr int UH = 8;                                  // rows in flight per lane
    for (; e + UH <= we; e += UH) {
      int4 v[UH];
      float sc[UH];
      int sidx[UH];
#pragma unroll
      for (int u = 0; u < UH; ++u) sidx[u] = a.idx[e + u];
#pragma unroll
      for (int u = 0; u < UH; ++u) {
        const int s = sidx[u];
        sc[u] = a.gscale ? a.gscale[s] : (a.escale ? a.escale[e + u] : 1.f);
        v[u] = vi < VPR ? ldg16(tab + (int64_t)s * a.ld_tab + vi * EPV) : make_int4(0, 0, 0, 0);
      }
#pragma unroll
      for (int u = 0; u < UH; ++u) VT<T>::add(acc, v[u], sc[u]);
    }
    for (; e < we; ++e) {
      const int s = a.idx[e];
      const float sc = a.gscale ? a.gscale[s] : (a.escale ? a.escale[e] : 1.f);
      if (vi < VPR) VT<T>::add(acc, ldg16(tab + (int64_t)s * a.ld_tab + vi * EPV), sc);
    }
    if (vi < VPR) {
#pragma unroll
      for (int i = 0; i < EPV; ++i) hsm[warp * Fp + vi * EPV + i] = acc[i];
    }
  }
  __syncwarp();                                            // reconverge before the block barrier
  __syncthreads();
  for (int c = threadIdx.x; c < Fp; c += blockDim.x) {     // CTA partial: warps in order
    float t = 0.f;
    for (int w = 0; w < WARPS; ++w) t += hsm[w * Fp + c];
    cta[c] = t;
  }
  __syncwarp();
  cl.sync();                                               // every CTA's partial is visible cluster-wide
  if (rank == 0) {
    for (int vi = threadIdx.x; vi < VPR; vi += blockDim.x) {
      float t[EPV];
#pragma unroll
      for (int i = 0; i < EPV; ++i) t[i] = 0.f;
      for (int r = 0; r < HC; ++r) {                       // ranks in order (deterministic)
        const float* peer = cl.map_shared_rank(cta, r);
#pragma unroll
        for (int i = 0; i < EPV; ++i) t[i] += peer[vi * EPV + i];
      }
      const float rs = a.rscale ? a.rscale[a.row_base + sr.row] : 1.f;
      epilogue_store<T>(t, sr.row, vi * EPV, rs, a.self_tab, a.ld_self, a.self_coef, a.bias, a.relu, a.mask_ref,
                        a.ld_mask, a.out, a.ld_out, a.F);
    }
    if (a.zero_out) {
      T* p = static_cast<T*>(a.zero_out) + (int64_t)sr.row * a.ld_zero;
      for (int c = threadIdx.x * EPV; c < a.zero_cols; c += blockDim.x * EPV)
        *reinterpret_cast<int4*>(p + c) = make_int4(0, 0, 0, 0);
    }
  }
  __syncwarp();
  cl.sync();                                               // peers keep their smem until the leader has read it
}

template <typename T, int LPE, int NV, int U>
wg_status launch_cfg(const AggArgs& a, int VPR, cudaStream_t s) {
  constexpr int EPV = VT<T>::EPV;
  const size_t smem = (size_t)WARPS * (32 / LPE) * 2 * LPE * NV * EPV * sizeof(float);
  if (smem > 48 * 1024) {
    static bool done = false;
    if (!done) {
      cudaFuncSetAttribute(k_agg<T, LPE, NV, U>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      done = true;
    }
  }
  WG_LAUNCH((k_agg<T, LPE, NV, U>), a.n_items, WARPS * 32, smem, s, a, VPR);
  return WG_OK;
}

template <typename T, int LPE, int NV, int RS, int NR, int MINB = 2>
wg_status launch_cp(const AggArgs& a, int VPR, cudaStream_t s) {
  constexpr int EPV = VT<T>::EPV;
  constexpr int W = WARPS * (32 / LPE), D = NR * RS;
  const size_t smem = (size_t)D * NV * WARPS * 32 * 16 + (size_t)W * 2 * LPE * NV * EPV * sizeof(float) +
                      (size_t)W * D * 8 + (size_t)(NR + 1) * WARPS * 32 * 4;
  static bool done = false;
  if (!done) {
    cudaFuncSetAttribute(k_agg_cp<T, LPE, NV, RS, NR, MINB>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    done = true;
  }
  WG_LAUNCH((k_agg_cp<T, LPE, NV, RS, NR, MINB>), a.n_items, WARPS * 32, smem, s, a, VPR);
  return WG_OK;
}

bool use_v2() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("WG_AGG_V2");
    v = (e && e[0] == '1') ? 1 : 0;
  }
  return v == 1;
}

template <typename T>
wg_status launch_t(const AggArgs& a, cudaStream_t s) {
  constexpr int EPV = VT<T>::EPV;
  const int VPR = (int)cdiv(a.F, EPV);
  if (VPR <= 1) return launch_cfg<T, 1, 1, 1>(a, VPR, s);
  if (VPR <= 2) return launch_cfg<T, 2, 1, 2>(a, VPR, s);
  static int cfg = -1, narrow = -1;
  if (cfg < 0) {
    const char* e = getenv("WG_AGG_CFG");
    cfg = e ? atoi(e) : 0;
    const char* n = getenv("WG_AGG_NARROW");
    narrow = n ? atoi(n) : 0;
  }
  if (VPR <= 4) {
    // 33-64-byte rows (C5's 32-wide bf16 layers): the staged ring at 4 CTAs /
    // SM (A/B on the C5 rank slice, 6 gathers / epoch: register kernel
    // 63.0 ms, ring 4x3 @ 3/SM 53.6, 4x2 @ 4/SM 51.6, 4x4 @ 2/SM 54.5 ms)
    if (narrow == 1) return launch_cfg<T, 4, 1, 4>(a, VPR, s);
    return launch_cp<T, 4, 1, 4, 2, 4>(a, VPR, s);
  }
  if (!use_v2() && cfg == 1) {   // 3 CTAs / SM, ring 5 x 2
    if (VPR <= 8) return launch_cp<T, 8, 1, 5, 2, 3>(a, VPR, s);
    if (VPR <= 16) return launch_cp<T, 16, 1, 5, 2, 3>(a, VPR, s);
    if (VPR <= 32) return launch_cp<T, 32, 1, 5, 2, 3>(a, VPR, s);
  } else if (!use_v2() && cfg == 2) {   // 4 CTAs / SM, ring 4 x 2
    if (VPR <= 8) return launch_cp<T, 8, 1, 4, 2, 4>(a, VPR, s);
    if (VPR <= 16) return launch_cp<T, 16, 1, 4, 2, 4>(a, VPR, s);
    if (VPR <= 32) return launch_cp<T, 32, 1, 4, 2, 4>(a, VPR, s);
  } else if (!use_v2()) {
    // default: 3 CTAs (24 warps) per SM, 10 edges in flight per worker
    // (65-128-byte rows, C4 epoch A/B: 5x2 @ 3/SM 24.0 ms; 8x2 @ 3 25.2, 5x3 @ 3 24.9,
    //  4x2 @ 4 24.4, 8x3 @ 2 27.3, 6x3 @ 3 24.8 ms)
    // (A/B on C4: 7x3 @ 2 CTAs/SM 72 %, 6x2 @ 3/SM 83 %, 5x2 @ 3/SM 84.5 %,
    //  4x2 @ 4/SM 82 % of HBM)
    if (VPR <= 8) return launch_cp<T, 8, 1, 5, 2, 3>(a, VPR, s);
    if (VPR <= 16) return launch_cp<T, 16, 1, 5, 2, 3>(a, VPR, s);
    if (VPR <= 32) return launch_cp<T, 32, 1, 5, 2, 3>(a, VPR, s);
  } else {
    if (VPR <= 8) return launch_cfg<T, 8, 1, 4>(a, VPR, s);
    if (VPR <= 16) return launch_cfg<T, 16, 1, 4>(a, VPR, s);
    if (VPR <= 32) return launch_cfg<T, 32, 1, 4>(a, VPR, s);
  }
  if (VPR <= 64) return launch_cfg<T, 32, 2, 2>(a, VPR, s);
  return launch_cfg<T, 32, 4, 1>(a, VPR, s);
}

}  // namespace

wg_status launch_agg(wg_dtype dt, const AggArgs& a, cudaStream_t s) {
  if (a.n_items == 0) return WG_OK;
  WG_REQ(a.key != nullptr || a.idx == nullptr, WG_ERR_STATE, "launch_agg: key array missing");  // E = 0: no key / idx
  // algorithmic bytes: per edge the index (4 B), the gathered row (F elements)
  // and the source scale if any; per row the output, row_ptr and optional
  // self / mask rows
  const double es = dt == WG_BF16 ? 2.0 : 4.0, rb = a.F * es;
  const double bytes = a.n_edges * (4.0 + rb + (a.gscale || a.escale ? 4.0 : 0.0)) +
                       a.n_rows * (rb + 8.0 + (a.self_tab ? rb : 0.0) + (a.mask_ref ? rb : 0.0) +
                                   (a.zero_out ? a.zero_cols * es : 0.0));
  ProfScope ps(PK_AGG, s, bytes, 2.0 * a.n_edges * a.F);
  return dt == WG_BF16 ? launch_t<__nv_bfloat16>(a, s) : launch_t<float>(a, s);
}

wg_status launch_combine(wg_dtype dt, const CombineArgs& a, cudaStream_t s) {
  if (a.n_rows == 0) return WG_OK;
  const int EPV = dt == WG_BF16 ? 8 : 4;
  const int VPR = (int)cdiv(a.F, EPV);
  ProfScope ps(PK_COMBINE, s, (double)a.n_rows * a.F * (EPV == 8 ? 2 : 4), 0.0);
  if (dt == WG_BF16) WG_LAUNCH(k_combine<__nv_bfloat16>, a.n_rows, 128, 0, s, a, VPR);
  else WG_LAUNCH(k_combine<float>, a.n_rows, 128, 0, s, a, VPR);
  return WG_OK;
}

// Differentiated outlier scheduling: the regular work items
// and the overfill rows (deg > E_max) run as two kernels -- the cluster
// kernel on a high-priority side stream ("increasing the priority of
// execution for overfill gTasks"), the regular gather on the caller's
// stream -- joined by events (CUDA-graph capturable).  `n_split_items`
// leading items of `a` are the SPLIT chunks the partial path would run.
// WG_HEAVY=0 selects the partial path (SPLIT items + k_combine).
namespace {
struct HeavyStreams {
  int device = -1;
  cudaStream_t hs = nullptr;
  cudaEvent_t fork = nullptr, join = nullptr;
};
HeavyStreams& heavy_streams() {
  static thread_local HeavyStreams h;
  int dev = 0;
  cudaGetDevice(&dev);
  if (h.device != dev) {
    int lo = 0, hi = 0;
    cudaDeviceGetStreamPriorityRange(&lo, &hi);
    cudaStreamCreateWithPriority(&h.hs, cudaStreamNonBlocking, hi);
    cudaEventCreateWithFlags(&h.fork, cudaEventDisableTiming);
    cudaEventCreateWithFlags(&h.join, cudaEventDisableTiming);
    h.device = dev;
  }
  return h;
}
bool heavy_enabled() {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("WG_HEAVY");
    v = (e && e[0] == '0') ? 0 : 1;
  }
  return v == 1;
}
template <typename T>
wg_status launch_heavy_t(const AggArgs& a, const SplitRow* rows, int n_rows, cudaStream_t s) {
  constexpr int EPV = VT<T>::EPV;
  const int VPR = (int)cdiv(a.F, EPV);
  const size_t smem = sizeof(float) * (size_t)(WARPS + 1) * VPR * EPV;
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(k_agg_heavy<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    cudaFuncSetAttribute(k_agg_heavy<T>, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    attr = true;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(n_rows * HC));
  cfg.blockDim = dim3(WARPS * 32);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = HC; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  cudaError_t e = cudaLaunchKernelEx(&cfg, k_agg_heavy<T>, a, rows, VPR);
  ++launch_counter();
  if (e != cudaSuccess) {
    set_error(std::string("launch k_agg_heavy: ") + cudaGetErrorString(e));
    return WG_ERR_CUDA;
  }
  return WG_OK;
}
}  // namespace

wg_status launch_agg_outliers(wg_dtype dt, const AggArgs& a, int n_split_items, const SplitRow* split_rows,
                              int n_split_rows, const CombineArgs& comb, cudaStream_t s) {
  // the cluster kernel pays off for a few very long rows (it overlaps the
  // regular items); many moderately long rows run better as SPLIT items
  // spread over all SMs (profiles/r02/outlier_breakdown.md: C4 with E_max =
  // 512, 1497 heavy rows, partials 10.96 ms vs clusters 11.90 ms)
  if (!heavy_enabled() || n_split_rows == 0 || n_split_rows > 64 || a.F > 64 * (dt == WG_BF16 ? 8 : 4)) {
    WG_TRY(launch_agg(dt, a, s));
    return launch_combine(dt, comb, s);
  }
  HeavyStreams& h = heavy_streams();
  WG_CK(cudaEventRecord(h.fork, s));
  WG_CK(cudaStreamWaitEvent(h.hs, h.fork, 0));
  {
    int64_t he = 0;
    ProfScope ps(PK_COMBINE, h.hs, 0.0, 0.0);
    WG_TRY(dt == WG_BF16 ? launch_heavy_t<__nv_bfloat16>(a, split_rows, n_split_rows, h.hs)
                         : launch_heavy_t<float>(a, split_rows, n_split_rows, h.hs));
    (void)he;
  }
  AggArgs r = a;
  r.items = a.items + n_split_items;
  r.n_items = a.n_items - n_split_items;
  if (r.n_items > 0) WG_TRY(launch_agg(dt, r, s));
  WG_CK(cudaEventRecord(h.join, h.hs));
  WG_CK(cudaStreamWaitEvent(s, h.join, 0));
  return WG_OK;
}

// ------------------------------------------------------------ small kernels
namespace {

template <typename T>
__global__ void k_prep_weight(const float* W, int batch, int rows, int cols, int transpose, T* out, int64_t ldo,
                              int out_rows) {
  // out is batch x [out_rows x ldo]; element (b, i, j) = transpose ? W[b][j][i] : W[b][i][j], 0 outside
  const int64_t n = (int64_t)batch * out_rows * ldo;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t bi = t / ldo;
    const int b = (int)(bi / out_rows), i = (int)(bi % out_rows), j = (int)(t % ldo);
    const float* Wb = W + (int64_t)b * rows * cols;
    float v = 0.f;
    if (transpose) { if (i < cols && j < rows) v = Wb[(int64_t)j * cols + i]; }
    else { if (i < rows && j < cols) v = Wb[(int64_t)i * cols + j]; }
    out[t] = (T)v;
  }
}

// Column partial sums of (optionally ReLU-masked) dy over blocks of rows,
// 16-byte vectors per thread; block partials reduced in a fixed order.
template <typename T>
__global__ void __launch_bounds__(256, 4) k_colsum(int64_t M, int N, const T* dy, int64_t lddy, const T* ref,
                                                int64_t ldref, T* dt, int64_t ldt, float* part, int64_t rows_per_blk,
                                                const float* rs2, T* dt2, int64_t ldt2, int fc2, int64_t cs2) {
  constexpr int EPV = VT<T>::EPV;
  extern __shared__ float red[];                       // [nsub][nv*EPV]
  const int nv = (N + EPV - 1) / EPV;                  // vectors per row (<= 256)
  const int nsub = blockDim.x / nv;
  const int vec = threadIdx.x % nv, sub = threadIdx.x / nv;
  const int64_t r0 = blockIdx.x * rows_per_blk, r1 = min(M, r0 + rows_per_blk);
  float acc[EPV] = {};
  if (sub < nsub) {
    // 4 rows' loads in flight per thread; rows are still added in increasing
    // order (the same fixed order as a one-row loop: results unchanged)
    constexpr int RU = 4;
    for (int64_t r4 = r0 + sub; r4 < r1; r4 += (int64_t)RU * nsub) {
      int4 pv[RU], pm[RU];
#pragma unroll
      for (int k = 0; k < RU; ++k) {
        const int64_t rr = r4 + (int64_t)k * nsub;
        pv[k] = rr < r1 ? ldg16(dy + rr * lddy + vec * EPV) : make_int4(0, 0, 0, 0);
        pm[k] = (ref && rr < r1) ? ldg16(ref + rr * ldref + vec * EPV) : make_int4(0, 0, 0, 0);
      }
#pragma unroll
      for (int k = 0; k < RU; ++k) {
      const int64_t r = r4 + (int64_t)k * nsub;
      if (r >= r1) break;
      float v[EPV];
      VT<T>::unpack(pv[k], v);
      if (ref) {
        float m[EPV];
        VT<T>::unpack(pm[k], m);
#pragma unroll
        for (int i = 0; i < EPV; ++i) v[i] = m[i] > 0.f ? v[i] : 0.f;
      }
#pragma unroll
      for (int i = 0; i < EPV; ++i) if (vec * EPV + i >= N) v[i] = 0.f;
      if (dt) *reinterpret_cast<int4*>(dt + r * ldt + vec * EPV) = VT<T>::pack(v);
      if (dt2) {   // second output: scaled by rs2 (if any), optionally column-chunked
        float w[EPV];
        const float sc = rs2 ? rs2[r] : 1.f;
#pragma unroll
        for (int i = 0; i < EPV; ++i) w[i] = sc * v[i];
        const int col = vec * EPV;
        T* q = fc2 > 0 ? dt2 + (int64_t)(col / fc2) * cs2 + r * ldt2 + col % fc2 : dt2 + r * ldt2 + col;
        *reinterpret_cast<int4*>(q) = VT<T>::pack(w);
      }
#pragma unroll
      for (int i = 0; i < EPV; ++i) acc[i] += v[i];
      }
    }
#pragma unroll
    for (int i = 0; i < EPV; ++i) red[sub * nv * EPV + vec * EPV + i] = acc[i];
  }
  __syncthreads();
  for (int c = threadIdx.x; c < N; c += blockDim.x) {
    float s = 0.f;
    for (int k = 0; k < nsub; ++k) s += red[k * nv * EPV + c];
    part[(int64_t)blockIdx.x * N + c] = s;
  }
}

// out[c] = sum_b part[b][c]: 32 columns per CTA, warp w of 32 sums blocks
// b = w mod 32 (4 loads in flight), then the 32 warp partials are added in
// warp order -- a fixed order, so the result is deterministic
__global__ void __launch_bounds__(1024) k_colsum_reduce(const float* part, int nblk, int N, float* out) {
  __shared__ float red[32][33];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int c = blockIdx.x * 32 + lane;
  float s = 0.f;
  if (c < N) {
#pragma unroll 4
    for (int b = warp; b < nblk; b += 32) s += part[(int64_t)b * N + c];
  }
  red[warp][lane] = s;
  __syncthreads();
  if (warp == 0 && c < N) {
    float t = 0.f;
#pragma unroll
    for (int w = 0; w < 32; ++w) t += red[w][lane];
    out[c] = t;
  }
}

constexpr int COLSUM_BLKS = 1184;  // 8 x 148 SMs

}  // namespace

wg_status prep_weight_batched(wg_dtype dt, const float* W, int batch, int rows, int cols, int transpose, void* out,
                              int64_t ldo, int out_rows, cudaStream_t s) {
  const int64_t n = (int64_t)batch * out_rows * ldo;
  const unsigned grid = (unsigned)std::min<int64_t>(cdiv(n, 256), 1184);
  ProfScope ps(PK_MISC, s, (double)batch * rows * cols * 4.0 + (double)n * (dt == WG_BF16 ? 2.0 : 4.0), 0.0);
  if (grid == 0) return WG_OK;
  if (dt == WG_BF16)
    WG_LAUNCH(k_prep_weight<__nv_bfloat16>, grid, 256, 0, s, W, batch, rows, cols, transpose, (__nv_bfloat16*)out, ldo,
              out_rows);
  else
    WG_LAUNCH(k_prep_weight<float>, grid, 256, 0, s, W, batch, rows, cols, transpose, (float*)out, ldo, out_rows);
  return WG_OK;
}

wg_status prep_weight(wg_dtype dt, const float* W, int rows, int cols, int transpose, void* out, int64_t ldo,
                      int out_rows, cudaStream_t s) {
  return prep_weight_batched(dt, W, 1, rows, cols, transpose, out, ldo, out_rows, s);
}

size_t bias_grad_scratch(int64_t M, int N) { return sizeof(float) * (size_t)COLSUM_BLKS * N; }

wg_status bias_grad_mask(wg_dtype dt, int64_t M, int N, const void* dy, int64_t lddy, const void* ref,
                         int64_t ldref, void* dt_out, int64_t ldt, float* db, float* scratch, cudaStream_t s,
                         const float* rs2, void* dt2, int64_t ldt2, int fc2, int64_t cs2) {
  const int EPV = dt == WG_BF16 ? 8 : 4;
  const int nv = (int)cdiv(N, EPV);
  WG_REQ(nv <= 256, WG_ERR_UNSUPPORTED, "bias gradient: more than 256 vectors per row");
  const int64_t rpb = std::max<int64_t>(1, cdiv(M, COLSUM_BLKS));
  const int nblk = (int)std::max<int64_t>(1, cdiv(M, rpb));
  const double es = dt == WG_BF16 ? 2.0 : 4.0;
  ProfScope ps(PK_MISC, s, (double)M * N * es * (1 + (ref ? 1 : 0) + (dt_out ? 1 : 0) + (dt2 ? 1 : 0)), (double)M * N);
  const int threads = 256;
  const size_t smem = (size_t)(threads / nv) * nv * EPV * sizeof(float);
  if (dt == WG_BF16)
    WG_LAUNCH(k_colsum<__nv_bfloat16>, nblk, threads, smem, s, M, N, (const __nv_bfloat16*)dy, lddy,
              (const __nv_bfloat16*)ref, ldref, (__nv_bfloat16*)dt_out, ldt, scratch, rpb, rs2, (__nv_bfloat16*)dt2,
              ldt2, fc2, cs2);
  else
    WG_LAUNCH(k_colsum<float>, nblk, threads, smem, s, M, N, (const float*)dy, lddy, (const float*)ref, ldref,
              (float*)dt_out, ldt, scratch, rpb, rs2, (float*)dt2, ldt2, fc2, cs2);
  if (db) WG_LAUNCH(k_colsum_reduce, (unsigned)cdiv(N, 32), 1024, 0, s, scratch, nblk, N, db);
  return WG_OK;
}

}  // namespace wg
