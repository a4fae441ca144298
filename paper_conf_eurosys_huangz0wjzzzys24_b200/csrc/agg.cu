// Gather + segment-reduce over gTask work items (SURVEY §8(a) a6 forward,
// a10 backward on the transposed partition) and the SPLIT-row combine (a8).
//
// Indexing ops of the paper: Index (h[src-id]) then Index-add (h[dst-id] +=)
// (Fig 2b); "indexing dominates" tensor-centric execution
// (P:L821-831).  Here one CTA executes one work item (the rows of one gTask);
// the destination ordering inside a gTask is sorted, so every output row is
// reduced in registers and stored ONCE with 16-byte vector stores -- no global
// atomics.  Per-edge coefficients are factored into a per-source scale
// (gathered with the row) and a per-destination scale.
//
//   out[r] = epi( rscale[r] * sum_{j in seg(r)} gscale[idx_j] * table[idx_j]
//                 + self_coef * self[r] )
//   epi(v) = mask( relu( v + bias ) )
//
// Differentiated execution: SPLIT chunks (frequent-value /
// overfill rows) run first and write fp32 partials that a combine kernel sums
// in chunk order; rows heavier than HEAVY_DEG inside a regular gTask are
// processed by all 8 warps of the CTA (edge-parallel, smem reduction); the
// other rows get one warp each.  All reductions use a fixed order, so results
// are run-to-run deterministic.
#include "wg_internal.cuh"

namespace wg {

namespace {

constexpr int WARPS = 8;
constexpr int HEAVY_DEG = 256;

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

// epilogue on one 16-byte output vector (EPV columns starting at column c0)
template <typename T>
__device__ __forceinline__ void epilogue_store(const float* acc_in, int64_t grow, int r, int cv, int c0,
                                               float rs, const void* self_tab, int64_t ld_self, float self_coef,
                                               const float* bias, int relu, const void* mask_ref, int64_t ld_mask,
                                               void* out, int64_t ld_out, int F) {
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
  (void)grow; (void)cv;
}

template <typename T>
__device__ __forceinline__ void zero_row(void* z, int64_t ldz, int cols, int r, int lane, int nl) {
  if (!z) return;
  constexpr int EPV = VT<T>::EPV;
  T* p = static_cast<T*>(z) + (int64_t)r * ldz;
  for (int c = lane * EPV; c < cols; c += nl * EPV) *reinterpret_cast<int4*>(p + c) = make_int4(0, 0, 0, 0);
}

// Warp accumulation of the vectors [cv0, cv0 + nvec) of rows table[idx[j]],
// j in [b, e).  LPE lanes cover one edge's row chunk (NV vectors per lane);
// G = 32 / LPE edges are processed in parallel, U batches in flight.
template <typename T, int LPE, int NV, int U>
__device__ __forceinline__ void warp_accumulate(const AggArgs& a, int64_t b, int64_t e, int cv0, int nvec,
                                                float (&acc)[NV][VT<T>::EPV]) {
  constexpr int EPV = VT<T>::EPV;
  constexpr int G = 32 / LPE;
  const int lane = threadIdx.x & 31, grp = lane / LPE, l = lane % LPE;
#pragma unroll
  for (int q = 0; q < NV; ++q)
#pragma unroll
    for (int i = 0; i < EPV; ++i) acc[q][i] = 0.f;
  const T* tab = static_cast<const T*>(a.table);
  for (int64_t base = b; base < e; base += 32) {
    const int n = (int)(e - base < 32 ? e - base : 32);
    const int my_idx = lane < n ? a.idx[base + lane] : 0;
    const float my_sc = (a.gscale && lane < n) ? a.gscale[my_idx] : 1.f;
    for (int j = 0; j < n; j += G * U) {
      int4 v[U][NV];
      float sc[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int k = j + u * G + grp;
        const bool ok = k < n;
        const int s = __shfl_sync(0xffffffffu, my_idx, ok ? k : 0);
        sc[u] = __shfl_sync(0xffffffffu, my_sc, ok ? k : 0);
        const T* row = tab + (int64_t)s * a.ld_tab + (int64_t)cv0 * EPV;
#pragma unroll
        for (int q = 0; q < NV; ++q) {
          const int vi = l + q * LPE;
          v[u][q] = (ok && vi < nvec) ? ldg16(row + vi * EPV) : make_int4(0, 0, 0, 0);
        }
        if (!ok) sc[u] = 0.f;
      }
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int q = 0; q < NV; ++q) VT<T>::add(acc[q], v[u][q], sc[u]);
    }
  }
#pragma unroll
  for (int off = LPE; off < 32; off <<= 1)
#pragma unroll
    for (int q = 0; q < NV; ++q)
#pragma unroll
      for (int i = 0; i < EPV; ++i) acc[q][i] += __shfl_xor_sync(0xffffffffu, acc[q][i], off);
}

template <typename T, int LPE, int NV, int U>
__device__ void do_row_warp(const AggArgs& a, int r, int64_t b, int64_t e, int VPR) {
  constexpr int EPV = VT<T>::EPV;
  constexpr int CW = LPE * NV;
  const int lane = threadIdx.x & 31, l = lane % LPE;
  const float rs = a.rscale ? a.rscale[a.row_base + r] : 1.f;
  for (int cv0 = 0; cv0 < VPR; cv0 += CW) {
    const int nvec = min(CW, VPR - cv0);
    float acc[NV][EPV];
    warp_accumulate<T, LPE, NV, U>(a, b, e, cv0, nvec, acc);
    if (lane < LPE) {
#pragma unroll
      for (int q = 0; q < NV; ++q) {
        const int vi = l + q * LPE;
        if (vi < nvec)
          epilogue_store<T>(acc[q], a.row_base + r, r, cv0 + vi, (cv0 + vi) * EPV, rs, a.self_tab, a.ld_self,
                            a.self_coef, a.bias, a.relu, a.mask_ref, a.ld_mask, a.out, a.ld_out, a.F);
      }
    }
  }
  zero_row<T>(a.zero_out, a.ld_zero, a.zero_cols, r, lane, 32);
}

// whole CTA on one row (heavy row or SPLIT chunk).  partial_slot >= 0: write
// the raw fp32 sum to the partial buffer instead of the epilogue.
template <typename T, int LPE, int NV, int U>
__device__ void do_row_cta(const AggArgs& a, int r, int64_t b, int64_t e, int VPR, int partial_slot, float* red) {
  constexpr int EPV = VT<T>::EPV;
  constexpr int CW = LPE * NV;
  const int lane = threadIdx.x & 31, l = lane % LPE, w = threadIdx.x >> 5;
  const int64_t len = e - b;
  const int64_t wb = b + len * w / WARPS, we = b + len * (w + 1) / WARPS;
  const float rs = a.rscale ? a.rscale[a.row_base + r] : 1.f;
  for (int cv0 = 0; cv0 < VPR; cv0 += CW) {
    const int nvec = min(CW, VPR - cv0);
    float acc[NV][EPV];
    warp_accumulate<T, LPE, NV, U>(a, wb, we, cv0, nvec, acc);
    __syncthreads();  // red[] reuse across chunks
    if (lane < LPE) {
#pragma unroll
      for (int q = 0; q < NV; ++q)
#pragma unroll
        for (int i = 0; i < EPV; ++i) red[(w * CW + l + q * LPE) * EPV + i] = acc[q][i];
    }
    __syncthreads();
    for (int vi = threadIdx.x; vi < nvec; vi += blockDim.x) {
      float s[EPV];
#pragma unroll
      for (int i = 0; i < EPV; ++i) s[i] = 0.f;
      for (int ww = 0; ww < WARPS; ++ww)
#pragma unroll
        for (int i = 0; i < EPV; ++i) s[i] += red[(ww * CW + vi) * EPV + i];
      const int c0 = (cv0 + vi) * EPV;
      if (partial_slot >= 0) {
        float* pp = a.partial + (int64_t)partial_slot * a.ld_part + c0;
#pragma unroll
        for (int i = 0; i < EPV; ++i) pp[i] = s[i];
      } else {
        epilogue_store<T>(s, a.row_base + r, r, cv0 + vi, c0, rs, a.self_tab, a.ld_self, a.self_coef, a.bias,
                          a.relu, a.mask_ref, a.ld_mask, a.out, a.ld_out, a.F);
      }
    }
  }
  if (partial_slot < 0) zero_row<T>(a.zero_out, a.ld_zero, a.zero_cols, r, threadIdx.x, blockDim.x);
}

template <typename T, int LPE, int NV, int U>
__global__ void __launch_bounds__(WARPS * 32) k_agg(AggArgs a, int VPR) {
  extern __shared__ float red[];
  __shared__ int heavy[1024];
  __shared__ int n_heavy;
  const WorkItem it = a.items[blockIdx.x];
  if (it.split_slot >= 0) {
    do_row_cta<T, LPE, NV, U>(a, it.row_lo, it.e_lo, it.e_hi, VPR, it.split_slot, red);
    return;
  }
  if (threadIdx.x == 0) n_heavy = 0;
  __syncthreads();
  const int nrows = it.row_hi - it.row_lo;
  // rows: heavy ones are collected (in row order, one pass of up to 1024 rows)
  for (int i = threadIdx.x; i < nrows && i < 1024; i += blockDim.x) {
    const int r = it.row_lo + i;
    const int64_t deg = a.row_ptr[r + 1] - a.row_ptr[r];
    if (deg >= HEAVY_DEG && deg <= a.E_max) heavy[atomicAdd(&n_heavy, 1)] = r;
  }
  __syncthreads();
  const int nh = n_heavy;
  for (int h = 0; h < nh; ++h) {
    const int r = heavy[h];
    do_row_cta<T, LPE, NV, U>(a, r, a.row_ptr[r], a.row_ptr[r + 1], VPR, -1, red);
    __syncthreads();
  }
  const int w = threadIdx.x >> 5;
  for (int i = w; i < nrows; i += WARPS) {
    const int r = it.row_lo + i;
    const int64_t b = a.row_ptr[r], e = a.row_ptr[r + 1];
    const int64_t deg = e - b;
    if (deg > a.E_max) continue;                       // SPLIT row: combine kernel
    if (deg >= HEAVY_DEG && i < 1024) continue;        // done cooperatively
    do_row_warp<T, LPE, NV, U>(a, r, b, e, VPR);
  }
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
    epilogue_store<T>(s, a.row_base + sr.row, sr.row, vi, c0, rs, a.self_tab, a.ld_self, a.self_coef, a.bias, a.relu,
                      a.mask_ref, a.ld_mask, a.out, a.ld_out, a.F);
  }
  zero_row<T>(a.zero_out, a.ld_zero, a.zero_cols, sr.row, threadIdx.x, blockDim.x);
}

template <typename T, int LPE, int NV, int U>
wg_status launch_cfg(const AggArgs& a, int VPR, cudaStream_t s) {
  constexpr int EPV = VT<T>::EPV;
  const size_t smem = (size_t)WARPS * LPE * NV * EPV * sizeof(float);
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

template <typename T>
wg_status launch_t(const AggArgs& a, cudaStream_t s) {
  constexpr int EPV = VT<T>::EPV;
  const int VPR = (int)cdiv(a.F, EPV);
  if (VPR <= 1) return launch_cfg<T, 1, 1, 1>(a, VPR, s);
  if (VPR <= 2) return launch_cfg<T, 2, 1, 2>(a, VPR, s);
  if (VPR <= 4) return launch_cfg<T, 4, 1, 4>(a, VPR, s);
  if (VPR <= 8) return launch_cfg<T, 8, 1, 4>(a, VPR, s);
  if (VPR <= 16) return launch_cfg<T, 16, 1, 8>(a, VPR, s);
  if (VPR <= 32) return launch_cfg<T, 32, 1, 8>(a, VPR, s);
  if (VPR <= 64) return launch_cfg<T, 32, 2, 4>(a, VPR, s);
  return launch_cfg<T, 32, 4, 2>(a, VPR, s);
}

}  // namespace

wg_status launch_agg(wg_dtype dt, const AggArgs& a, cudaStream_t s) {
  if (a.n_items == 0) return WG_OK;
  // algorithmic bytes: per edge the index (4 B), the gathered row (F elements)
  // and the source scale if any; per row the output, row_ptr and optional
  // self / mask rows
  const double es = dt == WG_BF16 ? 2.0 : 4.0, rb = a.F * es;
  const double bytes = a.n_edges * (4.0 + rb + (a.gscale ? 4.0 : 0.0)) +
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

// ------------------------------------------------------------ small kernels
namespace {

template <typename T>
__global__ void k_prep_weight(const float* W, int rows, int cols, int transpose, T* out, int64_t ldo, int out_rows) {
  // out is [out_rows x ldo]; element (i, j) = transpose ? W[j][i] : W[i][j], 0 outside
  int64_t n = (int64_t)out_rows * ldo;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
    int i = (int)(t / ldo), j = (int)(t % ldo);
    float v = 0.f;
    if (transpose) { if (i < cols && j < rows) v = W[(int64_t)j * cols + i]; }
    else { if (i < rows && j < cols) v = W[(int64_t)i * cols + j]; }
    out[t] = (T)v;
  }
}

// column partial sums of (optionally relu-masked) dy over row blocks
template <typename T>
__global__ void k_colsum(int64_t M, int N, const T* dy, int64_t lddy, const T* ref, int64_t ldref, T* dt,
                         int64_t ldt, float* part, int64_t rows_per_blk) {
  const int64_t r0 = blockIdx.x * rows_per_blk, r1 = min(M, r0 + rows_per_blk);
  for (int c = threadIdx.x; c < N; c += blockDim.x) {
    float s = 0.f;
    for (int64_t r = r0; r < r1; ++r) {
      float v = (float)dy[r * lddy + c];
      if (ref && !((float)ref[r * ldref + c] > 0.f)) v = 0.f;
      if (dt) dt[r * ldt + c] = (T)v;
      s += v;
    }
    part[(int64_t)blockIdx.x * N + c] = s;
  }
}

__global__ void k_colsum_reduce(const float* part, int nblk, int N, float* out) {
  int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= N) return;
  float s = 0.f;
  for (int b = 0; b < nblk; ++b) s += part[(int64_t)b * N + c];
  out[c] = s;
}

constexpr int COLSUM_BLKS = 1184;  // 8 x 148 SMs

}  // namespace

wg_status prep_weight(wg_dtype dt, const float* W, int rows, int cols, int transpose, void* out, int64_t ldo,
                      int out_rows, cudaStream_t s) {
  int64_t n = (int64_t)out_rows * ldo;
  unsigned grid = (unsigned)std::min<int64_t>(cdiv(n, 256), 1184);
  ProfScope ps(PK_MISC, s, (double)rows * cols * 4.0 + (double)n * (dt == WG_BF16 ? 2.0 : 4.0), 0.0);
  if (grid == 0) return WG_OK;
  if (dt == WG_BF16)
    WG_LAUNCH(k_prep_weight<__nv_bfloat16>, grid, 256, 0, s, W, rows, cols, transpose, (__nv_bfloat16*)out, ldo, out_rows);
  else
    WG_LAUNCH(k_prep_weight<float>, grid, 256, 0, s, W, rows, cols, transpose, (float*)out, ldo, out_rows);
  return WG_OK;
}

size_t bias_grad_scratch(int64_t M, int N) { return sizeof(float) * (size_t)COLSUM_BLKS * N; }

wg_status bias_grad_mask(wg_dtype dt, int64_t M, int N, const void* dy, int64_t lddy, const void* ref,
                         int64_t ldref, void* dt_out, int64_t ldt, float* db, float* scratch, cudaStream_t s) {
  const int64_t rpb = std::max<int64_t>(1, cdiv(M, COLSUM_BLKS));
  const int nblk = (int)std::max<int64_t>(1, cdiv(M, rpb));
  const double es = dt == WG_BF16 ? 2.0 : 4.0;
  ProfScope ps(PK_MISC, s, (double)M * N * es * (1 + (ref ? 1 : 0) + (dt_out ? 1 : 0)), (double)M * N);
  const int threads = N >= 256 ? 256 : (int)rup(N, 32);
  if (dt == WG_BF16)
    WG_LAUNCH(k_colsum<__nv_bfloat16>, nblk, threads, 0, s, M, N, (const __nv_bfloat16*)dy, lddy,
              (const __nv_bfloat16*)ref, ldref, (__nv_bfloat16*)dt_out, ldt, scratch, rpb);
  else
    WG_LAUNCH(k_colsum<float>, nblk, threads, 0, s, M, N, (const float*)dy, lddy, (const float*)ref, ldref,
              (float*)dt_out, ldt, scratch, rpb);
  if (db) WG_LAUNCH(k_colsum_reduce, (unsigned)cdiv(N, 128), 128, 0, s, scratch, nblk, N, db);
  return WG_OK;
}

}  // namespace wg
