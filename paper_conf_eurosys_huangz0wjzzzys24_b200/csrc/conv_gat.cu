// GAT layer (Velickovic et al. [40]; readings Q6):
// "MHA" is the neural op.  Per head k:
//   g_k = x W_k ; el[u] = g_k[u].a_l,k ; er[v] = g_k[v].a_r,k
//   t_e = el[s_e] + er[d_e] ; l_e = LeakyReLU(t_e)
//   alpha_e = softmax over in(v) of l_e ; y_k[v] = sum_{e in in(v)} alpha_e g_k[s_e]
// heads concatenated (hidden layers) or averaged (last layer), + bias.
//
// Plan: transform-before-gather only (g = x W is the vertex-level GEMM, T2
// indexing swapping).  The edge softmax is a
// single-pass online softmax per (destination, head) with warp-level
// primitives, so every edge's source row is read once; rows longer than
// GAT_CHUNK edges are split into chunks whose (max, sum, vector) triples are
// merged flash-style in a fixed order (overfill / frequent-value rows,
// P:L2554-2582).  Backward (exact gradients, Q8)
// runs a source-major pass over the transposed partition (dg, del, dt_e)
// and a destination-major pass for der.
#include <algorithm>

#include "plan.h"

namespace wg {

namespace {

constexpr int GAT_CHUNK = 256;

struct RowChunk {
  int32_t row;          // local row
  int32_t slot;         // partial slot (>= 0) when the row is split, else -1
  int64_t e_lo, e_hi;   // positions in the side's sorted edge order
};

struct GatPlan {
  RowChunk* fwd = nullptr;
  int n_fwd = 0;
  RowChunk* bwd = nullptr;
  int n_bwd = 0;
  SplitRow* fsplit = nullptr;   // split rows (forward), slots consecutive
  int n_fsplit = 0, n_fslots = 0;
  SplitRow* bsplit = nullptr;
  int n_bsplit = 0, n_bslots = 0;
};

void build_chunks(const Side& S, std::vector<RowChunk>& out, std::vector<SplitRow>& split, int* n_slots) {
  std::vector<std::pair<int64_t, RowChunk>> tmp;
  int slot = 0;
  for (int64_t r = 0; r < S.n_rows; ++r) {
    const int64_t b = S.h_row_ptr[r], e = S.h_row_ptr[r + 1];
    if (e - b <= GAT_CHUNK) {
      tmp.push_back({e - b, RowChunk{(int32_t)r, -1, b, e}});
      continue;
    }
    split.push_back(SplitRow{(int32_t)r, slot, 0, 0});
    for (int64_t c = b; c < e; c += GAT_CHUNK) {
      tmp.push_back({INT64_MAX / 2, RowChunk{(int32_t)r, slot++, c, std::min(c + GAT_CHUNK, e)}});
      split.back().n_slots++;
    }
  }
  std::stable_sort(tmp.begin(), tmp.end(), [](const auto& x, const auto& y) { return x.first > y.first; });
  for (auto& t : tmp) out.push_back(t.second);
  *n_slots = slot;
}

template <typename T> struct GV;
template <> struct GV<float> {
  static constexpr int EPV = 4;
  __device__ static void unpack(const int4& v, float* f) {
    f[0] = __int_as_float(v.x); f[1] = __int_as_float(v.y); f[2] = __int_as_float(v.z); f[3] = __int_as_float(v.w);
  }
  __device__ static int4 pack(const float* f) {
    return make_int4(__float_as_int(f[0]), __float_as_int(f[1]), __float_as_int(f[2]), __float_as_int(f[3]));
  }
};
template <> struct GV<__nv_bfloat16> {
  static constexpr int EPV = 8;
  __device__ static void unpack(const int4& v, float* f) {
    const uint32_t w[4] = {(uint32_t)v.x, (uint32_t)v.y, (uint32_t)v.z, (uint32_t)v.w};
#pragma unroll
    for (int i = 0; i < 4; ++i) { f[2 * i] = __uint_as_float(w[i] << 16); f[2 * i + 1] = __uint_as_float(w[i] & 0xffff0000u); }
  }
  __device__ static int4 pack(const float* f) {
    uint32_t w[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      __nv_bfloat162 h = __floats2bfloat162_rn(f[2 * i], f[2 * i + 1]);
      w[i] = *reinterpret_cast<uint32_t*>(&h);
    }
    return make_int4((int)w[0], (int)w[1], (int)w[2], (int)w[3]);
  }
};

__device__ __forceinline__ int4 ld16(const void* p) { return __ldg(reinterpret_cast<const int4*>(p)); }
__device__ __forceinline__ float lrelu(float t, float s) { return t > 0.f ? t : s * t; }

struct GatArgs {
  int H, Fo, HF;            // heads, per-head width, H*Fo
  int VPR;                  // vectors per G row
  float slope;
  const void* G; int64_t ldg;          // [V x ldg]
  const float* el; const float* er;    // [V x H]
  const int32_t* idx;                  // gathered ids (sorted order of the side)
  const RowChunk* chunks; int n_chunks;
  // forward outputs
  void* agg; int64_t ld_agg;           // per-head aggregation (pre-bias)
  float* m; float* l;                  // [V x H] softmax max / denominator
  float* part; int part_ld;            // partial slots [slots x part_ld]: HF acc + H m + H l
  // backward
  const void* dy; int64_t lddy; int concat;
  const float* s;                      // [V x H]  dy_k . agg_k
  const int64_t* fwdpos;               // transposed position -> forward position
  float* dt;                           // [E x H] (forward order)
  float* dg; int64_t ld_dg;            // [V x HF] fp32 (sum alpha dy)
  float* del;                          // [V x H]
};

// ---------------------------------------------------------------- el / er
template <typename T, int NV>
__global__ void k_gat_logits(int64_t V, GatArgs a, const float* al, const float* ar) {
  constexpr int EPV = GV<T>::EPV;
  const int lane = threadIdx.x & 31;
  const int64_t v = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (v >= V) return;
  float pl[NV], pr[NV];
  int hd[NV];
#pragma unroll
  for (int q = 0; q < NV; ++q) {
    const int vi = lane + 32 * q;
    pl[q] = pr[q] = 0.f;
    hd[q] = -1;
    if (vi < a.VPR) {
      float g[EPV];
      GV<T>::unpack(ld16(static_cast<const T*>(a.G) + v * a.ldg + vi * EPV), g);
      const int c0 = vi * EPV;
      hd[q] = c0 / a.Fo;
#pragma unroll
      for (int i = 0; i < EPV; ++i) {
        if (c0 + i < a.HF) { pl[q] += g[i] * al[c0 + i]; pr[q] += g[i] * ar[c0 + i]; }
      }
    }
  }
  for (int h = 0; h < a.H; ++h) {
    float sl = 0.f, sr = 0.f;
#pragma unroll
    for (int q = 0; q < NV; ++q) if (hd[q] == h) { sl += pl[q]; sr += pr[q]; }
#pragma unroll
    for (int o = 16; o; o >>= 1) { sl += __shfl_xor_sync(0xffffffffu, sl, o); sr += __shfl_xor_sync(0xffffffffu, sr, o); }
    if (lane == 0) { const_cast<float*>(a.el)[v * a.H + h] = sl; const_cast<float*>(a.er)[v * a.H + h] = sr; }
  }
}

// ------------------------------------------------- forward online softmax
// one warp per row chunk (destination row, in-edges [e_lo, e_hi))
template <typename T, int NV, int U>
__global__ void __launch_bounds__(256) k_gat_fwd(GatArgs a, int64_t row_base) {
  constexpr int EPV = GV<T>::EPV;
  const int lane = threadIdx.x & 31;
  const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (w >= a.n_chunks) return;
  const RowChunk ch = a.chunks[w];
  const int64_t d = row_base + ch.row;     // global destination id
  const T* G = static_cast<const T*>(a.G);
  int hd[NV];
  float erd[NV], m[NV], l[NV], acc[NV][EPV];
#pragma unroll
  for (int q = 0; q < NV; ++q) {
    const int vi = lane + 32 * q;
    hd[q] = vi < a.VPR ? (vi * EPV) / a.Fo : 0;
    erd[q] = a.er[d * a.H + hd[q]];
    m[q] = -INFINITY;
    l[q] = 0.f;
#pragma unroll
    for (int i = 0; i < EPV; ++i) acc[q][i] = 0.f;
  }
  for (int64_t base = ch.e_lo; base < ch.e_hi; base += 32) {
    const int n = (int)min((int64_t)32, ch.e_hi - base);
    const int my = lane < n ? a.idx[base + lane] : 0;
    for (int j = 0; j < n; j += U) {
      int4 v[U][NV];
      float ls[U][NV];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int k = j + u;
        const int s = __shfl_sync(0xffffffffu, my, k < n ? k : 0);
#pragma unroll
        for (int q = 0; q < NV; ++q) {
          const int vi = lane + 32 * q;
          const bool ok = k < n && vi < a.VPR;
          v[u][q] = ok ? ld16(G + (int64_t)s * a.ldg + vi * EPV) : make_int4(0, 0, 0, 0);
          ls[u][q] = k < n ? lrelu(a.el[(int64_t)s * a.H + hd[q]] + erd[q], a.slope) : -INFINITY;
        }
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
#pragma unroll
        for (int q = 0; q < NV; ++q) {
          if (ls[u][q] == -INFINITY) continue;
          const float mn = fmaxf(m[q], ls[u][q]);
          const float sc = __expf(m[q] - mn), p = __expf(ls[u][q] - mn);
          float g[EPV];
          GV<T>::unpack(v[u][q], g);
          l[q] = l[q] * sc + p;
#pragma unroll
          for (int i = 0; i < EPV; ++i) acc[q][i] = acc[q][i] * sc + p * g[i];
          m[q] = mn;
        }
      }
    }
  }
#pragma unroll
  for (int q = 0; q < NV; ++q) {
    const int vi = lane + 32 * q;
    if (vi >= a.VPR) continue;
    const int c0 = vi * EPV;
    const bool head_lead = (c0 % a.Fo) == 0;
    if (ch.slot >= 0) {
      float* pp = a.part + (int64_t)ch.slot * a.part_ld;
#pragma unroll
      for (int i = 0; i < EPV; ++i) pp[c0 + i] = acc[q][i];
      if (head_lead) { pp[a.HF + hd[q]] = m[q]; pp[a.HF + a.H + hd[q]] = l[q]; }
    } else {
      float o[EPV];
      const float inv = l[q] > 0.f ? 1.f / l[q] : 0.f;
#pragma unroll
      for (int i = 0; i < EPV; ++i) o[i] = (c0 + i < a.HF) ? acc[q][i] * inv : 0.f;
      float* ag = static_cast<float*>(a.agg) + (int64_t)ch.row * a.ld_agg + c0;
#pragma unroll
      for (int i = 0; i < EPV; ++i) ag[i] = o[i];
      if (head_lead) { a.m[d * a.H + hd[q]] = m[q]; a.l[d * a.H + hd[q]] = l[q]; }
    }
  }
}

// flash-style merge of the (m, l, acc) partials of split rows, chunk order
template <typename T>
__global__ void k_gat_fwd_combine(GatArgs a, const SplitRow* rows, int64_t row_base) {
  constexpr int EPV = GV<T>::EPV;
  const SplitRow sr = rows[blockIdx.x];
  const int64_t d = row_base + sr.row;
  for (int c = threadIdx.x; c < a.VPR * EPV; c += blockDim.x) {
    const int h = min(c / a.Fo, a.H - 1);
    float m = -INFINITY, l = 0.f, o = 0.f;
    for (int k = 0; k < sr.n_slots; ++k) {
      const float* pp = a.part + (int64_t)(sr.first_slot + k) * a.part_ld;
      const float mk = pp[a.HF + h], lk = pp[a.HF + a.H + h];
      if (lk <= 0.f) continue;
      const float mn = fmaxf(m, mk);
      const float s0 = __expf(m - mn), s1 = __expf(mk - mn);
      l = l * s0 + lk * s1;
      o = o * s0 + (c < a.HF ? pp[c] : 0.f) * s1;
      m = mn;
    }
    const float val = (c < a.HF && l > 0.f) ? o / l : 0.f;
    static_cast<float*>(a.agg)[(int64_t)sr.row * a.ld_agg + c] = val;
    if (c < a.HF && c % a.Fo == 0) { a.m[d * a.H + h] = m; a.l[d * a.H + h] = l; }
  }
}

// y = concat(agg) + b or mean_k(agg_k) + b, optional ReLU; also s = dy . agg (backward)
template <typename T>
__global__ void k_gat_out(int64_t rows, GatArgs a, const float* bias, int relu, void* y, int64_t ldy, int FO) {
  const int64_t n = rows * (int64_t)ldy;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n; t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = t / ldy;
    const int c = (int)(t % ldy);
    float v = 0.f;
    if (c < FO) {
      const float* ag = static_cast<const float*>(a.agg) + r * a.ld_agg;
      if (a.concat) v = ag[c];
      else {
        for (int h = 0; h < a.H; ++h) v += (float)ag[h * a.Fo + c];
        v /= (float)a.H;
      }
      if (bias) v += bias[c];
      if (relu) v = fmaxf(v, 0.f);
    }
    if (c < ((FO + 7) / 8) * 8) static_cast<T*>(y)[r * ldy + c] = (T)v;
  }
}

// s[v,h] = dy_k[v] . agg_k[v]   (= sum_{e in in(v)} alpha_e dalpha_e)
template <typename T>
__global__ void k_gat_s(int64_t rows, int64_t row_base, GatArgs a, float* s) {
  const int lane = threadIdx.x & 31;
  const int64_t r = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (r >= rows) return;
  const float* ag = static_cast<const float*>(a.agg) + r * a.ld_agg;
  const T* dy = static_cast<const T*>(a.dy) + r * a.lddy;
  for (int h = 0; h < a.H; ++h) {
    float acc = 0.f;
    for (int j = lane; j < a.Fo; j += 32) {
      const float g = a.concat ? (float)dy[h * a.Fo + j] : (float)dy[j] / (float)a.H;
      acc += g * (float)ag[h * a.Fo + j];
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
    if (lane == 0) s[(row_base + r) * a.H + h] = acc;
  }
}

// ---------------------------------------------- backward, source-major pass
// warp per (source row, out-edge chunk): dg[u] += sum alpha dy_k[d], del[u] +=
// sum dt_e, dt_e written at the edge's forward position.
template <typename T, int NV>
__global__ void __launch_bounds__(256) k_gat_bwd_src(GatArgs a, int64_t row_base) {
  constexpr int EPV = 4;                       // G is kept in fp32 (4 columns per 16-byte vector)
  const int lane = threadIdx.x & 31;
  const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (w >= a.n_chunks) return;
  const RowChunk ch = a.chunks[w];
  const int64_t u = row_base + ch.row;
  const float* G = static_cast<const float*>(a.G);
  const T* DY = static_cast<const T*>(a.dy);
  int hd[NV];
  float gu[NV][EPV], elu[NV], acc[NV][EPV], dl[NV];
#pragma unroll
  for (int q = 0; q < NV; ++q) {
    const int vi = lane + 32 * q;
    hd[q] = vi < a.VPR ? (vi * EPV) / a.Fo : 0;
    if (vi < a.VPR) GV<float>::unpack(ld16(G + u * a.ldg + vi * EPV), gu[q]);
    else {
#pragma unroll
      for (int i = 0; i < EPV; ++i) gu[q][i] = 0.f;
    }
    elu[q] = a.el[u * a.H + hd[q]];
    dl[q] = 0.f;
#pragma unroll
    for (int i = 0; i < EPV; ++i) acc[q][i] = 0.f;
  }
  const float dys = a.concat ? 1.f : 1.f / (float)a.H;
  for (int64_t e = ch.e_lo; e < ch.e_hi; ++e) {
    const int64_t dd = a.idx[e];
    float dyv[NV][EPV], part[NV];
#pragma unroll
    for (int q = 0; q < NV; ++q) {
      const int vi = lane + 32 * q;
      part[q] = 0.f;
      if (vi < a.VPR) {
        const int c0 = vi * EPV;
        const int cc = a.concat ? c0 : (c0 % a.Fo);
#pragma unroll
        for (int i = 0; i < EPV; ++i) dyv[q][i] = (c0 + i < a.HF) ? (float)DY[dd * a.lddy + cc + i] : 0.f;
#pragma unroll
        for (int i = 0; i < EPV; ++i) {
          dyv[q][i] = (c0 + i < a.HF) ? dyv[q][i] * dys : 0.f;
          part[q] += dyv[q][i] * gu[q][i];
        }
      } else {
#pragma unroll
        for (int i = 0; i < EPV; ++i) dyv[q][i] = 0.f;
      }
    }
    // dalpha per head: segmented (by head) warp reduction
    float dal[NV];
#pragma unroll
    for (int q = 0; q < NV; ++q) dal[q] = 0.f;
    for (int h = 0; h < a.H; ++h) {
      float sh = 0.f;
#pragma unroll
      for (int q = 0; q < NV; ++q) if (hd[q] == h) sh += part[q];
#pragma unroll
      for (int o = 16; o; o >>= 1) sh += __shfl_xor_sync(0xffffffffu, sh, o);
#pragma unroll
      for (int q = 0; q < NV; ++q) if (hd[q] == h) dal[q] = sh;
    }
#pragma unroll
    for (int q = 0; q < NV; ++q) {
      const int vi = lane + 32 * q;
      const int h = hd[q];
      const float t = elu[q] + a.er[dd * a.H + h];
      const float alpha = __expf(lrelu(t, a.slope) - a.m[dd * a.H + h]) / a.l[dd * a.H + h];
      const float dtv = alpha * (dal[q] - a.s[dd * a.H + h]) * (t > 0.f ? 1.f : a.slope);
#pragma unroll
      for (int i = 0; i < EPV; ++i) acc[q][i] += alpha * dyv[q][i];
      if (vi < a.VPR && (vi * EPV) % a.Fo == 0) {
        dl[q] += dtv;
        a.dt[a.fwdpos[e] * a.H + h] = dtv;
      }
    }
  }
#pragma unroll
  for (int q = 0; q < NV; ++q) {
    const int vi = lane + 32 * q;
    if (vi >= a.VPR) continue;
    const int c0 = vi * EPV;
    float* out = ch.slot >= 0 ? a.part + (int64_t)ch.slot * a.part_ld : a.dg + u * a.ld_dg;
#pragma unroll
    for (int i = 0; i < EPV; ++i) out[c0 + i] = acc[q][i];
    if (c0 % a.Fo == 0) {
      if (ch.slot >= 0) out[a.HF + hd[q]] = dl[q];
      else a.del[u * a.H + hd[q]] = dl[q];
    }
  }
}

__global__ void k_gat_bwd_combine(GatArgs a, const SplitRow* rows, int64_t row_base) {
  const SplitRow sr = rows[blockIdx.x];
  const int64_t u = row_base + sr.row;
  for (int c = threadIdx.x; c < a.HF + a.H; c += blockDim.x) {
    float s = 0.f;
    for (int k = 0; k < sr.n_slots; ++k) s += a.part[(int64_t)(sr.first_slot + k) * a.part_ld + c];
    if (c < a.HF) a.dg[u * a.ld_dg + c] = s;
    else a.del[u * a.H + (c - a.HF)] = s;
  }
}

// der[v,h] = sum_{e in in(v)} dt_e (forward order: contiguous per row)
__global__ void k_gat_der(int64_t rows, int64_t row_base, const int64_t* row_ptr, const float* dt, int H, float* der) {
  const int lane = threadIdx.x & 31;
  const int64_t r = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (r >= rows) return;
  for (int h = 0; h < H; ++h) {
    float s = 0.f;
    for (int64_t e = row_ptr[r] + lane; e < row_ptr[r + 1]; e += 32) s += dt[e * H + h];
#pragma unroll
    for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) der[(row_base + r) * H + h] = s;
  }
}

// dG = dg + del a_l + der a_r (conv dtype, GEMM operand); da_l / da_r block partials
// dG is written as hi (+ lo residual for bf16: dG = hi + lo to ~16 mantissa
// bits) so the GEMMs that consume it keep the cancellation in dg + del a_l +
// der a_r accurate.
template <typename T>
__global__ void k_gat_dG(int64_t rows, int64_t row_base, GatArgs a, const float* al, const float* ar,
                         const float* der, T* dG, T* dGlo, int64_t ld_dG, float* part, int64_t rows_per_blk) {
  // thread per column c (HF <= 1024), rows of this block
  const int64_t r0 = blockIdx.x * rows_per_blk, r1 = min(rows, r0 + rows_per_blk);
  const float* G = static_cast<const float*>(a.G);
  for (int c = threadIdx.x; c < a.HF; c += blockDim.x) {
    const int h = c / a.Fo;
    float sl = 0.f, sr = 0.f;
    for (int64_t r = r0; r < r1; ++r) {
      const int64_t v = row_base + r;
      const float dlv = a.del[v * a.H + h], drv = der[v * a.H + h];
      const float val = a.dg[v * a.ld_dg + c] + dlv * al[c] + drv * ar[c];
      const T hi = (T)val;
      dG[r * ld_dG + c] = hi;
      if (dGlo) dGlo[r * ld_dG + c] = (T)(val - (float)hi);
      const float g = (float)G[v * a.ldg + c];
      sl += dlv * g;
      sr += drv * g;
    }
    part[(int64_t)blockIdx.x * 2 * a.HF + c] = sl;
    part[(int64_t)blockIdx.x * 2 * a.HF + a.HF + c] = sr;
  }
}

__global__ void k_pair_reduce(const float* part, int nblk, int n, float* out0, float* out1) {
  const int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= 2 * n) return;
  float s = 0.f;
  for (int b = 0; b < nblk; ++b) s += part[(int64_t)b * 2 * n + c];
  if (c < n) { if (out0) out0[c] = s; }
  else if (out1) out1[c - n] = s;
}

constexpr int DG_BLKS = 592;

template <typename T>
int nv_for(int VPR) { return VPR <= 32 ? 1 : (VPR <= 64 ? 2 : 4); }

}  // namespace

void gat_layout(wg_plan_s* p) {
  const wg_conv_desc& d = p->d;
  wg_graph_s* g = p->g;
  const int s = dsize(d.dtype), H = d.heads;
  const int64_t HF = (int64_t)H * d.f_out;
  p->pi = pitch(d.f_in, d.dtype);
  p->po = pitch(HF, d.dtype);
  auto* gp = new GatPlan();
  p->rg = nullptr;
  std::vector<RowChunk> cf, cb;
  std::vector<SplitRow> sf, sb;
  build_chunks(g->fwd, cf, sf, &gp->n_fslots);
  build_chunks(g->bwd, cb, sb, &gp->n_bslots);
  auto up = [&](const auto& v, auto** dptr) {
    using E = typename std::remove_reference<decltype(v)>::type::value_type;
    *dptr = nullptr;
    if (v.empty()) return;
    void* q = nullptr;
    cudaMalloc(&q, sizeof(E) * v.size());
    cudaMemcpy(q, v.data(), sizeof(E) * v.size(), cudaMemcpyHostToDevice);
    p->allocs.push_back(q);
    *dptr = static_cast<E*>(q);
  };
  up(cf, &gp->fwd); gp->n_fwd = (int)cf.size();
  up(cb, &gp->bwd); gp->n_bwd = (int)cb.size();
  up(sf, &gp->fsplit); gp->n_fsplit = (int)sf.size();
  up(sb, &gp->bsplit); gp->n_bsplit = (int)sb.size();
  p->gat = gp;
  const int64_t V = g->V, nr = g->ve - g->vb;
  Layout& S = p->saved;
  Layout& W = p->ws;
  S = Layout();
  W = Layout();
  // g = x W is kept in fp32 for both dtypes: the attention logits and the
  // ill-conditioned der / da_r sums (the softmax gradient cancels exactly
  // for LeakyReLU slope 1) need its full accumulator precision
  S.add("G", sizeof(float) * (size_t)V * pitch(HF, WG_F32));
  S.add("agg", sizeof(float) * (size_t)nr * rup(HF, 4));   // fp32: s = dy.agg feeds a cancellation (dt)
  S.add("el", sizeof(float) * V * H);
  S.add("er", sizeof(float) * V * H);
  S.add("m", sizeof(float) * V * H);
  S.add("l", sizeof(float) * V * H);
  W.add("wt", (size_t)rup(HF, 16) * p->pi * s);
  W.add("w", (size_t)rup(d.f_in, 16) * p->po * s);
  W.add("part", sizeof(float) * std::max(1, std::max(gp->n_fslots, gp->n_bslots)) * (HF + 2 * H + 8));
  W.add("dt", sizeof(float) * std::max<int64_t>(1, g->fwd.E) * H);
  W.add("s", sizeof(float) * V * H);
  W.add("del", sizeof(float) * V * H);
  W.add("der", sizeof(float) * V * H);
  W.add("dg", sizeof(float) * V * HF);
  W.add("dG", (size_t)nr * p->po * s);
  W.add("dGlo", (size_t)nr * p->po * s);
  W.add("dyt", (size_t)nr * p->po * s);
  W.add("colsum", bias_grad_scratch(nr, (int)HF));
  W.add("dgp", sizeof(float) * DG_BLKS * 2 * HF);
  W.add("tn", gemm_tn_scratch(nr, d.f_in, (int)HF));
}

void gat_plan_free(wg_plan_s* p) {
  delete static_cast<GatPlan*>(p->gat);
  p->gat = nullptr;
}

template <typename T>
static wg_status gat_fwd_t(wg_plan_s* p, const wg_params* P, const wg_fwd_args* A, cudaStream_t st) {
  const wg_conv_desc& d = p->d;
  wg_graph_s* g = p->g;
  auto* gp = static_cast<GatPlan*>(p->gat);
  const int H = d.heads, Fo = d.f_out, HF = H * Fo;
  constexpr int EPV = GV<T>::EPV;
  const int64_t V = g->V, nr = g->ve - g->vb, vb = g->vb;
  WG_REQ(nr == V, WG_ERR_UNSUPPORTED, "GAT with a 1-D partition is not implemented");
  WG_REQ(Fo % EPV == 0, WG_ERR_UNSUPPORTED, "GAT: per-head width must be a multiple of 16 bytes");
  WG_REQ(P->W && P->attn_l && P->attn_r, WG_ERR_INVALID, "GAT needs W, attn_l, attn_r");
  const Layout &S = p->saved, &L = p->ws;
  void* ws = A->workspace;
  const int s = dsize(d.dtype);
  GatArgs a{};
  a.H = H; a.Fo = Fo; a.HF = HF; a.VPR = (int)cdiv(HF, 4); a.slope = d.neg_slope;
  a.G = S.at<void>(A->saved, "G"); a.ldg = pitch(HF, WG_F32);
  a.el = S.at<float>(A->saved, "el"); a.er = S.at<float>(A->saved, "er");
  a.m = S.at<float>(A->saved, "m"); a.l = S.at<float>(A->saved, "l");
  a.agg = S.at<void>(A->saved, "agg"); a.ld_agg = rup(HF, 4);
  a.part = L.at<float>(ws, "part"); a.part_ld = HF + 2 * H + 8;
  a.concat = d.concat_heads;
  // G = x W  (vertex-level transform, tcgen05 for bf16; fp32 accumulator kept)
  void* wt = L.at<void>(ws, "wt");
  WG_TRY(prep_weight(d.dtype, P->W, d.f_in, HF, 1, wt, p->pi, (int)rup(HF, 16), st));
  {
    GemmPart part{A->x, A->ldx, wt, p->pi, d.f_in, (int)rup(HF, 16)};
    GemmEpi e;
    e.D = const_cast<void*>(a.G); e.ldd = a.ldg; e.d_f32 = 1;
    WG_TRY(gemm_nt(d.dtype, V, (int)rup(HF, 8), &part, 1, e, nullptr, 0, st));
  }
  const int NV = nv_for<float>(a.VPR);
  ProfScope ps(PK_GAT, st, (double)g->fwd.E * (HF * 4.0 + 4.0 * H + 4) + (double)V * HF * (4.0 + s) * 2, 0.0);
  const unsigned wb = (unsigned)cdiv(V * 32, 256);
  if (NV == 1) WG_LAUNCH((k_gat_logits<float, 1>), wb, 256, 0, st, V, a, P->attn_l, P->attn_r);
  else if (NV == 2) WG_LAUNCH((k_gat_logits<float, 2>), wb, 256, 0, st, V, a, P->attn_l, P->attn_r);
  else WG_LAUNCH((k_gat_logits<float, 4>), wb, 256, 0, st, V, a, P->attn_l, P->attn_r);
  a.idx = g->fwd.idx;
  a.chunks = gp->fwd; a.n_chunks = gp->n_fwd;
  if (gp->n_fwd) {
    const unsigned cbk = (unsigned)cdiv((int64_t)gp->n_fwd * 32, 256);
    if (NV == 1) WG_LAUNCH((k_gat_fwd<float, 1, 4>), cbk, 256, 0, st, a, vb);
    else if (NV == 2) WG_LAUNCH((k_gat_fwd<float, 2, 4>), cbk, 256, 0, st, a, vb);
    else WG_LAUNCH((k_gat_fwd<float, 4, 2>), cbk, 256, 0, st, a, vb);
  }
  if (gp->n_fsplit) WG_LAUNCH(k_gat_fwd_combine<float>, gp->n_fsplit, 128, 0, st, a, gp->fsplit, vb);
  const int FO = d.concat_heads ? HF : Fo;
  WG_LAUNCH(k_gat_out<T>, 1184, 256, 0, st, nr, a, d.bias ? P->bias : nullptr, d.fuse_relu, A->y, A->ldy, FO);
  return WG_OK;
}

template <typename T>
static wg_status gat_bwd_t(wg_plan_s* p, const wg_params* P, const wg_bwd_args* A, const wg_grads* Gr,
                           cudaStream_t st) {
  const wg_conv_desc& d = p->d;
  wg_graph_s* g = p->g;
  auto* gp = static_cast<GatPlan*>(p->gat);
  const int H = d.heads, Fo = d.f_out, HF = H * Fo;
  constexpr int EPV = GV<T>::EPV;
  const int64_t V = g->V, nr = g->ve - g->vb, vb = g->vb;
  WG_REQ(nr == V, WG_ERR_UNSUPPORTED, "GAT with a 1-D partition is not implemented");
  WG_REQ(g->fwdpos != nullptr || g->fwd.E == 0, WG_ERR_STATE, "GAT backward needs fwdpos");
  const Layout &S = p->saved, &L = p->ws;
  void* ws = A->workspace;
  const int s = dsize(d.dtype);
  const int FO = d.concat_heads ? HF : Fo;
  GatArgs a{};
  a.H = H; a.Fo = Fo; a.HF = HF; a.VPR = (int)cdiv(HF, 4); a.slope = d.neg_slope;
  a.G = S.at<void>(A->saved, "G"); a.ldg = pitch(HF, WG_F32);
  a.el = S.at<float>(A->saved, "el"); a.er = S.at<float>(A->saved, "er");
  a.m = S.at<float>(A->saved, "m"); a.l = S.at<float>(A->saved, "l");
  a.agg = S.at<void>(A->saved, "agg"); a.ld_agg = rup(HF, 4);
  a.part = L.at<float>(ws, "part"); a.part_ld = HF + 2 * H + 8;
  a.concat = d.concat_heads;
  (void)EPV;
  // dT = dy (masked by the fused ReLU) ; db
  const void* dT = A->dy;
  int64_t lddT = A->lddy;
  if (d.fuse_relu) { dT = L.at<void>(ws, "dyt"); lddT = p->po; }
  WG_TRY(bias_grad_mask(d.dtype, nr, FO, A->dy, A->lddy, d.fuse_relu ? A->y : nullptr, A->ldy,
                        d.fuse_relu ? const_cast<void*>(dT) : nullptr, lddT, Gr ? Gr->bias : nullptr,
                        L.at<float>(ws, "colsum"), st));
  a.dy = dT; a.lddy = lddT;
  float* sbuf = L.at<float>(ws, "s");
  a.s = sbuf;
  ProfScope ps(PK_GAT, st, (double)g->bwd.E * (FO * s + 16.0 * H + 12) + (double)V * HF * (s + 12), 0.0);
  WG_LAUNCH(k_gat_s<T>, (unsigned)cdiv(nr * 32, 256), 256, 0, st, nr, vb, a, sbuf);
  a.idx = g->bwd.idx;
  a.fwdpos = g->fwdpos;
  a.dt = L.at<float>(ws, "dt");
  a.dg = L.at<float>(ws, "dg"); a.ld_dg = HF;
  a.del = L.at<float>(ws, "del");
  a.chunks = gp->bwd; a.n_chunks = gp->n_bwd;
  const int NV = nv_for<float>(a.VPR);
  if (gp->n_bwd) {
    const unsigned cbk = (unsigned)cdiv((int64_t)gp->n_bwd * 32, 256);
    if (NV == 1) WG_LAUNCH((k_gat_bwd_src<T, 1>), cbk, 256, 0, st, a, vb);
    else if (NV == 2) WG_LAUNCH((k_gat_bwd_src<T, 2>), cbk, 256, 0, st, a, vb);
    else WG_LAUNCH((k_gat_bwd_src<T, 4>), cbk, 256, 0, st, a, vb);
  }
  // rows without out-edges have no chunk: their dg / del are zero
  // (chunks cover every row, including empty ones -- see build_chunks)
  if (gp->n_bsplit) WG_LAUNCH(k_gat_bwd_combine, gp->n_bsplit, 128, 0, st, a, gp->bsplit, vb);
  float* der = L.at<float>(ws, "der");
  WG_LAUNCH(k_gat_der, (unsigned)cdiv(nr * 32, 256), 256, 0, st, nr, vb, g->fwd.row_ptr, a.dt, H, der);
  void* dG = L.at<void>(ws, "dG");
  void* dGlo = d.dtype == WG_BF16 ? L.at<void>(ws, "dGlo") : nullptr;
  const int64_t rpb = std::max<int64_t>(1, cdiv(nr, DG_BLKS));
  const int nblk = (int)cdiv(nr, rpb);
  float* dgp = L.at<float>(ws, "dgp");
  WG_LAUNCH(k_gat_dG<T>, nblk, 256, 0, st, nr, vb, a, P->attn_l, P->attn_r, der, (T*)dG, (T*)dGlo, p->po, dgp,
            rpb);
  WG_LAUNCH(k_pair_reduce, (unsigned)cdiv(2 * HF, 128), 128, 0, st, dgp, nblk, HF, Gr ? Gr->attn_l : nullptr,
            Gr ? Gr->attn_r : nullptr);
  // dW = x^T dG ; dx = dG W^T   (dG = hi + lo for bf16)
  if (Gr && Gr->W) {
    WG_TRY(gemm_tn(d.dtype, nr, d.f_in, HF, A->x, A->ldx, dG, p->po, Gr->W, L.at<void>(ws, "tn"), st));
    if (dGlo) WG_TRY(gemm_tn(d.dtype, nr, d.f_in, HF, A->x, A->ldx, dGlo, p->po, Gr->W, L.at<void>(ws, "tn"), st, 1));
  }
  if (d.need_dx) {
    void* w = L.at<void>(ws, "w");
    WG_TRY(prep_weight(d.dtype, P->W, d.f_in, HF, 0, w, p->po, (int)rup(d.f_in, 16), st));
    GemmPart parts[2] = {GemmPart{dG, p->po, w, p->po, HF, (int)rup(d.f_in, 16)},
                         GemmPart{dGlo, p->po, w, p->po, HF, (int)rup(d.f_in, 16)}};
    GemmEpi e;
    e.D = A->dx; e.ldd = A->lddx;
    e.mask_ref = A->dx_mask; e.ld_mask = A->ld_dx_mask;
    WG_TRY(gemm_nt(d.dtype, nr, (int)rup(d.f_in, 16 / s), parts, dGlo ? 2 : 1, e, nullptr, 0, st));
  }
  return WG_OK;
}

wg_status gat_forward(wg_plan_s* p, const wg_params* P, const wg_fwd_args* a, cudaStream_t s) {
  WG_REQ(a->x && a->y && a->saved && a->workspace, WG_ERR_INVALID, "GAT forward: null buffer");
  return p->d.dtype == WG_BF16 ? gat_fwd_t<__nv_bfloat16>(p, P, a, s) : gat_fwd_t<float>(p, P, a, s);
}

wg_status gat_backward(wg_plan_s* p, const wg_params* P, const wg_bwd_args* a, const wg_grads* G, cudaStream_t s) {
  WG_REQ(a->dy && a->x && a->saved && a->workspace, WG_ERR_INVALID, "GAT backward: null buffer");
  WG_REQ(!p->d.fuse_relu || a->y, WG_ERR_INVALID, "fuse_relu backward needs y");
  return p->d.dtype == WG_BF16 ? gat_bwd_t<__nv_bfloat16>(p, P, a, G, s) : gat_bwd_t<float>(p, P, a, G, s);
}

}  // namespace wg
