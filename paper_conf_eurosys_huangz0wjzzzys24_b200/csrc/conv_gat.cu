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
  void* y; int64_t ldy; int FO;        // layer output (conv dtype): concat -> HF columns, mean -> Fo
  const float* bias; int relu;
  float* part; int part_ld;            // partial slots [slots x part_ld]: HF acc + H m + H l
  // backward
  const void* dy; int64_t lddy; int concat;
  const float4* bs;                    // [V x H] {er, m + log l, s, 0}: per-destination backward stats
  const int64_t* fwdpos;               // transposed position -> forward position
  float* dt;                           // [E x H] (forward order)
  float* dg; int64_t ld_dg;            // [V x HF] fp32 (sum alpha dy)
  float* del;                          // [V x H]
};

// ---------------------------------------------------------------- el / er
// One warp per vertex row of G (fp32): el[v,h] = g[v, head h] . a_l[h],
// er[v,h] = g[v, head h] . a_r[h].  a_l / a_r are read as float4 (one 16-byte
// load per G vector); SEG > 0: heads are aligned groups of SEG lanes (Fo / 4,
// a power of two <= 32), reduced by log2(SEG) xor-shuffles per vector, the
// group's first lane stores; SEG == 0: generic head loop over the warp.
template <typename T, int NV, int SEG>
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
      if (c0 + EPV <= a.HF) {
        const float4 l4 = __ldg(reinterpret_cast<const float4*>(al + c0));
        const float4 r4 = __ldg(reinterpret_cast<const float4*>(ar + c0));
        pl[q] = g[0] * l4.x + g[1] * l4.y + g[2] * l4.z + g[3] * l4.w;
        pr[q] = g[0] * r4.x + g[1] * r4.y + g[2] * r4.z + g[3] * r4.w;
      } else {
#pragma unroll
        for (int i = 0; i < EPV; ++i)
          if (c0 + i < a.HF) { pl[q] += g[i] * al[c0 + i]; pr[q] += g[i] * ar[c0 + i]; }
      }
    }
  }
  if constexpr (SEG > 0) {
#pragma unroll
    for (int q = 0; q < NV; ++q) {
      float sl = pl[q], sr = pr[q];
#pragma unroll
      for (int o = SEG / 2; o; o >>= 1) {
        sl += __shfl_xor_sync(0xffffffffu, sl, o);
        sr += __shfl_xor_sync(0xffffffffu, sr, o);
      }
      if ((lane & (SEG - 1)) == 0 && hd[q] >= 0 && hd[q] < a.H) {
        const_cast<float*>(a.el)[v * a.H + hd[q]] = sl;
        const_cast<float*>(a.er)[v * a.H + hd[q]] = sr;
      }
    }
  } else {
    for (int h = 0; h < a.H; ++h) {
      float sl = 0.f, sr = 0.f;
#pragma unroll
      for (int q = 0; q < NV; ++q) if (hd[q] == h) { sl += pl[q]; sr += pr[q]; }
#pragma unroll
      for (int o = 16; o; o >>= 1) { sl += __shfl_xor_sync(0xffffffffu, sl, o); sr += __shfl_xor_sync(0xffffffffu, sr, o); }
      if (lane == 0) { const_cast<float*>(a.el)[v * a.H + h] = sl; const_cast<float*>(a.er)[v * a.H + h] = sr; }
    }
  }
}

// y row of destination `row` from its per-head aggregate row `o` (fp32, HF
// values, shared memory): concat -> o + b, mean over heads -> mean_k o_k + b;
// optional ReLU; pad columns up to a multiple of 8 written as 0.  Threads
// t = 0..nt-1 of the caller each write 4 columns at a time.
template <typename TO>
__device__ __forceinline__ void gat_write_y(const GatArgs& a, int64_t row, const float* o, int t, int nt) {
  const int wcols = ((a.FO + 7) / 8) * 8;
  for (int c = 4 * t; c < wcols; c += 4 * nt) {
    float v[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      const int cc = c + i;
      float x = 0.f;
      if (cc < a.FO) {
        if (a.concat) x = o[cc];
        else {
          for (int h = 0; h < a.H; ++h) x += o[h * a.Fo + cc];
          x /= (float)a.H;
        }
        if (a.bias) x += a.bias[cc];
        if (a.relu) x = fmaxf(x, 0.f);
      }
      v[i] = x;
    }
    TO* yp = static_cast<TO*>(a.y) + row * a.ldy + c;
    if constexpr (sizeof(TO) == 4) {
      *reinterpret_cast<float4*>(yp) = make_float4(v[0], v[1], v[2], v[3]);
    } else {
      __nv_bfloat162 h0 = __floats2bfloat162_rn(v[0], v[1]), h1 = __floats2bfloat162_rn(v[2], v[3]);
      uint2 u;
      u.x = *reinterpret_cast<uint32_t*>(&h0);
      u.y = *reinterpret_cast<uint32_t*>(&h1);
      *reinterpret_cast<uint2*>(yp) = u;
    }
  }
}

// ------------------------------------------------- forward online softmax
// one warp per row chunk (destination row, in-edges [e_lo, e_hi))
template <typename T, typename TO, int NV, int U>
__global__ void __launch_bounds__(256) k_gat_fwd(GatArgs a, int64_t row_base) {
  constexpr int EPV = GV<T>::EPV;
  __shared__ float orow[8][NV * 32 * EPV];          // per-warp aggregate row (y epilogue)
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
      for (int i = 0; i < EPV; ++i) { ag[i] = o[i]; orow[threadIdx.x >> 5][c0 + i] = o[i]; }
      if (head_lead) { a.m[d * a.H + hd[q]] = m[q]; a.l[d * a.H + hd[q]] = l[q]; }
    }
  }
  if (ch.slot < 0) {                               // warp-uniform
    __syncwarp();
    gat_write_y<TO>(a, ch.row, orow[threadIdx.x >> 5], lane, 32);
  }
}

// Forward, chunked softmax: one warp per row chunk; the row's edges are taken
// 32 at a time -- lane k computes the logits of edge k for every head, the
// chunk max / exp run once per edge (not once per edge and feature), the
// accumulator is rescaled once per 32 edges, and the gather loop is a plain
// alpha-weighted row sum (alpha and source id broadcast through shared
// memory).  Same outputs as k_gat_fwd (agg, m, l, y / split partials).
constexpr int GAT_HM = 8;   // heads handled by k_gat_fwd2

template <typename T, typename TO, int NV, int U, int HM, int MINB = (HM <= 4 && NV == 2) ? 4 : 3>
__global__ void __launch_bounds__(256, MINB) k_gat_fwd2(GatArgs a, int64_t row_base) {
  constexpr int EPV = GV<T>::EPV;
  static_assert(EPV == 4, "G is fp32 (agg rows are stored as float4)");
  static_assert(HM <= GAT_HM, "heads");
  __shared__ float orow[8][NV * 32 * EPV];
  __shared__ float alp[8][32][HM + 1];       // p_e per head of the chunk's edges
  __shared__ int sid[8][32];                  // source ids of the chunk's edges
  __shared__ float hsc[8][3][HM];             // per head: rescale factor, m, l
  const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5;
  const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (w >= a.n_chunks) return;
  const RowChunk ch = a.chunks[w];
  const int64_t d = row_base + ch.row;
  const int H = a.H;
  const T* G = static_cast<const T*>(a.G);
  float erd[HM], m[HM], lp[HM];
#pragma unroll
  for (int h = 0; h < HM; ++h) {
    erd[h] = h < H ? a.er[d * H + h] : 0.f;
    m[h] = -INFINITY;
    lp[h] = 0.f;
  }
  int hd[NV];
  float acc[NV][EPV];
#pragma unroll
  for (int q = 0; q < NV; ++q) {
    const int vi = lane + 32 * q;
    hd[q] = vi < a.VPR ? min((vi * EPV) / a.Fo, HM - 1) : 0;
#pragma unroll
    for (int i = 0; i < EPV; ++i) acc[q][i] = 0.f;
  }
  for (int64_t base = ch.e_lo; base < ch.e_hi; base += 32) {
    const int n = (int)min((int64_t)32, ch.e_hi - base);
    int s = 0;
    float lg[HM];
    if (lane < n) {
      s = a.idx[base + lane];
#pragma unroll
      for (int h = 0; h < HM; ++h) lg[h] = h < H ? lrelu(a.el[(int64_t)s * H + h] + erd[h], a.slope) : -INFINITY;
    } else {
#pragma unroll
      for (int h = 0; h < HM; ++h) lg[h] = -INFINITY;
    }
    sid[wi][lane] = s;
#pragma unroll
    for (int h = 0; h < HM; ++h) {
      if (h >= H) break;
      float mc = lg[h];
#pragma unroll
      for (int o = 16; o; o >>= 1) mc = fmaxf(mc, __shfl_xor_sync(0xffffffffu, mc, o));
      const float mn = fmaxf(m[h], mc);
      const float sc = __expf(m[h] - mn);      // m = -inf on the first chunk: 0
      const float p = lane < n ? __expf(lg[h] - mn) : 0.f;
      lp[h] = lp[h] * sc + p;
      m[h] = mn;
      alp[wi][lane][h] = p;
      if (lane == 0) hsc[wi][0][h] = sc;
    }
    __syncwarp();
#pragma unroll
    for (int q = 0; q < NV; ++q) {
      const float f = hsc[wi][0][hd[q]];
#pragma unroll
      for (int i = 0; i < EPV; ++i) acc[q][i] *= f;
    }
    for (int j = 0; j < n; j += U) {
      int4 v[U][NV];
      float al[U][NV];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int k = j + u;
        const bool ok = k < n;
        const int sk = sid[wi][ok ? k : 0];
#pragma unroll
        for (int q = 0; q < NV; ++q) {
          const int vi = lane + 32 * q;
          v[u][q] = (ok && vi < a.VPR) ? ld16(G + (int64_t)sk * a.ldg + vi * EPV) : make_int4(0, 0, 0, 0);
          al[u][q] = ok ? alp[wi][k][hd[q]] : 0.f;
        }
      }
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int q = 0; q < NV; ++q) {
          float g[EPV];
          GV<T>::unpack(v[u][q], g);
#pragma unroll
          for (int i = 0; i < EPV; ++i) acc[q][i] += al[u][q] * g[i];
        }
    }
    __syncwarp();
  }
  // per-head denominators (lane partials -> warp sums); m / l to shared memory
#pragma unroll
  for (int h = 0; h < HM; ++h) {
    if (h >= H) break;
    float l = lp[h];
#pragma unroll
    for (int o = 16; o; o >>= 1) l += __shfl_xor_sync(0xffffffffu, l, o);
    if (lane == 0) { hsc[wi][1][h] = m[h]; hsc[wi][2][h] = l; }
  }
  __syncwarp();
  if (ch.slot >= 0) {
    float* pp = a.part + (int64_t)ch.slot * a.part_ld;
#pragma unroll
    for (int q = 0; q < NV; ++q) {
      const int vi = lane + 32 * q;
      if (vi >= a.VPR) continue;
#pragma unroll
      for (int i = 0; i < EPV; ++i) pp[vi * EPV + i] = acc[q][i];
    }
    if (lane < H) { pp[a.HF + lane] = hsc[wi][1][lane]; pp[a.HF + a.H + lane] = hsc[wi][2][lane]; }
    return;
  }
#pragma unroll
  for (int q = 0; q < NV; ++q) {
    const int vi = lane + 32 * q;
    if (vi >= a.VPR) continue;
    const int c0 = vi * EPV;
    const float l = hsc[wi][2][hd[q]];
    const float inv = l > 0.f ? 1.f / l : 0.f;
    float o[EPV];
#pragma unroll
    for (int i = 0; i < EPV; ++i) o[i] = (c0 + i < a.HF) ? acc[q][i] * inv : 0.f;
    float* ag = static_cast<float*>(a.agg) + (int64_t)ch.row * a.ld_agg + c0;
    *reinterpret_cast<float4*>(ag) = make_float4(o[0], o[1], o[2], o[3]);
#pragma unroll
    for (int i = 0; i < EPV; ++i) orow[wi][c0 + i] = o[i];
  }
  if (lane < H) { a.m[d * H + lane] = hsc[wi][1][lane]; a.l[d * H + lane] = hsc[wi][2][lane]; }
  __syncwarp();
  gat_write_y<TO>(a, ch.row, orow[wi], lane, 32);
}

// Forward, two row chunks per warp (one per half-warp, 16 lanes): the per-row
// softmax set-up (logit loads, per-head max / sum reductions, rescale, the
// epilogue) is issued once for two rows, which halves its instruction cost on
// the short rows that dominate power-law graphs (C2: mean in-degree 6.9).
// Adjacent chunks in the heavy-first order have similar lengths, so the two
// halves run nearly the same number of iterations.  Each half takes its
// row's edges 16 at a time; lane k of a half computes edge k's logits for
// every head; per-head reductions are xor-shuffles of offset < 16 (inside the
// half).  Same outputs as k_gat_fwd2.
template <typename T, typename TO, int NV2, int U, int HM, int MINB = (NV2 >= 4 ? 2 : 3)>
__global__ void __launch_bounds__(256, MINB) k_gat_fwd3(GatArgs a, int64_t row_base) {
  constexpr int EPV = GV<T>::EPV;
  static_assert(EPV == 4, "G is fp32");
  __shared__ float orow[8][2][NV2 * 16 * EPV];
  __shared__ float alp[8][2][16][HM + 1];
  __shared__ int sid[8][2][16];
  __shared__ float hsc[8][2][3][HM];
  const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5, half = lane >> 4, hl = lane & 15;
  const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t ci = 2 * w + half;
  if (2 * w >= a.n_chunks) return;
  const bool live = ci < a.n_chunks;
  const RowChunk ch = live ? a.chunks[ci] : RowChunk{0, -1, 0, 0};
  const int64_t d = row_base + ch.row;
  const int H = a.H;
  const T* G = static_cast<const T*>(a.G);
  float erd[HM], m[HM], lp[HM];
#pragma unroll
  for (int h = 0; h < HM; ++h) {
    erd[h] = (live && h < H) ? a.er[d * H + h] : 0.f;
    m[h] = -INFINITY;
    lp[h] = 0.f;
  }
  int hd[NV2];
  float acc[NV2][EPV];
#pragma unroll
  for (int q = 0; q < NV2; ++q) {
    const int vi = hl + 16 * q;
    hd[q] = vi < a.VPR ? min((vi * EPV) / a.Fo, HM - 1) : 0;
#pragma unroll
    for (int i = 0; i < EPV; ++i) acc[q][i] = 0.f;
  }
  const int64_t len = ch.e_hi - ch.e_lo;
  const int64_t len_o = __shfl_xor_sync(0xffffffffu, len, 16);
  const int64_t iters = (max(len, len_o) + 15) / 16;      // warp-uniform
  for (int64_t it = 0; it < iters; ++it) {
    const int64_t base = ch.e_lo + it * 16;
    const int n = (int)max((int64_t)0, min((int64_t)16, ch.e_hi - base));
    int s = 0;
    float lg[HM];
    if (hl < n) {
      s = a.idx[base + hl];
      if constexpr (HM == 4) {
        if (H == 4) {
          const float4 e4 = __ldg(reinterpret_cast<const float4*>(a.el + (int64_t)s * 4));
          lg[0] = lrelu(e4.x + erd[0], a.slope); lg[1] = lrelu(e4.y + erd[1], a.slope);
          lg[2] = lrelu(e4.z + erd[2], a.slope); lg[3] = lrelu(e4.w + erd[3], a.slope);
        } else {
#pragma unroll
          for (int h = 0; h < HM; ++h) lg[h] = h < H ? lrelu(a.el[(int64_t)s * H + h] + erd[h], a.slope) : -INFINITY;
        }
      } else {
#pragma unroll
        for (int h = 0; h < HM; ++h) lg[h] = h < H ? lrelu(a.el[(int64_t)s * H + h] + erd[h], a.slope) : -INFINITY;
      }
    } else {
#pragma unroll
      for (int h = 0; h < HM; ++h) lg[h] = -INFINITY;
    }
    sid[wi][half][hl] = s;
#pragma unroll
    for (int h = 0; h < HM; ++h) {
      if (h >= H) break;
      float mc = lg[h];
#pragma unroll
      for (int o = 8; o; o >>= 1) mc = fmaxf(mc, __shfl_xor_sync(0xffffffffu, mc, o));
      const float mn = fmaxf(m[h], mc);
      const float sc = (mn == -INFINITY) ? 1.f : __expf(m[h] - mn);
      const float pe = hl < n ? __expf(lg[h] - mn) : 0.f;
      lp[h] = lp[h] * sc + pe;
      m[h] = mn;
      alp[wi][half][hl][h] = pe;
      if (hl == 0) hsc[wi][half][0][h] = sc;
    }
    __syncwarp();
#pragma unroll
    for (int q = 0; q < NV2; ++q) {
      const float f = hsc[wi][half][0][hd[q]];
#pragma unroll
      for (int i = 0; i < EPV; ++i) acc[q][i] *= f;
    }
    const int n_o = __shfl_xor_sync(0xffffffffu, n, 16);
    const int nmax = max(n, n_o);
    for (int j = 0; j < nmax; j += U) {
      int4 v[U][NV2];
      float al[U][NV2];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int k = j + u;
        const bool ok = k < n;
        const int sk = sid[wi][half][ok ? k : 0];
#pragma unroll
        for (int q = 0; q < NV2; ++q) {
          const int vi = hl + 16 * q;
          v[u][q] = (ok && vi < a.VPR) ? ld16(G + (int64_t)sk * a.ldg + vi * EPV) : make_int4(0, 0, 0, 0);
          al[u][q] = ok ? alp[wi][half][k][hd[q]] : 0.f;
        }
      }
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int q = 0; q < NV2; ++q) {
          float g[EPV];
          GV<T>::unpack(v[u][q], g);
#pragma unroll
          for (int i = 0; i < EPV; ++i) acc[q][i] += al[u][q] * g[i];
        }
    }
    __syncwarp();
  }
#pragma unroll
  for (int h = 0; h < HM; ++h) {
    if (h >= H) break;
    float l = lp[h];
#pragma unroll
    for (int o = 8; o; o >>= 1) l += __shfl_xor_sync(0xffffffffu, l, o);
    if (hl == 0) { hsc[wi][half][1][h] = m[h]; hsc[wi][half][2][h] = l; }
  }
  __syncwarp();
  if (!live) return;
  if (ch.slot >= 0) {
    float* pp = a.part + (int64_t)ch.slot * a.part_ld;
#pragma unroll
    for (int q = 0; q < NV2; ++q) {
      const int vi = hl + 16 * q;
      if (vi >= a.VPR) continue;
#pragma unroll
      for (int i = 0; i < EPV; ++i) pp[vi * EPV + i] = acc[q][i];
    }
    if (hl < H) { pp[a.HF + hl] = hsc[wi][half][1][hl]; pp[a.HF + a.H + hl] = hsc[wi][half][2][hl]; }
    return;
  }
#pragma unroll
  for (int q = 0; q < NV2; ++q) {
    const int vi = hl + 16 * q;
    if (vi >= a.VPR) continue;
    const int c0 = vi * EPV;
    const float l = hsc[wi][half][2][hd[q]];
    const float inv = l > 0.f ? 1.f / l : 0.f;
    float o[EPV];
#pragma unroll
    for (int i = 0; i < EPV; ++i) o[i] = (c0 + i < a.HF) ? acc[q][i] * inv : 0.f;
    float* ag = static_cast<float*>(a.agg) + (int64_t)ch.row * a.ld_agg + c0;
    *reinterpret_cast<float4*>(ag) = make_float4(o[0], o[1], o[2], o[3]);
#pragma unroll
    for (int i = 0; i < EPV; ++i) orow[wi][half][c0 + i] = o[i];
  }
  if (hl < H) { a.m[d * H + hl] = hsc[wi][half][1][hl]; a.l[d * H + hl] = hsc[wi][half][2][hl]; }
  __syncwarp(0xffffu << (16 * half));
  gat_write_y<TO>(a, ch.row, orow[wi][half], hl, 16);
}

// flash-style merge of the (m, l, acc) partials of split rows:
// M = max_k m_k, then l = sum_k l_k e^{m_k - M}, o = sum_k acc_k e^{m_k - M};
// writes agg, m, l and the y row.  The 8 warps of the CTA take slots
// k = w, w + 8, ... (two independent slots in flight per lane) and their
// sums are added in warp order (fixed order: deterministic); one thread per
// column walking every slot was a serial latency chain (~50 us per launch).
constexpr int CMB_HMAX = 128;   // heads <= HF / 4 <= 128
template <typename TO>
__global__ void __launch_bounds__(256) k_gat_fwd_combine(GatArgs a, const SplitRow* rows, int64_t row_base) {
  __shared__ float Mw[8][CMB_HMAX];
  __shared__ float Mg[CMB_HMAX];
  __shared__ __align__(16) float red[8][512 + CMB_HMAX];
  __shared__ __align__(16) float orow[512];
  const SplitRow sr = rows[blockIdx.x];
  const int64_t d = row_base + sr.row;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int H = a.H, HF = a.HF, VPR = HF / 4;
  const float* p0 = a.part + (int64_t)sr.first_slot * a.part_ld;
  // pass 1: per-head maxima over the slots with l > 0
  for (int h = lane; h < H; h += 32) {
    float M = -INFINITY;
#pragma unroll 4
    for (int k = w; k < sr.n_slots; k += 8) {    // independent loads (max is order-free)
      const float* pp = p0 + (int64_t)k * a.part_ld;
      const float lk = pp[HF + H + h], mk = pp[HF + h];
      if (lk > 0.f) M = fmaxf(M, mk);
    }
    Mw[w][h] = M;
  }
  __syncthreads();
  for (int h = threadIdx.x; h < H; h += blockDim.x) {
    float M = Mw[0][h];
#pragma unroll
    for (int j = 1; j < 8; ++j) M = fmaxf(M, Mw[j][h]);
    Mg[h] = M;
  }
  __syncthreads();
  // pass 2: this warp's rescaled sums (lane: float4 columns lane, lane + 32, ...)
  float4 o[4];
  float lh[4];
#pragma unroll
  for (int q = 0; q < 4; ++q) { o[q] = make_float4(0.f, 0.f, 0.f, 0.f); lh[q] = 0.f; }
#pragma unroll 2
  for (int k = w; k < sr.n_slots; k += 8) {
    const float* pp = p0 + (int64_t)k * a.part_ld;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int vi = lane + 32 * q;
      if (vi < VPR) {
        const int h = (4 * vi) / a.Fo;
        const float lk = pp[HF + H + h];
        const float sc = lk > 0.f ? __expf(pp[HF + h] - Mg[h]) : 0.f;
        const float4 v = *reinterpret_cast<const float4*>(pp + 4 * vi);
        o[q].x += v.x * sc; o[q].y += v.y * sc; o[q].z += v.z * sc; o[q].w += v.w * sc;
      }
      const int h = lane + 32 * q;
      if (h < H) {
        const float lk = pp[HF + H + h];
        if (lk > 0.f) lh[q] += lk * __expf(pp[HF + h] - Mg[h]);
      }
    }
  }
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const int vi = lane + 32 * q;
    if (vi < VPR) *reinterpret_cast<float4*>(&red[w][4 * vi]) = o[q];
    if (lane + 32 * q < H) red[w][512 + lane + 32 * q] = lh[q];
  }
  __syncthreads();
  for (int c = threadIdx.x; c < HF; c += blockDim.x) {
    const int h = c / a.Fo;
    float oc = 0.f, l = 0.f;
#pragma unroll
    for (int j = 0; j < 8; ++j) { oc += red[j][c]; l += red[j][512 + h]; }
    const float val = l > 0.f ? oc / l : 0.f;
    static_cast<float*>(a.agg)[(int64_t)sr.row * a.ld_agg + c] = val;
    orow[c] = val;
    if (c % a.Fo == 0) { a.m[d * H + h] = Mg[h]; a.l[d * H + h] = l; }
  }
  __syncthreads();
  gat_write_y<TO>(a, sr.row, orow, threadIdx.x, blockDim.x);
}

// dy columns [c, c+4) of destination row dd as fp32 (16-byte or 8-byte load)
template <typename T> __device__ __forceinline__ void ld_dy4(const T* p, float* f);
template <> __device__ __forceinline__ void ld_dy4<float>(const float* p, float* f) {
  const int4 v = ld16(p);
  f[0] = __int_as_float(v.x); f[1] = __int_as_float(v.y); f[2] = __int_as_float(v.z); f[3] = __int_as_float(v.w);
}
template <> __device__ __forceinline__ void ld_dy4<__nv_bfloat16>(const __nv_bfloat16* p, float* f) {
  const uint2 v = __ldg(reinterpret_cast<const uint2*>(p));
  f[0] = __uint_as_float(v.x << 16); f[1] = __uint_as_float(v.x & 0xffff0000u);
  f[2] = __uint_as_float(v.y << 16); f[3] = __uint_as_float(v.y & 0xffff0000u);
}

// per-head sum of a lane value: SEG > 0: heads are aligned groups of SEG
// lanes (SEG = Fo / 4, a power of two <= 32); SEG == 0: generic (any Fo)
template <int NV, int SEG>
__device__ __forceinline__ void head_sums(const float* part, const int* hd, int H, float* out) {
  if constexpr (SEG > 0) {
#pragma unroll
    for (int q = 0; q < NV; ++q) {
      float v = part[q];
#pragma unroll
      for (int o = SEG / 2; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
      out[q] = v;
    }
  } else {
#pragma unroll
    for (int q = 0; q < NV; ++q) out[q] = 0.f;
    for (int h = 0; h < H; ++h) {
      float sh = 0.f;
#pragma unroll
      for (int q = 0; q < NV; ++q) if (hd[q] == h) sh += part[q];
#pragma unroll
      for (int o = 16; o; o >>= 1) sh += __shfl_xor_sync(0xffffffffu, sh, o);
#pragma unroll
      for (int q = 0; q < NV; ++q) if (hd[q] == h) out[q] = sh;
    }
  }
}

// Source-major backward pass, U out-edges in flight per warp: per out-edge e
// = (u -> dd): dalpha = dy_k[dd] . g_k[u], alpha = exp(lrelu(t) - lse[dd]),
// dt_e = alpha (dalpha - s[dd]) lrelu'(t); dg[u] += alpha dy_k[dd]; del[u] += dt_e.
template <typename T, int NV, int U, int SEG>
__global__ void __launch_bounds__(256, 2) k_gat_bwd_src2(GatArgs a, int64_t row_base) {
  constexpr int EPV = 4;                       // G is fp32: 4 columns per 16-byte vector
  const int lane = threadIdx.x & 31;
  const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (w >= a.n_chunks) return;
  const RowChunk ch = a.chunks[w];
  const int64_t u = row_base + ch.row;
  const float* G = static_cast<const float*>(a.G);
  const T* DY = static_cast<const T*>(a.dy);
  int hd[NV], cc[NV];
  bool on[NV], lead[NV];
  float gu[NV][EPV], elu[NV], acc[NV][EPV], dl[NV];
  const float dys = a.concat ? 1.f : 1.f / (float)a.H;
#pragma unroll
  for (int q = 0; q < NV; ++q) {
    const int vi = lane + 32 * q;
    on[q] = vi < a.VPR;
    const int c0 = vi * EPV;
    hd[q] = on[q] ? c0 / a.Fo : 0;
    cc[q] = a.concat ? c0 : c0 % a.Fo;
    lead[q] = on[q] && (c0 % a.Fo) == 0;
    if (on[q]) GV<float>::unpack(ld16(G + u * a.ldg + c0), gu[q]);
    else {
#pragma unroll
      for (int i = 0; i < EPV; ++i) gu[q][i] = 0.f;
    }
    elu[q] = a.el[u * a.H + hd[q]];
    dl[q] = 0.f;
#pragma unroll
    for (int i = 0; i < EPV; ++i) acc[q][i] = 0.f;
  }
  for (int64_t base = ch.e_lo; base < ch.e_hi; base += 32) {
    const int n = (int)min((int64_t)32, ch.e_hi - base);
    const int my = lane < n ? a.idx[base + lane] : 0;
    const int64_t myp = lane < n ? a.fwdpos[base + lane] : 0;
    for (int j = 0; j < n; j += U) {
      float dyv[U][NV][EPV];
      float4 st[U][NV];
#pragma unroll
      for (int k = 0; k < U; ++k) {
        const int64_t dd = __shfl_sync(0xffffffffu, my, j + k < n ? j + k : 0);
#pragma unroll
        for (int q = 0; q < NV; ++q) {
          if (on[q] && j + k < n) {
            ld_dy4<T>(DY + dd * a.lddy + cc[q], dyv[k][q]);
            st[k][q] = __ldg(a.bs + dd * a.H + hd[q]);
          } else {
#pragma unroll
            for (int i = 0; i < EPV; ++i) dyv[k][q][i] = 0.f;
            st[k][q] = make_float4(0.f, 0.f, 0.f, 0.f);
          }
        }
      }
#pragma unroll
      for (int k = 0; k < U; ++k) {
        if (j + k >= n) break;                 // warp-uniform
        float part[NV], dal[NV];
#pragma unroll
        for (int q = 0; q < NV; ++q) {
          part[q] = 0.f;
#pragma unroll
          for (int i = 0; i < EPV; ++i) {
            dyv[k][q][i] *= dys;
            part[q] += dyv[k][q][i] * gu[q][i];
          }
        }
        head_sums<NV, SEG>(part, hd, a.H, dal);
        const int64_t fp = __shfl_sync(0xffffffffu, myp, j + k);
#pragma unroll
        for (int q = 0; q < NV; ++q) {
          const float t = elu[q] + st[k][q].x;
          const float alpha = __expf(lrelu(t, a.slope) - st[k][q].y);
          const float dtv = alpha * (dal[q] - st[k][q].z) * (t > 0.f ? 1.f : a.slope);
#pragma unroll
          for (int i = 0; i < EPV; ++i) acc[q][i] += alpha * dyv[k][q][i];
          if (lead[q]) {
            dl[q] += dtv;
            a.dt[fp * a.H + hd[q]] = dtv;
          }
        }
      }
    }
  }
#pragma unroll
  for (int q = 0; q < NV; ++q) {
    if (!on[q]) continue;
    const int c0 = (lane + 32 * q) * EPV;
    float* out = ch.slot >= 0 ? a.part + (int64_t)ch.slot * a.part_ld : a.dg + u * a.ld_dg;
    *reinterpret_cast<float4*>(out + c0) = make_float4(acc[q][0], acc[q][1], acc[q][2], acc[q][3]);
    if (lead[q]) {
      if (ch.slot >= 0) out[a.HF + hd[q]] = dl[q];
      else a.del[u * a.H + hd[q]] = dl[q];
    }
  }
}

// Source-major backward pass, per-edge pre-pass: for each 32-edge chunk of the
// source row, lane k evaluates edge k's per-head terms once (alpha_e,
// alpha_e * lrelu'(t_e), s[dd]) into shared memory; the gather loop then only
// reads dy rows, forms the per-head dot products and accumulates.  The
// head-mean factor (last layer) is folded into g[u] and applied to dg once.
// Same outputs as k_gat_bwd_src2 (dg, del, dt_e, split partials).
template <typename T, int NV, int U, int SEG, int HM, int MINB = 2>
__global__ void __launch_bounds__(256, MINB) k_gat_bwd_src3(GatArgs a, int64_t row_base) {
  constexpr int EPV = 4;                       // G is fp32: 4 columns per 16-byte vector
  __shared__ float e_al[8][32][HM + 1];        // alpha_e per head
  __shared__ float e_af[8][32][HM + 1];        // alpha_e * lrelu'(t_e)
  __shared__ float e_s[8][32][HM + 1];         // s[dd] per head
  __shared__ int e_dd[8][32];
  __shared__ int64_t e_fp[8][32];
  const int lane = threadIdx.x & 31, wi = threadIdx.x >> 5;
  const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (w >= a.n_chunks) return;
  const RowChunk ch = a.chunks[w];
  const int64_t u = row_base + ch.row;
  const int H = a.H;
  const float* G = static_cast<const float*>(a.G);
  const T* DY = static_cast<const T*>(a.dy);
  int hd[NV], cc[NV];
  bool on[NV], lead[NV];
  float gu[NV][EPV], acc[NV][EPV], dl[NV], elu[HM];
  const float dys = a.concat ? 1.f : 1.f / (float)a.H;
#pragma unroll
  for (int h = 0; h < HM; ++h) elu[h] = h < H ? a.el[u * H + h] : 0.f;
#pragma unroll
  for (int q = 0; q < NV; ++q) {
    const int vi = lane + 32 * q;
    on[q] = vi < a.VPR;
    const int c0 = vi * EPV;
    hd[q] = on[q] ? min(c0 / a.Fo, HM - 1) : 0;
    cc[q] = a.concat ? c0 : c0 % a.Fo;
    lead[q] = on[q] && (c0 % a.Fo) == 0;
    if (on[q]) GV<float>::unpack(ld16(G + u * a.ldg + c0), gu[q]);
    else {
#pragma unroll
      for (int i = 0; i < EPV; ++i) gu[q][i] = 0.f;
    }
#pragma unroll
    for (int i = 0; i < EPV; ++i) { gu[q][i] *= dys; acc[q][i] = 0.f; }
    dl[q] = 0.f;
  }
  for (int64_t base = ch.e_lo; base < ch.e_hi; base += 32) {
    const int n = (int)min((int64_t)32, ch.e_hi - base);
    int dd = 0;
    int64_t fp = 0;
    if (lane < n) {
      dd = a.idx[base + lane];
      fp = a.fwdpos[base + lane];
#pragma unroll
      for (int h = 0; h < HM; ++h) {
        if (h >= H) break;
        const float4 st = __ldg(a.bs + (int64_t)dd * H + h);
        const float t = elu[h] + st.x;
        const float al = __expf(lrelu(t, a.slope) - st.y);
        e_al[wi][lane][h] = al;
        e_af[wi][lane][h] = al * (t > 0.f ? 1.f : a.slope);
        e_s[wi][lane][h] = st.z;
      }
    }
    e_dd[wi][lane] = dd;
    e_fp[wi][lane] = fp;
    __syncwarp();
    for (int j = 0; j < n; j += U) {
      float dyv[U][NV][EPV];
#pragma unroll
      for (int k = 0; k < U; ++k) {
        const bool ok = j + k < n;
        const int64_t ddk = e_dd[wi][ok ? j + k : 0];
#pragma unroll
        for (int q = 0; q < NV; ++q) {
          if (on[q] && ok) ld_dy4<T>(DY + ddk * a.lddy + cc[q], dyv[k][q]);
          else {
#pragma unroll
            for (int i = 0; i < EPV; ++i) dyv[k][q][i] = 0.f;
          }
        }
      }
#pragma unroll
      for (int k = 0; k < U; ++k) {
        if (j + k >= n) break;                 // warp-uniform
        float part[NV], dal[NV];
#pragma unroll
        for (int q = 0; q < NV; ++q) {
          part[q] = 0.f;
#pragma unroll
          for (int i = 0; i < EPV; ++i) part[q] += dyv[k][q][i] * gu[q][i];
        }
        head_sums<NV, SEG>(part, hd, a.H, dal);
#pragma unroll
        for (int q = 0; q < NV; ++q) {
          const float al = e_al[wi][j + k][hd[q]];
#pragma unroll
          for (int i = 0; i < EPV; ++i) acc[q][i] += al * dyv[k][q][i];
          if (lead[q]) {
            const float dtv = e_af[wi][j + k][hd[q]] * (dal[q] - e_s[wi][j + k][hd[q]]);
            dl[q] += dtv;
            a.dt[e_fp[wi][j + k] * a.H + hd[q]] = dtv;
          }
        }
      }
    }
    __syncwarp();
  }
#pragma unroll
  for (int q = 0; q < NV; ++q) {
    if (!on[q]) continue;
    const int c0 = (lane + 32 * q) * EPV;
    float* out = ch.slot >= 0 ? a.part + (int64_t)ch.slot * a.part_ld : a.dg + u * a.ld_dg;
    *reinterpret_cast<float4*>(out + c0) =
        make_float4(acc[q][0] * dys, acc[q][1] * dys, acc[q][2] * dys, acc[q][3] * dys);
    if (lead[q]) {
      if (ch.slot >= 0) out[a.HF + hd[q]] = dl[q];
      else a.del[u * a.H + hd[q]] = dl[q];
    }
  }
}

// per destination row and head: s = dy_k . agg_k (fp32 agg), and the packed
// backward stats bs = {er, m + log l, s, 0}
template <typename T, int NV, int SEG>
__global__ void __launch_bounds__(256) k_gat_s2(int64_t rows, int64_t row_base, GatArgs a, float4* bs) {
  constexpr int EPV = 4;
  const int lane = threadIdx.x & 31;
  const int64_t r = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (r >= rows) return;
  const int64_t v = row_base + r;
  const float* ag = static_cast<const float*>(a.agg) + r * a.ld_agg;
  const T* dy = static_cast<const T*>(a.dy) + r * a.lddy;
  const float dys = a.concat ? 1.f : 1.f / (float)a.H;
  float part[NV], sums[NV];
  int hd[NV];
  bool lead[NV];
#pragma unroll
  for (int q = 0; q < NV; ++q) {
    const int vi = lane + 32 * q;
    const int c0 = vi * EPV;
    part[q] = 0.f;
    hd[q] = vi < a.VPR ? c0 / a.Fo : 0;
    lead[q] = vi < a.VPR && (c0 % a.Fo) == 0;
    if (vi < a.VPR) {
      float g[EPV], d[EPV];
      GV<float>::unpack(ld16(ag + c0), g);
      ld_dy4<T>(dy + (a.concat ? c0 : c0 % a.Fo), d);
#pragma unroll
      for (int i = 0; i < EPV; ++i) part[q] += d[i] * dys * g[i];
    }
  }
  head_sums<NV, SEG>(part, hd, a.H, sums);
#pragma unroll
  for (int q = 0; q < NV; ++q) {
    if (!lead[q]) continue;
    const int64_t k = v * a.H + hd[q];
    const float l = a.l[k];
    bs[k] = make_float4(a.er[k], l > 0.f ? a.m[k] + __logf(l) : 0.f, sums[q], 0.f);
  }
}

// der over the forward row chunks (<= GAT_CHUNK edges each, SPLIT rows cut
// into several): eight lanes per chunk, four independent loads in flight per
// lane, fixed-order reduction; SPLIT chunks leave H partials in their slot,
// summed in chunk order by k_gat_der_combine
template <int H>
__global__ void k_gat_der3(const RowChunk* chunks, int n, int64_t row_base, const float* dt, float* der,
                           float* part, int part_ld) {
  const int sub = threadIdx.x & 7;
  const int64_t c = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 3;
  float s[H];
#pragma unroll
  for (int h = 0; h < H; ++h) s[h] = 0.f;
  RowChunk ch{};
  if (c < n) {
    ch = chunks[c];
    auto add = [&](int64_t e) {
      if constexpr (H == 4) {
        const float4 v = __ldg(reinterpret_cast<const float4*>(dt) + e);
        s[0] += v.x; s[1] += v.y; s[2] += v.z; s[3] += v.w;
      } else {
#pragma unroll
        for (int h = 0; h < H; ++h) s[h] += dt[e * H + h];
      }
    };
    int64_t e = ch.e_lo + sub;
    for (; e + 24 < ch.e_hi; e += 32) {
      if constexpr (H == 4) {
        const float4 v0 = __ldg(reinterpret_cast<const float4*>(dt) + e);
        const float4 v1 = __ldg(reinterpret_cast<const float4*>(dt) + e + 8);
        const float4 v2 = __ldg(reinterpret_cast<const float4*>(dt) + e + 16);
        const float4 v3 = __ldg(reinterpret_cast<const float4*>(dt) + e + 24);
        s[0] += v0.x; s[1] += v0.y; s[2] += v0.z; s[3] += v0.w;
        s[0] += v1.x; s[1] += v1.y; s[2] += v1.z; s[3] += v1.w;
        s[0] += v2.x; s[1] += v2.y; s[2] += v2.z; s[3] += v2.w;
        s[0] += v3.x; s[1] += v3.y; s[2] += v3.z; s[3] += v3.w;
      } else {
        add(e); add(e + 8); add(e + 16); add(e + 24);
      }
    }
    for (; e < ch.e_hi; e += 8) add(e);
  }
#pragma unroll
  for (int h = 0; h < H; ++h) {
#pragma unroll
    for (int o = 4; o; o >>= 1) s[h] += __shfl_xor_sync(0xffffffffu, s[h], o);
  }
  if (c < n && sub < H) {
    float o = s[0];
#pragma unroll
    for (int h = 1; h < H; ++h) if (sub == h) o = s[h];
    if (ch.slot >= 0) part[(int64_t)ch.slot * part_ld + sub] = o;
    else der[(row_base + ch.row) * H + sub] = o;
  }
}

// split-row sums of the slot partials: one warp per (row, column group) --
// lane j sums slots j, j + 32, ... then a fixed xor tree (deterministic)
__global__ void k_gat_der_combine(const SplitRow* rows, int n, int64_t row_base, const float* part, int part_ld,
                                  int H, float* der) {
  const int lane = threadIdx.x & 31;
  const int64_t t = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  if (t >= (int64_t)n * H) return;
  const SplitRow sr = rows[t / H];
  const int h = (int)(t % H);
  float s = 0.f;
#pragma unroll 4
  for (int k = lane; k < sr.n_slots; k += 32) s += part[(int64_t)(sr.first_slot + k) * part_ld + h];
#pragma unroll
  for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if (lane == 0) der[(row_base + sr.row) * H + h] = s;
}

// dg / del of a split source row: the 8 warps take slots w, w + 8, ...
// (float4 columns per lane), summed in warp order
__global__ void __launch_bounds__(256) k_gat_bwd_combine(GatArgs a, const SplitRow* rows, int64_t row_base) {
  __shared__ __align__(16) float red[8][512 + CMB_HMAX];
  const SplitRow sr = rows[blockIdx.x];
  const int64_t u = row_base + sr.row;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int HF = a.HF, NC = (HF + a.H + 3) / 4;   // float4 columns of a slot (acc then del)
  float4 o[5];
#pragma unroll
  for (int q = 0; q < 5; ++q) o[q] = make_float4(0.f, 0.f, 0.f, 0.f);
  for (int k = w; k < sr.n_slots; k += 8) {
    const float4* pp = reinterpret_cast<const float4*>(a.part + (int64_t)(sr.first_slot + k) * a.part_ld);
#pragma unroll
    for (int q = 0; q < 5; ++q) {
      const int vi = lane + 32 * q;
      if (vi < NC) {
        const float4 v = pp[vi];
        o[q].x += v.x; o[q].y += v.y; o[q].z += v.z; o[q].w += v.w;
      }
    }
  }
#pragma unroll
  for (int q = 0; q < 5; ++q) {
    const int vi = lane + 32 * q;
    if (vi < NC) *reinterpret_cast<float4*>(&red[w][4 * vi]) = o[q];
  }
  __syncthreads();
  for (int c = threadIdx.x; c < HF + a.H; c += blockDim.x) {
    float sum = 0.f;
#pragma unroll
    for (int j = 0; j < 8; ++j) sum += red[j][c];
    if (c < HF) a.dg[u * a.ld_dg + c] = sum;
    else a.del[u * a.H + (c - HF)] = sum;
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
  // thread per column c (HF <= 1024), rows of this block, 4 rows in flight
  constexpr int RB = 4;
  const int64_t r0 = blockIdx.x * rows_per_blk, r1 = min(rows, r0 + rows_per_blk);
  const float* G = static_cast<const float*>(a.G);
  for (int c = threadIdx.x; c < a.HF; c += blockDim.x) {
    const int h = c / a.Fo;
    const float alc = al[c], arc = ar[c];
    float sl = 0.f, sr = 0.f;
    for (int64_t rb = r0; rb < r1; rb += RB) {
      float dlv[RB], drv[RB], dgv[RB], gv[RB];
#pragma unroll
      for (int i = 0; i < RB; ++i) {
        const int64_t v = row_base + min(rb + i, r1 - 1);
        dlv[i] = a.del[v * a.H + h];
        drv[i] = der[v * a.H + h];
        dgv[i] = a.dg[v * a.ld_dg + c];
        gv[i] = G[v * a.ldg + c];
      }
#pragma unroll
      for (int i = 0; i < RB; ++i) {
        if (rb + i >= r1) break;
        const int64_t r = rb + i;
        const float val = dgv[i] + dlv[i] * alc + drv[i] * arc;
        const T hi = (T)val;
        dG[r * ld_dG + c] = hi;
        if (dGlo) dGlo[r * ld_dG + c] = (T)(val - (float)hi);
        sl += dlv[i] * gv[i];
        sr += drv[i] * gv[i];
      }
    }
    part[(int64_t)blockIdx.x * 2 * a.HF + c] = sl;
    part[(int64_t)blockIdx.x * 2 * a.HF + a.HF + c] = sr;
  }
}

// out0 / out1 = column sums of the [nblk x 2n] block partials (first / second
// half): 32 columns per CTA, fixed-order warp split as k_colsum_reduce
__global__ void __launch_bounds__(1024) k_pair_reduce(const float* part, int nblk, int n, float* out0, float* out1) {
  __shared__ float red[32][33];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int c = blockIdx.x * 32 + lane;
  float s = 0.f;
  if (c < 2 * n) {
#pragma unroll 4
    for (int b = warp; b < nblk; b += 32) s += part[(int64_t)b * 2 * n + c];
  }
  red[warp][lane] = s;
  __syncthreads();
  if (warp == 0 && c < 2 * n) {
    float t = 0.f;
#pragma unroll
    for (int w = 0; w < 32; ++w) t += red[w][lane];
    if (c < n) { if (out0) out0[c] = t; }
    else if (out1) out1[c - n] = t;
  }
}

constexpr int DG_BLKS = 592;

unsigned gs_grid(int64_t threads) { return (unsigned)std::max<int64_t>(1, cdiv(threads, 256)); }

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
  W.add("part", sizeof(float) * std::max(1, std::max(gp->n_fslots, gp->n_bslots)) * rup(HF + 2 * H + 8, 4));
  W.add("dt", sizeof(float) * std::max<int64_t>(1, g->fwd.E) * H);
  W.add("bs", sizeof(float4) * V * H);
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
  WG_REQ(HF <= 512, WG_ERR_UNSUPPORTED, "GAT: heads * f_out must be <= 512");
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
  a.part = L.at<float>(ws, "part"); a.part_ld = (int)rup(HF + 2 * H + 8, 4);   // 16-byte rows (float4 partial stores)
  a.concat = d.concat_heads;
  a.y = A->y; a.ldy = A->ldy; a.FO = d.concat_heads ? HF : Fo;
  a.bias = d.bias ? P->bias : nullptr; a.relu = d.fuse_relu;
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
  // algorithmic bytes: logits (G row), per edge the gathered G row + el + index,
  // per row the aggregate (saved) and y
  ProfScope ps(PK_GAT, st,
               (double)g->fwd.E * (HF * 4.0 + 4.0 * H + 4) + (double)V * HF * 8.0 + (double)V * a.FO * s, 0.0);
  const unsigned wb = gs_grid(V * 32);
  {
    const int vph = d.f_out / 4;             // fp32 G vectors per head
    const int SEG = (vph == 4 || vph == 8 || vph == 16 || vph == 32) ? vph : 0;
#define WG_GAT_L(NV_)                                                                                      \
  do {                                                                                                     \
    if (SEG == 4) WG_LAUNCH((k_gat_logits<float, NV_, 4>), wb, 256, 0, st, V, a, P->attn_l, P->attn_r);    \
    else if (SEG == 8) WG_LAUNCH((k_gat_logits<float, NV_, 8>), wb, 256, 0, st, V, a, P->attn_l, P->attn_r); \
    else if (SEG == 16) WG_LAUNCH((k_gat_logits<float, NV_, 16>), wb, 256, 0, st, V, a, P->attn_l, P->attn_r); \
    else if (SEG == 32) WG_LAUNCH((k_gat_logits<float, NV_, 32>), wb, 256, 0, st, V, a, P->attn_l, P->attn_r); \
    else WG_LAUNCH((k_gat_logits<float, NV_, 0>), wb, 256, 0, st, V, a, P->attn_l, P->attn_r);            \
  } while (0)
    if (NV == 1) WG_GAT_L(1);
    else if (NV == 2) WG_GAT_L(2);
    else WG_GAT_L(4);
#undef WG_GAT_L
  }
  a.idx = g->fwd.idx;
  a.chunks = gp->fwd; a.n_chunks = gp->n_fwd;
  if (gp->n_fwd) {
    const unsigned cbk = gs_grid((int64_t)gp->n_fwd * 32);
    // two row chunks per warp: 40 % fewer instructions on C2 but fewer rows in
    // flight per SM (register limit) -- measured 306 vs 290 us per forward
    // (profiles/r02/ncu_gat_C2.csv), so opt-in (WG_GAT_HALF=1)
    static int half = -1;
    if (half < 0) {
      const char* e = getenv("WG_GAT_HALF");
      half = e ? atoi(e) : 0;
    }
    if (H <= 4 && NV <= 2 && half) {   // two row chunks per warp (half-warps)
      const unsigned hbk = gs_grid(cdiv((int64_t)gp->n_fwd, 2) * 32);
      if (NV == 1) WG_LAUNCH((k_gat_fwd3<float, T, 2, 4, 4>), hbk, 256, 0, st, a, vb);
      else if (half == 2) WG_LAUNCH((k_gat_fwd3<float, T, 4, 1, 4, 3>), hbk, 256, 0, st, a, vb);
      else if (half == 3) WG_LAUNCH((k_gat_fwd3<float, T, 4, 1, 4, 4>), hbk, 256, 0, st, a, vb);
      else WG_LAUNCH((k_gat_fwd3<float, T, 4, 2, 4>), hbk, 256, 0, st, a, vb);
    } else if (H <= 4) {
      if (NV == 1) WG_LAUNCH((k_gat_fwd2<float, T, 1, 8, 4>), cbk, 256, 0, st, a, vb);
      else if (NV == 2) WG_LAUNCH((k_gat_fwd2<float, T, 2, 4, 4>), cbk, 256, 0, st, a, vb);
      else WG_LAUNCH((k_gat_fwd2<float, T, 4, 2, 4>), cbk, 256, 0, st, a, vb);
    } else if (H <= GAT_HM) {
      if (NV == 1) WG_LAUNCH((k_gat_fwd2<float, T, 1, 8, 8>), cbk, 256, 0, st, a, vb);
      else if (NV == 2) WG_LAUNCH((k_gat_fwd2<float, T, 2, 4, 8>), cbk, 256, 0, st, a, vb);
      else WG_LAUNCH((k_gat_fwd2<float, T, 4, 2, 8>), cbk, 256, 0, st, a, vb);
    } else {
      if (NV == 1) WG_LAUNCH((k_gat_fwd<float, T, 1, 4>), cbk, 256, 0, st, a, vb);
      else if (NV == 2) WG_LAUNCH((k_gat_fwd<float, T, 2, 4>), cbk, 256, 0, st, a, vb);
      else WG_LAUNCH((k_gat_fwd<float, T, 4, 2>), cbk, 256, 0, st, a, vb);
    }
  }
  if (gp->n_fsplit) WG_LAUNCH(k_gat_fwd_combine<T>, gp->n_fsplit, 256, 0, st, a, gp->fsplit, vb);
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
  a.part = L.at<float>(ws, "part"); a.part_ld = (int)rup(HF + 2 * H + 8, 4);   // 16-byte rows (float4 partial stores)
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
  float4* bs = L.at<float4>(ws, "bs");
  a.bs = bs;
  void* dG = L.at<void>(ws, "dG");
  void* dGlo = d.dtype == WG_BF16 ? L.at<void>(ws, "dGlo") : nullptr;
  {
  // algorithmic bytes: s/bs (agg, dy rows), per out-edge the gathered dy row +
  // stats + index + fwdpos + dt, per row G and dg; der (dt again); dG
  ProfScope ps(PK_GAT, st,
               (double)g->bwd.E * (HF * s + 16.0 * H + 12 + 8.0 * H) +
                   (double)V * HF * (4.0 + s + 4.0 + 4.0 + 4.0 + 4.0 + s * (d.dtype == WG_BF16 ? 2 : 1)), 0.0);
  const int NV = nv_for<float>(a.VPR);
  const int vph = Fo / 4;                      // fp32 G vectors per head
  const int SEG = (vph == 8 || vph == 16 || vph == 32) ? vph : 0;
  const unsigned rbk = gs_grid(nr * 32);
#define WG_GAT_S(NV_, SEG_) WG_LAUNCH((k_gat_s2<T, NV_, SEG_>), rbk, 256, 0, st, nr, vb, a, bs)
#define WG_GAT_SEG(M, NV_)                      \
  do {                                          \
    if (SEG == 8) M(NV_, 8);                    \
    else if (SEG == 16) M(NV_, 16);             \
    else if (SEG == 32) M(NV_, 32);             \
    else M(NV_, 0);                             \
  } while (0)
  if (NV == 1) WG_GAT_SEG(WG_GAT_S, 1);
  else if (NV == 2) WG_GAT_SEG(WG_GAT_S, 2);
  else WG_GAT_SEG(WG_GAT_S, 4);
  a.idx = g->bwd.idx;
  a.fwdpos = g->fwdpos;
  a.dt = L.at<float>(ws, "dt");
  a.dg = L.at<float>(ws, "dg"); a.ld_dg = HF;
  a.del = L.at<float>(ws, "del");
  a.chunks = gp->bwd; a.n_chunks = gp->n_bwd;
  if (gp->n_bwd) {
    const unsigned cbk = gs_grid((int64_t)gp->n_bwd * 32);
#define WG_GAT_B1(NV_, SEG_) do { if (H <= 4) WG_LAUNCH((k_gat_bwd_src3<T, NV_, 8, SEG_, 4>), cbk, 256, 0, st, a, vb); \
    else if (H <= GAT_HM) WG_LAUNCH((k_gat_bwd_src3<T, NV_, 8, SEG_, 8>), cbk, 256, 0, st, a, vb);             \
    else WG_LAUNCH((k_gat_bwd_src2<T, NV_, 8, SEG_>), cbk, 256, 0, st, a, vb); } while (0)
// NV = 2 (the C2 widths): two dy rows in flight per warp at 4 CTAs / SM beats
// four rows at 2 CTAs / SM (per-row latency chains, C2 A/B: 4.94 -> 4.76 ms)
#define WG_GAT_B2(NV_, SEG_) do { if (H <= 4) WG_LAUNCH((k_gat_bwd_src3<T, NV_, 2, SEG_, 4, 4>), cbk, 256, 0, st, a, vb); \
    else if (H <= GAT_HM) WG_LAUNCH((k_gat_bwd_src3<T, NV_, 4, SEG_, 8>), cbk, 256, 0, st, a, vb);             \
    else WG_LAUNCH((k_gat_bwd_src2<T, NV_, 4, SEG_>), cbk, 256, 0, st, a, vb); } while (0)
#define WG_GAT_B4(NV_, SEG_) do { if (H <= 4) WG_LAUNCH((k_gat_bwd_src3<T, NV_, 2, SEG_, 4>), cbk, 256, 0, st, a, vb); \
    else if (H <= GAT_HM) WG_LAUNCH((k_gat_bwd_src3<T, NV_, 2, SEG_, 8>), cbk, 256, 0, st, a, vb);             \
    else WG_LAUNCH((k_gat_bwd_src2<T, NV_, 2, SEG_>), cbk, 256, 0, st, a, vb); } while (0)
    if (NV == 1) WG_GAT_SEG(WG_GAT_B1, 1);
    else if (NV == 2) WG_GAT_SEG(WG_GAT_B2, 2);
    else WG_GAT_SEG(WG_GAT_B4, 4);
#undef WG_GAT_B1
#undef WG_GAT_B2
#undef WG_GAT_B4
  }
#undef WG_GAT_S
#undef WG_GAT_SEG
  // rows without out-edges have no chunk: their dg / del are zero
  // (chunks cover every row, including empty ones -- see build_chunks)
  if (gp->n_bsplit) WG_LAUNCH(k_gat_bwd_combine, gp->n_bsplit, 256, 0, st, a, gp->bsplit, vb);
  float* der = L.at<float>(ws, "der");
  // (the split-row partial slots of the source-major pass were consumed by
  // k_gat_bwd_combine above: `part` is reused for the der partials)
  const unsigned tbk = gs_grid((int64_t)gp->n_fwd * 8), tbk32 = gs_grid(nr * 32);
  if (H == 4 || H == 1 || H == 2 || H == 8) {
    if (H == 4) WG_LAUNCH(k_gat_der3<4>, tbk, 256, 0, st, gp->fwd, gp->n_fwd, vb, a.dt, der, a.part, a.part_ld);
    else if (H == 1) WG_LAUNCH(k_gat_der3<1>, tbk, 256, 0, st, gp->fwd, gp->n_fwd, vb, a.dt, der, a.part, a.part_ld);
    else if (H == 2) WG_LAUNCH(k_gat_der3<2>, tbk, 256, 0, st, gp->fwd, gp->n_fwd, vb, a.dt, der, a.part, a.part_ld);
    else WG_LAUNCH(k_gat_der3<8>, tbk, 256, 0, st, gp->fwd, gp->n_fwd, vb, a.dt, der, a.part, a.part_ld);
    if (gp->n_fsplit)
      WG_LAUNCH(k_gat_der_combine, gs_grid((int64_t)gp->n_fsplit * H * 32), 256, 0, st, gp->fsplit, gp->n_fsplit, vb,
                a.part, a.part_ld, H, der);
  } else {
    WG_LAUNCH(k_gat_der, tbk32, 256, 0, st, nr, vb, g->fwd.row_ptr, a.dt, H, der);
  }
  const int64_t rpb = std::max<int64_t>(1, cdiv(nr, DG_BLKS));
  const int nblk = (int)cdiv(nr, rpb);
  float* dgp = L.at<float>(ws, "dgp");
  WG_LAUNCH(k_gat_dG<T>, nblk, 256, 0, st, nr, vb, a, P->attn_l, P->attn_r, der, (T*)dG, (T*)dGlo, p->po, dgp,
            rpb);
  WG_LAUNCH(k_pair_reduce, (unsigned)cdiv(2 * HF, 32), 1024, 0, st, dgp, nblk, HF, Gr ? Gr->attn_l : nullptr,
            Gr ? Gr->attn_r : nullptr);
  }
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
