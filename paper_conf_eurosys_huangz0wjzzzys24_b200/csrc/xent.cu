// Fused softmax cross-entropy (loss + gradient) for the training step: one
// warp per row, fixed-order block partials for the loss (deterministic).
#include "wg_internal.cuh"

namespace wg {
namespace {

constexpr int XENT_BLKS = 1184;   // 8 x 148 SMs; partials fit WG_XENT_SCRATCH_BYTES

template <typename T> __device__ __forceinline__ float ld_f(const T* p) { return (float)*p; }
template <> __device__ __forceinline__ float ld_f<__nv_bfloat16>(const __nv_bfloat16* p) { return __bfloat162float(*p); }

template <typename T, int PER>
__global__ void __launch_bounds__(256) k_xent(int64_t M, int C, const T* x, int64_t ld, const int64_t* labels,
                                              float scale, T* dx, int64_t ldd, float* part, int64_t rows_per_blk) {
  __shared__ float wsum[8];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t r0 = blockIdx.x * rows_per_blk, r1 = min(M, r0 + rows_per_blk);
  const int Cpad = (C + 7) / 8 * 8;
  float lsum = 0.f;
  for (int64_t r = r0 + warp; r < r1; r += 8) {
    float v[PER];
    float m = -INFINITY;
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      const int j = lane + 32 * k;
      v[k] = j < C ? ld_f<T>(x + r * ld + j) : -INFINITY;
      m = fmaxf(m, v[k]);
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
    float s = 0.f, t_lab = 0.f;
    const int64_t lab = labels[r];
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      const int j = lane + 32 * k;
      const float t = j < C ? v[k] - m : 0.f;
      if (j == lab) t_lab = t;
      v[k] = j < C ? __expf(t) : 0.f;
      s += v[k];
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    const float inv = 1.f / s;
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      const int j = lane + 32 * k;
      if (j < Cpad) {
        const float p = j < C ? v[k] * inv : 0.f;
        dx[r * ldd + j] = (T)(j < C ? scale * (p - (j == lab ? 1.f : 0.f)) : 0.f);
        if (j == lab) lsum += scale * (logf(s) - t_lab);
      }
    }
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) lsum += __shfl_xor_sync(0xffffffffu, lsum, o);
  if (lane == 0) wsum[warp] = lsum;
  __syncthreads();
  if (threadIdx.x == 0) {
    float t = 0.f;
    for (int w = 0; w < 8; ++w) t += wsum[w];
    part[blockIdx.x] = t;
  }
}

// small C: groups of 8 lanes per row (4 rows per warp in flight), lane j holds
// columns j, j+8, ..., reductions are 3-step shuffles inside the group
template <typename T, int PER>
__global__ void __launch_bounds__(256) k_xent_row(int64_t M, int C, const T* x, int64_t ld, const int64_t* labels,
                                                  float scale, T* dx, int64_t ldd, float* part) {
  __shared__ float wsum[8];
  const int Cpad = (C + 7) / 8 * 8;
  const int lane = threadIdx.x & 31, g = lane >> 3, l = lane & 7;
  const unsigned gm = 0xffu << (g * 8);
  float lsum = 0.f;
  const int64_t rows_per_iter = (int64_t)gridDim.x * (blockDim.x / 8);
  for (int64_t r = blockIdx.x * (int64_t)(blockDim.x / 8) + (threadIdx.x >> 3); r < M; r += rows_per_iter) {
    float v[PER];
    float m = -INFINITY;
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      const int j = l + 8 * k;
      v[k] = j < C ? ld_f<T>(x + r * ld + j) : -INFINITY;
      m = fmaxf(m, v[k]);
    }
#pragma unroll
    for (int o = 4; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(gm, m, o, 8));
    const int64_t lab = labels[r];
    float s = 0.f, t_lab = 0.f;
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      const int j = l + 8 * k;
      const float t = j < C ? v[k] - m : 0.f;
      if (j == lab) t_lab = t;
      v[k] = j < C ? __expf(t) : 0.f;
      s += v[k];
    }
#pragma unroll
    for (int o = 4; o; o >>= 1) s += __shfl_xor_sync(gm, s, o, 8);
    const float inv = 1.f / s;
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      const int j = l + 8 * k;
      if (j < Cpad) dx[r * ldd + j] = (T)(j < C ? scale * (v[k] * inv - (j == lab ? 1.f : 0.f)) : 0.f);
      if (j == lab) lsum += scale * (logf(s) - t_lab);
    }
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) lsum += __shfl_xor_sync(0xffffffffu, lsum, o);
  if ((threadIdx.x & 31) == 0) wsum[threadIdx.x >> 5] = lsum;
  __syncthreads();
  if (threadIdx.x == 0) {
    float t = 0.f;
    for (int w = 0; w < 8; ++w) t += wsum[w];
    part[blockIdx.x] = t;
  }
}


// small C, vectorised: groups of 8 lanes per row (4 rows per warp), lane l
// loads / stores 16-byte vectors l, l + 8, ... of the row (NVL per lane), so a
// row is one coalesced load and one store per lane instead of C scalar ones
// (the rows are ld-aligned: ld * sizeof(T) is a multiple of 16 bytes).
template <typename T> struct XV;
template <> struct XV<float> {
  static constexpr int EPV = 4;
  __device__ static void unpack(const int4& q, float* f) {
    f[0] = __int_as_float(q.x); f[1] = __int_as_float(q.y); f[2] = __int_as_float(q.z); f[3] = __int_as_float(q.w);
  }
  __device__ static int4 pack(const float* f) {
    return make_int4(__float_as_int(f[0]), __float_as_int(f[1]), __float_as_int(f[2]), __float_as_int(f[3]));
  }
};
template <> struct XV<__nv_bfloat16> {
  static constexpr int EPV = 8;
  __device__ static void unpack(const int4& q, float* f) {
    const uint32_t w[4] = {(uint32_t)q.x, (uint32_t)q.y, (uint32_t)q.z, (uint32_t)q.w};
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

template <typename T, int NVL, int RPG, int MINB = 4>
__global__ void __launch_bounds__(256, MINB) k_xent_vec(int64_t M, int C, const T* x, int64_t ld, const int64_t* labels,
                                                  float scale, T* dx, int64_t ldd, float* part) {
  // RPG rows per 8-lane group per iteration: all their loads are issued
  // before any is used (one row per group left ~24 KB in flight per SM)
  constexpr int EPV = XV<T>::EPV;
  __shared__ float wsum[8];
  const int Cpad = (C + 7) / 8 * 8;
  const int lane = threadIdx.x & 31, g = lane >> 3, l = lane & 7;
  const unsigned gm = 0xffu << (g * 8);
  float lsum = 0.f;
  const int64_t groups = (int64_t)gridDim.x * (blockDim.x / 8);
  const int64_t gid = blockIdx.x * (int64_t)(blockDim.x / 8) + (threadIdx.x >> 3);
  for (int64_t r0 = gid * RPG; r0 < M; r0 += groups * RPG) {
    // raw 16-byte vectors of all RPG rows in flight (4 registers each), the
    // rows unpacked one at a time
    int4 raw[RPG][NVL];
    int32_t lab[RPG];
#pragma unroll
    for (int j = 0; j < RPG; ++j) {
      const int64_t r = r0 + j;
      lab[j] = r < M ? (int32_t)__ldg(labels + r) : -1;
#pragma unroll
      for (int q = 0; q < NVL; ++q) {
        const int c0 = (l + 8 * q) * EPV;
        raw[j][q] = (r < M && c0 < Cpad) ? __ldg(reinterpret_cast<const int4*>(x + r * ld + c0)) : make_int4(0, 0, 0, 0);
      }
    }
#pragma unroll
    for (int j = 0; j < RPG; ++j) {
      const int64_t r = r0 + j;
      if (r >= M) break;                       // group-uniform
      float v[1][NVL][EPV];
#pragma unroll
      for (int q = 0; q < NVL; ++q) XV<T>::unpack(raw[j][q], v[0][q]);
      float m = -INFINITY;
#pragma unroll
      for (int q = 0; q < NVL; ++q) {
        const int c0 = (l + 8 * q) * EPV;
#pragma unroll
        for (int i = 0; i < EPV; ++i) {
          if (c0 + i >= C) v[0][q][i] = -INFINITY;
          m = fmaxf(m, v[0][q][i]);
        }
      }
#pragma unroll
      for (int o = 4; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(gm, m, o, 8));
      float s = 0.f, t_lab = 0.f;
#pragma unroll
      for (int q = 0; q < NVL; ++q) {
        const int c0 = (l + 8 * q) * EPV;
#pragma unroll
        for (int i = 0; i < EPV; ++i) {
          const bool in = c0 + i < C;
          const float t = in ? v[0][q][i] - m : 0.f;
          if (c0 + i == lab[j]) t_lab = t;
          v[0][q][i] = in ? __expf(t) : 0.f;
          s += v[0][q][i];
        }
      }
#pragma unroll
      for (int o = 4; o; o >>= 1) s += __shfl_xor_sync(gm, s, o, 8);
      const float inv = 1.f / s;
#pragma unroll
      for (int q = 0; q < NVL; ++q) {
        const int c0 = (l + 8 * q) * EPV;
        if (c0 >= Cpad) continue;
        float o[EPV];
#pragma unroll
        for (int i = 0; i < EPV; ++i)
          o[i] = c0 + i < C ? scale * (v[0][q][i] * inv - (c0 + i == lab[j] ? 1.f : 0.f)) : 0.f;
        *reinterpret_cast<int4*>(dx + r * ldd + c0) = XV<T>::pack(o);
        if (lab[j] >= c0 && lab[j] < c0 + EPV) lsum += scale * (logf(s) - t_lab);
      }
    }
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) lsum += __shfl_xor_sync(0xffffffffu, lsum, o);
  if ((threadIdx.x & 31) == 0) wsum[threadIdx.x >> 5] = lsum;
  __syncthreads();
  if (threadIdx.x == 0) {
    float t = 0.f;
    for (int w = 0; w < 8; ++w) t += wsum[w];
    part[blockIdx.x] = t;
  }
}

// one warp: lane l sums part[l], part[l + 32], ... then a fixed xor tree
__global__ void k_sum(const float* part, int n, float* out) {
  const int lane = threadIdx.x & 31;
  float t = 0.f;
#pragma unroll 4
  for (int i = lane; i < n; i += 32) t += part[i];
#pragma unroll
  for (int o = 16; o; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
  if (lane == 0) *out = t;
}

template <typename T, int PER>
wg_status run(int64_t M, int C, const void* x, int64_t ld, const int64_t* labels, float scale, void* dx, int64_t ldd,
              float* loss, float* part, cudaStream_t s) {
  const int64_t rpb = std::max<int64_t>(1, cdiv(M, XENT_BLKS));
  const int nblk = (int)std::max<int64_t>(1, cdiv(M, rpb));
  WG_LAUNCH((k_xent<T, PER>), nblk, 256, 0, s, M, C, (const T*)x, ld, labels, scale, (T*)dx, ldd, part, rpb);
  WG_LAUNCH(k_sum, 1, 32, 0, s, part, nblk, loss);
  return WG_OK;
}

}  // namespace
}  // namespace wg

extern "C" wg_status wg_softmax_xent(wg_dtype dtype, int64_t M, int32_t C, const void* logits, int64_t ld,
                                     const int64_t* labels, float scale, void* dlogits, int64_t ldd, float* loss_out,
                                     void* scratch, wg_stream stream) {
  using namespace wg;
  WG_REQ(logits && labels && dlogits && loss_out && scratch, WG_ERR_INVALID, "wg_softmax_xent: null argument");
  WG_REQ(C >= 1 && C <= 1024 && ld >= C && ldd >= C, WG_ERR_INVALID, "wg_softmax_xent: C / ld");
  cudaStream_t s = (cudaStream_t)stream;
  ProfScope ps(PK_MISC, s, (double)M * C * (dtype == WG_BF16 ? 4.0 : 8.0) + M * 8.0, 0.0);
  float* part = static_cast<float*>(scratch);
  const int per = (C + 31) / 32;
  const bool vec = ((ld * (dtype == WG_BF16 ? 2 : 4)) % 16 == 0) && ((ldd * (dtype == WG_BF16 ? 2 : 4)) % 16 == 0) &&
                   (reinterpret_cast<uintptr_t>(logits) % 16 == 0) && (reinterpret_cast<uintptr_t>(dlogits) % 16 == 0);
  // wider rows (C5's 172 classes): the same 8-lane groups with 2-4 vectors
  // per lane -- the one-warp-per-row kernel below walks ~12 K rows per CTA
  // with one dependent row at a time (C5 rank slice: misc class 8.4 -> 6.3 ms;
  // 16-lane groups with two rows in flight measured slower)
  if (vec && C > 64 && C <= (dtype == WG_BF16 ? 256 : 128)) {
    const unsigned nb = (unsigned)std::min<int64_t>(XENT_BLKS, std::max<int64_t>(1, cdiv(M, 32)));
    const int nvl = (int)cdiv(cdiv(C, dtype == WG_BF16 ? 8 : 4), 8);   // vectors per lane
    if (dtype == WG_BF16) {
      if (nvl <= 2) WG_LAUNCH((k_xent_vec<__nv_bfloat16, 2, 2, 3>), nb, 256, 0, s, M, C, (const __nv_bfloat16*)logits, ld,
                              labels, scale, (__nv_bfloat16*)dlogits, ldd, part);
      else WG_LAUNCH((k_xent_vec<__nv_bfloat16, 4, 1, 2>), nb, 256, 0, s, M, C, (const __nv_bfloat16*)logits, ld, labels,
                     scale, (__nv_bfloat16*)dlogits, ldd, part);
    } else {
      if (nvl <= 3) WG_LAUNCH((k_xent_vec<float, 3, 1>), nb, 256, 0, s, M, C, (const float*)logits, ld, labels, scale,
                              (float*)dlogits, ldd, part);
      else WG_LAUNCH((k_xent_vec<float, 4, 1, 3>), nb, 256, 0, s, M, C, (const float*)logits, ld, labels, scale,
                     (float*)dlogits, ldd, part);
    }
    WG_LAUNCH(k_sum, 1, 32, 0, s, part, (int)nb, loss_out);
    return WG_OK;
  }
  if (C <= 64) {
    const unsigned nb = (unsigned)std::min<int64_t>(XENT_BLKS, std::max<int64_t>(1, cdiv(M, 32)));
    if (dtype == WG_BF16 && vec)
      WG_LAUNCH((k_xent_vec<__nv_bfloat16, 1, 4>), nb, 256, 0, s, M, C, (const __nv_bfloat16*)logits, ld, labels, scale,
                (__nv_bfloat16*)dlogits, ldd, part);
    else if (vec)
      WG_LAUNCH((k_xent_vec<float, 2, 2>), nb, 256, 0, s, M, C, (const float*)logits, ld, labels, scale,
                (float*)dlogits, ldd, part);
    else if (dtype == WG_BF16)
      WG_LAUNCH((k_xent_row<__nv_bfloat16, 8>), nb, 256, 0, s, M, C, (const __nv_bfloat16*)logits, ld, labels, scale,
                (__nv_bfloat16*)dlogits, ldd, part);
    else
      WG_LAUNCH((k_xent_row<float, 8>), nb, 256, 0, s, M, C, (const float*)logits, ld, labels, scale,
                (float*)dlogits, ldd, part);
    WG_LAUNCH(k_sum, 1, 32, 0, s, part, (int)nb, loss_out);
    return WG_OK;
  }
  if (dtype == WG_BF16) {
    if (per <= 2) return run<__nv_bfloat16, 2>(M, C, logits, ld, labels, scale, dlogits, ldd, loss_out, part, s);
    if (per <= 8) return run<__nv_bfloat16, 8>(M, C, logits, ld, labels, scale, dlogits, ldd, loss_out, part, s);
    return run<__nv_bfloat16, 32>(M, C, logits, ld, labels, scale, dlogits, ldd, loss_out, part, s);
  }
  if (per <= 2) return run<float, 2>(M, C, logits, ld, labels, scale, dlogits, ldd, loss_out, part, s);
  if (per <= 8) return run<float, 8>(M, C, logits, ld, labels, scale, dlogits, ldd, loss_out, part, s);
  return run<float, 32>(M, C, logits, ld, labels, scale, dlogits, ldd, loss_out, part, s);
}
