// Fused Adam step for the training-step benchmark (the epoch
// = forward + loss + backward + optimizer).  Kingma & Ba's update as torch.optim.Adam
// computes it (no weight decay, no amsgrad):
//   m = b1 m + (1 - b1) g ; v = b2 v + (1 - b2) g^2 ; t = t + 1
//   p -= (lr / (1 - b1^t)) * m / (sqrt(v) / sqrt(1 - b2^t) + eps)
// over ONE flat fp32 buffer holding every parameter of the model (one launch
// instead of torch's ~20 per-op kernels per step).  The step count t lives on
// the device (state[0]) so a captured CUDA graph replays real steps; the last
// CTA to finish advances it (state[1] counts finished CTAs and is reset by it).
#include "wg_internal.cuh"

namespace wg {
namespace {

__global__ void __launch_bounds__(256) k_adam(int64_t n, float* __restrict__ p, const float* __restrict__ g,
                                              float* __restrict__ m, float* __restrict__ v, int32_t* state, float lr,
                                              float b1, float b2, float eps) {
  // every CTA reads t before any CTA can have advanced it (the advance waits
  // for all CTAs to finish)
  const int t = *reinterpret_cast<volatile int32_t*>(state) + 1;
  const float bc1 = 1.f - powf(b1, (float)t), bc2 = 1.f - powf(b2, (float)t);
  const float step = lr / bc1, rs2 = 1.f / sqrtf(bc2);
  const int64_t n4 = n / 4;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n4; i += stride) {
    float4 pp = reinterpret_cast<float4*>(p)[i], mm = reinterpret_cast<float4*>(m)[i],
           vv = reinterpret_cast<float4*>(v)[i];
    const float4 gg = __ldg(reinterpret_cast<const float4*>(g) + i);
    float* P = &pp.x; float* M = &mm.x; float* Q = &vv.x;
    const float* G = &gg.x;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      M[k] = b1 * M[k] + (1.f - b1) * G[k];
      Q[k] = b2 * Q[k] + (1.f - b2) * G[k] * G[k];
      P[k] -= step * M[k] / (sqrtf(Q[k]) * rs2 + eps);
    }
    reinterpret_cast<float4*>(p)[i] = pp;
    reinterpret_cast<float4*>(m)[i] = mm;
    reinterpret_cast<float4*>(v)[i] = vv;
  }
  for (int64_t i = 4 * n4 + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += stride) {
    m[i] = b1 * m[i] + (1.f - b1) * g[i];
    v[i] = b2 * v[i] + (1.f - b2) * g[i] * g[i];
    p[i] -= step * m[i] / (sqrtf(v[i]) * rs2 + eps);
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    if (atomicAdd(reinterpret_cast<unsigned*>(state + 1), 1u) == gridDim.x - 1) {
      state[0] = t;
      state[1] = 0;
      __threadfence();
    }
  }
}

}  // namespace
}  // namespace wg

extern "C" wg_status wg_adam_step(int64_t n, float* param, const float* grad, float* exp_avg, float* exp_avg_sq,
                                  int32_t* state, float lr, float beta1, float beta2, float eps, wg_stream stream) {
  using namespace wg;
  WG_REQ(n >= 0, WG_ERR_INVALID, "wg_adam_step: n < 0");
  if (n == 0) return WG_OK;
  WG_REQ(param && grad && exp_avg && exp_avg_sq && state, WG_ERR_INVALID, "wg_adam_step: null argument");
  WG_REQ(reinterpret_cast<uintptr_t>(param) % 16 == 0 && reinterpret_cast<uintptr_t>(grad) % 16 == 0 &&
             reinterpret_cast<uintptr_t>(exp_avg) % 16 == 0 && reinterpret_cast<uintptr_t>(exp_avg_sq) % 16 == 0,
         WG_ERR_INVALID, "wg_adam_step: buffers must be 16-byte aligned");
  cudaStream_t s = (cudaStream_t)stream;
  ProfScope ps(PK_MISC, s, (double)n * 28.0, 0.0);
  const unsigned nb = (unsigned)std::min<int64_t>(2 * 148, std::max<int64_t>(1, cdiv(cdiv(n, 4), 256)));
  WG_LAUNCH(k_adam, nb, 256, 0, s, n, param, grad, exp_avg, exp_avg_sq, state, lr, beta1, beta2, eps);
  return WG_OK;
}
