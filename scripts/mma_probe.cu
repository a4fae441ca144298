// tcgen05.mma issue-rate probe: cycles per MMA for the shapes the layer
// GEMMs use (operands resident in shared memory, no TMA, one CTA per SM on
// every SM).  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o
// mma_probe scripts/mma_probe.cu ; run: ./mma_probe
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t addr, uint32_t lbo, uint32_t sbo, uint32_t layout) {
  uint64_t d = 0;
  d |= (uint64_t)((addr >> 4) & 0x3FFF);
  d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)layout << 61;
  return d;
}

// KIND 0: kind::f16 (bf16), 1: kind::tf32.  MN: both operands MN-major.
template <int KIND, bool MN>
__global__ void __launch_bounds__(128, 1) k_probe(int N, int iters, long long* out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  uint8_t* base = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(sm) + 1023) & ~uintptr_t(1023));
  __shared__ uint64_t bar;
  __shared__ uint32_t slot;
  for (int i = threadIdx.x; i < 96 * 1024 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(base)[i] = 0;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 256;" ::"r"(su32(&slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = slot;
  if (threadIdx.x == 0) {
    const uint32_t fmt = KIND == 1 ? 2u : 1u;
    const uint32_t idesc = (1u << 4) | (fmt << 7) | (fmt << 10) | ((MN ? 1u : 0u) << 15) | ((MN ? 1u : 0u) << 16) |
                           ((uint32_t)(N >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
    const uint32_t a0 = su32(base), b0 = a0 + 32 * 1024;
    const uint32_t lbo = MN ? (KIND == 1 ? 32 * 128 : 64 * 128) : 16;
    const uint32_t sbo = (MN && KIND == 1) ? 512 : 1024;
    const uint32_t lay = (MN && KIND == 1) ? 1 : 2;
    long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
      const int k = it & 3;
      const uint32_t step = MN ? (uint32_t)(k * (KIND == 1 ? 8 : 16) * 128) : (uint32_t)(k * 32);
      const uint64_t ad = desc(a0 + step, lbo, sbo, lay), bd = desc(b0 + step, lbo, sbo, lay);
      const uint32_t acc = it ? 1u : 0u;
      if (KIND == 1)
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}\n"
                     ::"r"(tmem), "l"(ad), "l"(bd), "r"(idesc), "r"(acc));
      else
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n"
                     ::"r"(tmem), "l"(ad), "l"(bd), "r"(idesc), "r"(acc));
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(&bar)) : "memory");
    asm volatile("{\n.reg .pred p;\nW:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n@!p bra W;\n}\n" ::"r"(su32(&bar)) : "memory");
    long long t1 = clock64();
    out[blockIdx.x] = t1 - t0;
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 256;" ::"r"(tmem));
}

template <int KIND, bool MN>
void run(const char* name, int N, int blocks) {
  const int iters = 20000;
  long long* d;
  cudaMalloc(&d, sizeof(long long) * blocks);
  auto k = k_probe<KIND, MN>;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
  k<<<blocks, 128, 100 * 1024>>>(N, 100, d);   // warm-up
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  k<<<blocks, 128, 100 * 1024>>>(N, iters, d);
  cudaEventRecord(e1);
  cudaError_t err = cudaDeviceSynchronize();
  float ms = 0;
  cudaEventElapsedTime(&ms, e0, e1);
  long long h[148];
  cudaMemcpy(h, d, sizeof(long long) * blocks, cudaMemcpyDeviceToHost);
  double mean = 0;
  for (int i = 0; i < blocks; ++i) mean += (double)h[i] / blocks;
  const double flop = 2.0 * 128 * N * (KIND == 1 ? 8 : 16) * (double)iters * blocks;
  const double opb = (128.0 + N) * 32;   // operand bytes per MMA (32 bytes of K per row)
  printf("%-28s N=%3d blocks=%3d  %7.1f cycles/MMA  %6.1f operand B/cycle  %7.1f TFLOP/s  %s\n", name, N, blocks,
         mean / iters, opb / (mean / iters), flop / (ms * 1e-3) / 1e12, err == cudaSuccess ? "" : cudaGetErrorString(err));
  cudaFree(d);
}

int main() {
  for (int blocks : {1, 148}) {
    run<1, false>("tf32 K-major", 64, blocks);
    run<1, false>("tf32 K-major", 128, blocks);
    run<1, false>("tf32 K-major", 256, blocks);
    run<1, true>("tf32 MN-major", 64, blocks);
    run<1, true>("tf32 MN-major", 128, blocks);
    run<0, false>("bf16 K-major", 64, blocks);
    run<0, false>("bf16 K-major", 128, blocks);
    run<0, false>("bf16 K-major", 256, blocks);
    run<0, true>("bf16 MN-major", 64, blocks);
    run<0, true>("bf16 MN-major", 256, blocks);
  }
  return 0;
}
