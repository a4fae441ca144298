// DRAM fetch granularity probe for random row gathers (the a6/a10 access
// pattern): each launch reads N_IDX random rows of `row` bytes at pitch
// `pitch` from a 4 GiB table (>> 126 MB L2) with 16-byte vector loads, one
// row per group of row/16 lanes.  Run under
//   ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum ./gran_probe
// and compare dram bytes per row with `row`.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gran_probe gran_probe.cu
#include <cstdio>
#include <cstdint>
#include <vector>
#include <random>
#include <cuda_runtime.h>

template <int MODE>
__device__ __forceinline__ int4 ld16(const int4* p) {
  int4 v;
  if (MODE == 0) {
    v = __ldg(p);
  } else if (MODE == 1) {
    asm volatile("ld.global.nc.L2::64B.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  } else if (MODE == 2) {
    asm volatile("ld.global.cg.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  } else {
    asm volatile("ld.global.nc.L1::no_allocate.L2::64B.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  }
  return v;
}

template <int MODE>
__global__ void k_gather(const int4* __restrict__ tab, int64_t pitch16, int vecs, const int* __restrict__ idx,
                         int64_t n, int4* out) {
  const int lanes = vecs;                       // lanes per row
  const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const int64_t groups = (int64_t)gridDim.x * blockDim.x / lanes;
  int4 acc = make_int4(0, 0, 0, 0);
  const int l = (int)(t % lanes);
  for (int64_t r = t / lanes; r < n; r += groups) {
    const int4 v = ld16<MODE>(tab + (int64_t)idx[r] * pitch16 + l);
    acc.x ^= v.x; acc.y ^= v.y; acc.z ^= v.z; acc.w ^= v.w;
  }
  if (acc.x == 0x12345678) out[t] = acc;
}

int main() {
  const size_t bytes = 4ull << 30;
  int4* tab;
  cudaMalloc(&tab, bytes);
  cudaMemset(tab, 1, bytes);
  const int64_t n = 1 << 24;
  int* idx;
  cudaMalloc(&idx, n * 4);
  int4* out;
  cudaMalloc(&out, 1 << 26);
  struct Case { int row, pitch; } cases[] = {{32, 32}, {64, 64}, {96, 96}, {96, 128}, {128, 128}, {256, 256}};
  std::mt19937_64 rng(1);
  for (int lim = 0; lim < 2; ++lim) {
    if (lim) cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, 32);
    size_t g = 0;
    cudaDeviceGetLimit(&g, cudaLimitMaxL2FetchGranularity);
    for (int mode = 0; mode < 4; ++mode) {
      for (auto c : cases) {
        const int64_t rows = bytes / c.pitch;
        std::vector<int> h(n);
        for (auto& v : h) v = (int)(rng() % rows);
        cudaMemcpy(idx, h.data(), n * 4, cudaMemcpyHostToDevice);
        const int vecs = c.row / 16;
        cudaEvent_t a, b;
        cudaEventCreate(&a); cudaEventCreate(&b);
        auto launch = [&]() {
          if (mode == 0) k_gather<0><<<148 * 8, 256>>>(tab, c.pitch / 16, vecs, idx, n, out);
          else if (mode == 1) k_gather<1><<<148 * 8, 256>>>(tab, c.pitch / 16, vecs, idx, n, out);
          else if (mode == 2) k_gather<2><<<148 * 8, 256>>>(tab, c.pitch / 16, vecs, idx, n, out);
          else k_gather<3><<<148 * 8, 256>>>(tab, c.pitch / 16, vecs, idx, n, out);
        };
        launch();
        cudaEventRecord(a);
        launch();
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms = 0;
        cudaEventElapsedTime(&ms, a, b);
        printf("limit %zu mode %d row %4d pitch %4d: %.3f ms  rows/s %.2f G  (%s)\n", g, mode, c.row, c.pitch, ms,
               n / ms / 1e6, cudaGetErrorString(cudaGetLastError()));
      }
    }
  }
  return 0;
}
