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

__global__ void k_gather(const int4* __restrict__ tab, int64_t pitch16, int vecs, const int* __restrict__ idx,
                         int64_t n, int4* out) {
  const int lanes = vecs;                       // lanes per row
  const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const int64_t groups = (int64_t)gridDim.x * blockDim.x / lanes;
  int4 acc = make_int4(0, 0, 0, 0);
  const int l = (int)(t % lanes);
  for (int64_t r = t / lanes; r < n; r += groups) {
    const int4 v = __ldg(tab + (int64_t)idx[r] * pitch16 + l);
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
  struct Case { int row, pitch; } cases[] = {{32, 32}, {64, 64}, {64, 128}, {96, 96}, {96, 128}, {128, 128},
                                             {192, 192}, {224, 224}, {256, 256}, {512, 512}};
  std::mt19937_64 rng(1);
  for (auto c : cases) {
    const int64_t rows = bytes / c.pitch;
    std::vector<int> h(n);
    for (auto& v : h) v = (int)(rng() % rows);
    cudaMemcpy(idx, h.data(), n * 4, cudaMemcpyHostToDevice);
    const int vecs = c.row / 16;
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    k_gather<<<148 * 8, 256>>>(tab, c.pitch / 16, vecs, idx, n, out);   // warm
    cudaEventRecord(a);
    k_gather<<<148 * 8, 256>>>(tab, c.pitch / 16, vecs, idx, n, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms = 0;
    cudaEventElapsedTime(&ms, a, b);
    const double useful = (double)n * (c.row + 4);
    printf("row %4d pitch %4d: %.3f ms  useful %.2f GB/s  (%.1f ns/row)\n", c.row, c.pitch, ms, useful / ms / 1e6,
           ms * 1e6 / n);
  }
  return 0;
}
