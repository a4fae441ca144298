// L2 residency probe for the power-law gathers of a6/a10: V rows at `pitch`
// bytes, E row reads whose source ranks follow the synthetic recipe
// (rank = floor(V * u^2), alpha = 0.5, hubs scattered by a permutation).
// Modes: 0 default loads; 1 hot rows (the H highest-rank sources) with an
// L2 evict_last policy, the rest evict_first; 2 hot default, rest evict_first;
// 3 = mode 1 after raising cudaLimitPersistingL2CacheSize to the maximum.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o l2_probe l2_probe.cu
#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <numeric>
#include <random>
#include <vector>
#include <cuda_runtime.h>

template <int MODE>
__device__ __forceinline__ int4 ld16(const int4* p, bool hot, uint64_t pl, uint64_t pf) {
  int4 v;
  if (MODE == 0) {
    asm volatile("ld.global.nc.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  } else if (MODE == 2 && hot) {
    asm volatile("ld.global.nc.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
  } else {
    const uint64_t pol = hot ? pl : pf;
    asm volatile("ld.global.nc.L2::cache_hint.v4.s32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p), "l"(pol));
  }
  return v;
}

template <int MODE>
__global__ void k_gather(const int4* __restrict__ tab, int64_t pitch16, int vecs, const int* __restrict__ idx,
                         int64_t n, int seg, int4* out) {
  uint64_t pl, pf;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pl));
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pf));
  const int lanes = vecs;
  const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const int64_t groups = (int64_t)gridDim.x * blockDim.x / lanes;
  const int l = (int)(t % lanes);
  // each group owns segments of `seg` consecutive indices (a destination row)
  for (int64_t s = t / lanes; s * seg < n; s += groups) {
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
    const int64_t e1 = min(n, (s + 1) * (int64_t)seg);
    for (int64_t r = s * seg; r < e1; ++r) {
      const int id = idx[r];
      const int4 v = ld16<MODE>(tab + (int64_t)(id & 0x7fffffff) * pitch16 + l, id < 0, pl, pf);
      acc.x += __int_as_float(v.x); acc.y += __int_as_float(v.y);
      acc.z += __int_as_float(v.z); acc.w += __int_as_float(v.w);
    }
    out[s * lanes + l] = make_int4(__float_as_int(acc.x), __float_as_int(acc.y), __float_as_int(acc.z),
                                   __float_as_int(acc.w));
  }
}

// cp.async (LDGSTS) variant with a D-deep per-lane ring, as k_agg_cp:
// MODE 4 default .L2::64B, 5 cold evict_first + .L2::64B, 6 cold evict_first (no 64B),
// 7 every row evict_first + .L2::64B
template <int MODE>
__device__ __forceinline__ void cpa(uint32_t s, const void* g, bool hot, uint64_t pf) {
  if (MODE == 4 || (hot && MODE != 7)) {
    if (MODE == 6) asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(s), "l"(g) : "memory");
    else asm volatile("cp.async.cg.shared.global.L2::64B [%0], [%1], 16;" ::"r"(s), "l"(g) : "memory");
  } else if (MODE == 6) {
    asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2;" ::"r"(s), "l"(g), "l"(pf) : "memory");
  } else {
    asm volatile("cp.async.cg.shared.global.L2::cache_hint.L2::64B [%0], [%1], 16, %2;" ::"r"(s), "l"(g), "l"(pf)
                 : "memory");
  }
}
template <int MODE>
__global__ void k_gather_cp(const int4* __restrict__ tab, int64_t pitch16, int vecs, const int* __restrict__ idx,
                            int64_t n, int seg, int4* out) {
  constexpr int D = 8;
  __shared__ int4 ring[D][256];
  uint64_t pf;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pf));
  const int lanes = vecs;
  const int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  const int64_t groups = (int64_t)gridDim.x * blockDim.x / lanes;
  const int l = (int)(t % lanes);
  for (int64_t s = t / lanes; s * seg < n; s += groups) {
    float4 acc = make_float4(0.f, 0.f, 0.f, 0.f);
    const int64_t e0 = s * seg, e1 = min(n, (s + 1) * (int64_t)seg);
    for (int64_t r = e0; r < e0 + D; ++r) {
      if (r < e1) {
        const int id = idx[r];
        cpa<MODE>((uint32_t)__cvta_generic_to_shared(&ring[(r - e0) % D][threadIdx.x]),
                  tab + (int64_t)(id & 0x7fffffff) * pitch16 + l, id < 0, pf);
      }
      asm volatile("cp.async.commit_group;" ::: "memory");
    }
    for (int64_t r = e0; r < e1; ++r) {
      asm volatile("cp.async.wait_group %0;" ::"n"(D - 1) : "memory");
      const int4 v = ring[(r - e0) % D][threadIdx.x];
      acc.x += __int_as_float(v.x); acc.y += __int_as_float(v.y);
      acc.z += __int_as_float(v.z); acc.w += __int_as_float(v.w);
      const int64_t rn = r + D;
      if (rn < e1) {
        const int id = idx[rn];
        cpa<MODE>((uint32_t)__cvta_generic_to_shared(&ring[(rn - e0) % D][threadIdx.x]),
                  tab + (int64_t)(id & 0x7fffffff) * pitch16 + l, id < 0, pf);
      }
      asm volatile("cp.async.commit_group;" ::: "memory");
    }
    asm volatile("cp.async.wait_group 0;" ::: "memory");
    out[s * lanes + l] = make_int4(__float_as_int(acc.x), __float_as_int(acc.y), __float_as_int(acc.z),
                                   __float_as_int(acc.w));
  }
}

int main() {
  const int64_t V = 2449029, E = 61859140;
  int dev_persist = 0;
  cudaDeviceGetAttribute(&dev_persist, cudaDevAttrMaxPersistingL2CacheSize, 0);
  int l2 = 0;
  cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, 0);
  printf("L2 %d B, max persisting %d B\n", l2, dev_persist);
  std::mt19937_64 rng(7);
  std::vector<int> perm(V);
  std::iota(perm.begin(), perm.end(), 0);
  std::shuffle(perm.begin(), perm.end(), rng);
  std::uniform_real_distribution<double> U(0.0, 1.0);
  std::vector<int64_t> rank(E);
  for (auto& r : rank) { const double u = U(rng); r = std::min<int64_t>(V - 1, (int64_t)(V * u * u)); }
  int* idx;
  cudaMalloc(&idx, E * 4);
  int4* tab;
  cudaMalloc(&tab, V * 512);
  cudaMemset(tab, 0, V * 512);
  int4* out;
  cudaMalloc(&out, (E / 25 + 2) * 512);
  struct Case { int row, pitch; } cases[] = {{512, 512}, {96, 128}};
  for (auto c : cases) {
    for (double mb : {0.0, 48.0, 96.0}) {
      const int64_t H = (int64_t)(mb * 1048576.0 / c.pitch);
      std::vector<int> h(E);
      for (int64_t i = 0; i < E; ++i) h[i] = perm[rank[i]] | (rank[i] < H ? (int)0x80000000 : 0);
      cudaMemcpy(idx, h.data(), E * 4, cudaMemcpyHostToDevice);
      for (int mode = 0; mode < 8; ++mode) {
        if (mode == 1 || mode == 3) continue;
        if (mb == 0.0 && mode != 0 && mode != 4) continue;
        cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, mode == 3 ? (size_t)dev_persist : 0);
        const int vecs = c.row / 16;
        const int seg = 25;
        auto launch = [&]() {
          const int grid = 148 * 8;
          if (mode == 0) k_gather<0><<<grid, 256>>>(tab, c.pitch / 16, vecs, idx, E, seg, out);
          else if (mode == 2) k_gather<2><<<grid, 256>>>(tab, c.pitch / 16, vecs, idx, E, seg, out);
          else if (mode == 1) k_gather<1><<<grid, 256>>>(tab, c.pitch / 16, vecs, idx, E, seg, out);
          else if (mode == 4) k_gather_cp<4><<<grid, 256>>>(tab, c.pitch / 16, vecs, idx, E, seg, out);
          else if (mode == 5) k_gather_cp<5><<<grid, 256>>>(tab, c.pitch / 16, vecs, idx, E, seg, out);
          else if (mode == 6) k_gather_cp<6><<<grid, 256>>>(tab, c.pitch / 16, vecs, idx, E, seg, out);
          else k_gather_cp<7><<<grid, 256>>>(tab, c.pitch / 16, vecs, idx, E, seg, out);
        };
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        launch();
        launch();
        cudaEventRecord(a);
        for (int k = 0; k < 5; ++k) launch();
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms = 0;
        cudaEventElapsedTime(&ms, a, b);
        ms /= 5;
        const double alg = (double)E * (c.row + 4) + (double)(E / seg) * c.row;
        printf("row %3d pitch %3d hot %5.1f MB (H=%8lld) mode %d: %.3f ms  %.0f GB/s algorithmic  %.1f G rows/s\n",
               c.row, c.pitch, mb, (long long)H, mode, ms, alg / ms / 1e6, E / ms / 1e6);
        fflush(stdout);
      }
    }
  }
  cudaError_t e = cudaGetLastError();
  printf("status %s\n", cudaGetErrorString(e));
  return 0;
}
