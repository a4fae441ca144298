// CUDA-core (FFMA) GEMMs: the fallback for shapes / alignments the tcgen05
// kernels (bf16, and fp32 through 3xTF32) do not take.  Dispatch: gemm_nt /
// gemm_tn / gemm_tn_grouped try the tensor-core path first.
#include <algorithm>

#include "wg_internal.cuh"

namespace wg {

bool tc_gemm_nt(wg_dtype dt, int64_t M, int N, const GemmPart* parts, int n_parts, const GemmEpi& epi,
                cudaStream_t s, wg_status* st);
bool tc_gemm_tn_grouped(wg_dtype dt, const TnUnits& U, int M, int N, const void* A, int64_t lda, const void* B,
                        int64_t ldb, float* D, float* part, cudaStream_t s, wg_status* st);
bool tc_gemm_tn(wg_dtype dt, int64_t K, int M, int N, const void* A, int64_t lda, const void* B, int64_t ldb, float* D,
                float* part, cudaStream_t s, wg_status* st, int acc);

namespace {

template <typename T> __device__ __forceinline__ float tof(T v) { return (float)v; }
template <> __device__ __forceinline__ float tof<__nv_bfloat16>(__nv_bfloat16 v) { return __bfloat162float(v); }

constexpr int BM = 64, BN = 64, BK = 16;

struct NTArgs {
  int64_t M;
  int N;
  GemmPart parts[3];
  int n_parts;
  GemmEpi epi;
};

template <typename T>
__global__ void __launch_bounds__(256) k_gemm_nt(NTArgs a) {
  __shared__ float As[BK][BM + 4];
  __shared__ float Bs[BK][BN + 4];
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  const int64_t m0 = (int64_t)blockIdx.x * BM;
  const int n0 = blockIdx.y * BN;
  float acc[4][4] = {};
  for (int p = 0; p < a.n_parts; ++p) {
    const GemmPart P = a.parts[p];
    const T* A = static_cast<const T*>(P.A);
    const T* B = static_cast<const T*>(P.B);
    if (P.tile_group) B += (int64_t)P.tile_group[m0 / 128] * P.group_rows * P.ldb;
    for (int k0 = 0; k0 < P.K; k0 += BK) {
      for (int t = threadIdx.x; t < BM * BK; t += 256) {
        int mm = t / BK, kk = t % BK;
        int64_t m = m0 + mm;
        int k = k0 + kk;
        const int64_t am = P.a_rows ? (m < a.M ? (int64_t)P.a_rows[m] : 0) : m;   // row-gathered A
        As[kk][mm] = (m < a.M && k < P.K) ? tof<T>(A[am * P.lda + k]) : 0.f;
        int n = n0 + mm;
        Bs[kk][mm] = (n < a.N && n < P.nb && k < P.K) ? tof<T>(B[(int64_t)n * P.ldb + k]) : 0.f;
      }
      __syncthreads();
#pragma unroll
      for (int kk = 0; kk < BK; ++kk) {
        float av[4], bv[4];
#pragma unroll
        for (int i = 0; i < 4; ++i) { av[i] = As[kk][ty * 4 + i]; bv[i] = Bs[kk][tx * 4 + i]; }
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
          for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
      }
      __syncthreads();
    }
  }
  const GemmEpi& e = a.epi;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const int64_t m = m0 + ty * 4 + i;
    if (m >= a.M) continue;
    const float rs = e.rscale ? e.rscale[m] : 1.f;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int n = n0 + tx * 4 + j;
      if (n >= a.N) continue;
      float v = (e.D2 && n >= e.n_split) ? acc[i][j] : rs * acc[i][j];
      if (e.addend) v += tof<T>(static_cast<const T*>(e.addend)[m * e.ld_add + n]);
      if (e.bias) v += e.bias[n];
      if (e.relu) v = fmaxf(v, 0.f);
      if (e.mask_ref && !(tof<T>(static_cast<const T*>(e.mask_ref)[m * e.ld_mask + n]) > 0.f)) v = 0.f;
      void* Dp = e.D;
      int64_t ld = e.ldd, nn = n;
      if (e.D2 && n >= e.n_split) { Dp = e.D2; ld = e.ldd2; nn = n - e.n_split; }
      if (e.d_f32) static_cast<float*>(Dp)[m * ld + nn] = v;
      else static_cast<T*>(Dp)[m * ld + nn] = (T)v;
    }
  }
}

// D[M x N] partials: part[z][m][n] = sum_{k in split z} A[k][m] * B[k][n]
template <typename T>
__global__ void __launch_bounds__(256) k_gemm_tn(int64_t K, int M, int N, const T* A, int64_t lda, const T* B,
                                                 int64_t ldb, float* part, int64_t kchunk) {
  __shared__ float As[BK][BM + 4];
  __shared__ float Bs[BK][BN + 4];
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  const int m0 = blockIdx.x * BM, n0 = blockIdx.y * BN;
  const int64_t kb = (int64_t)blockIdx.z * kchunk, ke = min(K, kb + kchunk);
  float acc[4][4] = {};
  for (int64_t k0 = kb; k0 < ke; k0 += BK) {
    for (int t = threadIdx.x; t < BM * BK; t += 256) {
      int kk = t / BM, mm = t % BM;
      int64_t k = k0 + kk;
      As[kk][mm] = (k < ke && m0 + mm < M) ? tof<T>(A[k * lda + m0 + mm]) : 0.f;
      Bs[kk][mm] = (k < ke && n0 + mm < N) ? tof<T>(B[k * ldb + n0 + mm]) : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < BK; ++kk) {
      float av[4], bv[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) { av[i] = As[kk][ty * 4 + i]; bv[i] = Bs[kk][tx * 4 + i]; }
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
    }
    __syncthreads();
  }
  float* P = part + (int64_t)blockIdx.z * M * N;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    int m = m0 + ty * 4 + i;
    if (m >= M) continue;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      int n = n0 + tx * 4 + j;
      if (n < N) P[(int64_t)m * N + n] = acc[i][j];
    }
  }
}

// grouped: part[u] = the product over unit u's K rows [u.x, u.x + u.y * kb_rows)
template <typename T>
__global__ void __launch_bounds__(256) k_gemm_tn_units(const int4* units, int kb_rows, int M, int N, const T* A,
                                                       int64_t lda, const T* B, int64_t ldb, float* part) {
  __shared__ float As[BK][BM + 4];
  __shared__ float Bs[BK][BN + 4];
  const int tx = threadIdx.x % 16, ty = threadIdx.x / 16;
  const int m0 = blockIdx.x * BM, n0 = blockIdx.y * BN;
  const int4 u = units[blockIdx.z];
  const int64_t kb = u.x, ke = (int64_t)u.x + (int64_t)u.y * kb_rows;
  float acc[4][4] = {};
  for (int64_t k0 = kb; k0 < ke; k0 += BK) {
    for (int t = threadIdx.x; t < BM * BK; t += 256) {
      int kk = t / BM, mm = t % BM;
      int64_t k = k0 + kk;
      As[kk][mm] = (k < ke && m0 + mm < M) ? tof<T>(A[k * lda + m0 + mm]) : 0.f;
      Bs[kk][mm] = (k < ke && n0 + mm < N) ? tof<T>(B[k * ldb + n0 + mm]) : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < BK; ++kk) {
      float av[4], bv[4];
#pragma unroll
      for (int i = 0; i < 4; ++i) { av[i] = As[kk][ty * 4 + i]; bv[i] = Bs[kk][tx * 4 + i]; }
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(av[i], bv[j], acc[i][j]);
    }
    __syncthreads();
  }
  float* P = part + (int64_t)blockIdx.z * M * N;
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    int m = m0 + ty * 4 + i;
    if (m >= M) continue;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      int n = n0 + tx * 4 + j;
      if (n < N) P[(int64_t)m * N + n] = acc[i][j];
    }
  }
}

__global__ void k_units_reduce(const float* part, const int32_t* unit_off, int groups, int64_t MN, float* D) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= MN * groups) return;
  const int64_t g = i / MN, e = i % MN;
  float s = 0.f;
  for (int u = unit_off[g]; u < unit_off[g + 1]; ++u) s += part[(int64_t)u * MN + e];
  D[i] = s;
}

__global__ void k_split_reduce(const float* part, int splits, int64_t MN, float* D, int acc) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= MN) return;
  float s = 0.f;
  for (int z = 0; z < splits; ++z) s += part[z * MN + i];
  D[i] = acc ? D[i] + s : s;
}

int tn_splits(int64_t K, int M, int N) {
  const int64_t tiles = cdiv(M, BM) * cdiv(N, BN);
  int64_t want = std::max<int64_t>(1, (148 * 4) / std::max<int64_t>(1, tiles));
  want = std::min<int64_t>(want, std::max<int64_t>(1, cdiv(K, 512)));
  return (int)std::min<int64_t>(want, 1024);
}

}  // namespace

wg_status gemm_nt(wg_dtype dt, int64_t M, int N, const GemmPart* parts, int n_parts, const GemmEpi& epi,
                  void* scratch, size_t scratch_bytes, cudaStream_t s) {
  (void)scratch; (void)scratch_bytes;
  if (M == 0 || N == 0) return WG_OK;
  WG_REQ(n_parts >= 1 && n_parts <= 3, WG_ERR_INVALID, "gemm_nt: 1..3 parts");
  wg_status st = WG_OK;
  if (tc_gemm_nt(dt, M, N, parts, n_parts, epi, s, &st)) return st;
  // a column-chunked output (exchange layout) is written by the persistent
  // tcgen05 kernel's 3-D store maps only
  WG_REQ(epi.d_chunk_cols <= 0, WG_ERR_UNSUPPORTED, "gemm_nt: chunked output needs the tcgen05 path");
  NTArgs a{};
  a.M = M; a.N = N; a.n_parts = n_parts; a.epi = epi;
  double kt = 0;
  for (int i = 0; i < n_parts; ++i) { a.parts[i] = parts[i]; kt += parts[i].K; }
  const double es = dt == WG_BF16 ? 2.0 : 4.0;
  ProfScope ps(PK_SIMT, s, (double)M * (kt + N) * es, 2.0 * M * N * kt);
  dim3 grid((unsigned)cdiv(M, BM), (unsigned)cdiv(N, BN));
  if (dt == WG_BF16) WG_LAUNCH(k_gemm_nt<__nv_bfloat16>, grid, 256, 0, s, a);
  else WG_LAUNCH(k_gemm_nt<float>, grid, 256, 0, s, a);
  return WG_OK;
}

void make_tn_units(const std::vector<int64_t>& h_off, int64_t target_units, int kb_rows, std::vector<int4>* units,
                   std::vector<int32_t>* unit_off) {
  const int groups = (int)h_off.size() - 1;
  const int64_t total = h_off.back();
  const int64_t span = std::max<int64_t>(kb_rows, rup(cdiv(std::max<int64_t>(total, 1), target_units), kb_rows));
  units->clear();
  unit_off->assign(groups + 1, 0);
  for (int g = 0; g < groups; ++g) {
    (*unit_off)[g] = (int32_t)units->size();
    for (int64_t k = h_off[g]; k < h_off[g + 1]; k += span) {
      const int64_t rows = std::min(span, h_off[g + 1] - k);
      units->push_back(make_int4((int)k, (int)cdiv(rows, kb_rows), g, 0));
    }
  }
  (*unit_off)[groups] = (int32_t)units->size();
}

size_t gemm_tn_grouped_scratch(int n_units, int M, int N) {
  return sizeof(float) * (size_t)std::max(n_units, 1) * M * N;
}

wg_status gemm_tn_grouped(wg_dtype dt, const TnUnits& U, int M, int N, const void* A, int64_t lda, const void* B,
                          int64_t ldb, float* D, void* scratch, cudaStream_t s) {
  if (U.groups == 0 || M == 0 || N == 0) return WG_OK;
  float* part = static_cast<float*>(scratch);
  const int64_t MN = (int64_t)M * N;
  if (U.n_units == 0) {
    WG_CK(cudaMemsetAsync(D, 0, sizeof(float) * MN * U.groups, s));
    return WG_OK;
  }
  wg_status st = WG_OK;
  if (tc_gemm_tn_grouped(dt, U, M, N, A, lda, B, ldb, D, part, s, &st)) return st;
  dim3 grid((unsigned)cdiv(M, BM), (unsigned)cdiv(N, BN), (unsigned)U.n_units);
  ProfScope ps(PK_SIMT, s, (double)U.k_total * (M + N) * (dt == WG_BF16 ? 2.0 : 4.0), 2.0 * U.k_total * M * N);
  const int kb_rows = 128 / (dt == WG_BF16 ? 2 : 4);
  if (dt == WG_BF16)
    WG_LAUNCH(k_gemm_tn_units<__nv_bfloat16>, grid, 256, 0, s, U.units, kb_rows, M, N, (const __nv_bfloat16*)A, lda,
              (const __nv_bfloat16*)B, ldb, part);
  else
    WG_LAUNCH(k_gemm_tn_units<float>, grid, 256, 0, s, U.units, kb_rows, M, N, (const float*)A, lda, (const float*)B,
              ldb, part);
  WG_LAUNCH(k_units_reduce, (unsigned)cdiv(MN * U.groups, 256), 256, 0, s, part, U.unit_off, U.groups, MN, D);
  return WG_OK;
}

size_t gemm_tn_scratch(int64_t K, int M, int N) {
  return sizeof(float) * (size_t)std::max(tn_splits(K, M, N), 160) * M * N;
}

wg_status gemm_tn(wg_dtype dt, int64_t K, int M, int N, const void* A, int64_t lda, const void* B, int64_t ldb,
                  float* D, void* scratch, cudaStream_t s, int acc) {
  if (M == 0 || N == 0) return WG_OK;
  if (K == 0) {
    if (!acc) WG_CK(cudaMemsetAsync(D, 0, sizeof(float) * M * N, s));
    return WG_OK;
  }
  float* part = static_cast<float*>(scratch);
  int splits = tn_splits(K, M, N);
  wg_status st = WG_OK;
  if (tc_gemm_tn(dt, K, M, N, A, lda, B, ldb, D, part, s, &st, acc)) return st;
  const int64_t kchunk = rup(cdiv(K, splits), BK);
  splits = (int)cdiv(K, kchunk);
  ProfScope ps(PK_SIMT, s, (double)K * (M + N) * (dt == WG_BF16 ? 2.0 : 4.0), 2.0 * K * M * N);
  dim3 grid((unsigned)cdiv(M, BM), (unsigned)cdiv(N, BN), (unsigned)splits);
  if (dt == WG_BF16)
    WG_LAUNCH(k_gemm_tn<__nv_bfloat16>, grid, 256, 0, s, K, M, N, (const __nv_bfloat16*)A, lda,
              (const __nv_bfloat16*)B, ldb, part, kchunk);
  else
    WG_LAUNCH(k_gemm_tn<float>, grid, 256, 0, s, K, M, N, (const float*)A, lda, (const float*)B, ldb, part, kchunk);
  const int64_t MN = (int64_t)M * N;
  WG_LAUNCH(k_split_reduce, (unsigned)cdiv(MN, 256), 256, 0, s, part, splits, MN, D, acc);
  return WG_OK;
}

}  // namespace wg
