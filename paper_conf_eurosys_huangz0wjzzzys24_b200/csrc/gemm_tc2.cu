// Persistent, warp-specialized tcgen05 GEMM (NT, bf16) with a TMA epilogue.
//
//   D[M x N] = sum_p A_p[M x K_p] B_p[N x K_p]^T  (+ row scale, bias, addend, ReLU, ReLU-mask)
//
// These layer transforms are HBM-bound (K <= 512), so what matters is keeping
// loads, MMAs and the output stream overlapped across tiles:
//   warp 0      TMA producer: A/B k-blocks of all of this CTA's tiles into an
//               S-stage shared-memory ring (full / empty mbarriers);
//   warp 1      TMEM allocator + MMA issuer: tcgen05.mma (M=128, N=BN, K=16)
//               into one of TWO accumulator buffers (2 x BN TMEM columns), so
//               tile i+1's MMAs run while tile i is drained;
//   warp 6      epilogue loader: TMA loads of the addend / mask tiles, 64
//               columns at a time, into a 2-deep buffer;
//   warps 2-5   epilogue: tcgen05.ld (warp w drains TMEM lanes 32*(w%4)..),
//               fused epilogue math, bf16 pack into a 128-byte-swizzled staging
//               tile, TMA store (bulk_group, 2-deep) -- coalesced writes.
// One CTA per SM loops over 128 x BN tiles (N fastest, so A tiles of the N
// tiles of one row block are adjacent in time).
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstring>
#include <mutex>

#include "wg_internal.cuh"

namespace wg {

bool tc_make_map(CUtensorMap* m, const void* ptr, uint64_t inner, uint64_t outer, uint64_t ld_bytes, uint32_t box_in,
                 uint32_t box_out);
bool tc_enabled_pub();

namespace {

constexpr int BM = 128, BK = 64, CH = 64;          // CH: epilogue column chunk (one 128-B swizzle box)
constexpr int A_STAGE = BM * BK * 2;               // 16 KB
constexpr int CHUNK_BYTES = BM * CH * 2;           // 16 KB
constexpr int NTHREADS = 224;                      // 7 warps

struct P2 {
  int64_t M;
  int N, BN, n_tiles, stages, nparts, n_split;
  int64_t num_tiles;
  int kblocks[3];
  const float* rscale;
  const float* bias;
  int relu, has_add, has_mask;
};

__device__ __forceinline__ uint32_t su32(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }
__device__ __forceinline__ void mbar_init(uint32_t b, uint32_t c) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(b), "r"(c));
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(b) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t b, uint32_t parity) {
  asm volatile(
      "{\n.reg .pred p;\nW_%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W_%=;\n}\n" ::"r"(b),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_load(uint32_t dst, const CUtensorMap* m, int c0, int c1, uint32_t bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::
          "r"(dst), "l"(reinterpret_cast<uint64_t>(m)), "r"(c0), "r"(c1), "r"(bar)
      : "memory");
}
__device__ __forceinline__ void tma_store(const CUtensorMap* m, int c0, int c1, uint32_t src) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];" ::"l"(
                   reinterpret_cast<uint64_t>(m)),
               "r"(c0), "r"(c1), "r"(src)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void epi_bar() { asm volatile("bar.sync 1, 128;" ::: "memory"); }

__device__ __forceinline__ uint64_t desc_sw128(uint32_t addr) {
  uint64_t d = 0;
  d |= (uint64_t)((addr >> 4) & 0x3FFF);
  d |= (uint64_t)1 << 16;                  // LBO (unused for swizzled K-major)
  d |= (uint64_t)(1024 >> 4) << 32;        // SBO: 8 rows x 128 B
  d |= (uint64_t)1 << 46;                  // sm100 descriptor version
  d |= (uint64_t)2 << 61;                  // SWIZZLE_128B
  return d;
}
__device__ __forceinline__ void mma(uint32_t tmem, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(tmem),
      "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void mma_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void tmem_ld16(uint32_t taddr, uint32_t* r) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
        "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
}

// element offset of (row r, col c) inside a [128 x 64] bf16 tile with 128-byte swizzle
__device__ __forceinline__ uint32_t sw_off(int r, int c) {
  return (uint32_t)(r * 128 + ((((c >> 3) ^ (r & 7))) << 4) + ((c & 7) << 1));
}

__global__ void __launch_bounds__(NTHREADS, 1)
    k_gemm_nt_p(const __grid_constant__ CUtensorMap tA0, const __grid_constant__ CUtensorMap tB0,
                const __grid_constant__ CUtensorMap tA1, const __grid_constant__ CUtensorMap tB1,
                const __grid_constant__ CUtensorMap tA2, const __grid_constant__ CUtensorMap tB2,
                const __grid_constant__ CUtensorMap tD, const __grid_constant__ CUtensorMap tD2,
                const __grid_constant__ CUtensorMap tAdd, const __grid_constant__ CUtensorMap tMask, P2 p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int BN = p.BN, S = p.stages;
  const int b_stage = BN * 128;
  uint8_t* a_sm = smem;
  uint8_t* b_sm = a_sm + S * A_STAGE;
  uint8_t* st_sm = b_sm + S * b_stage;             // 2 x 16 KB output staging
  uint8_t* ad_sm = st_sm + 2 * CHUNK_BYTES;        // 2 x 16 KB addend
  uint8_t* mk_sm = ad_sm + 2 * CHUNK_BYTES;        // 2 x 16 KB mask
  uint64_t* bars = reinterpret_cast<uint64_t*>(mk_sm + 2 * CHUNK_BYTES);
  uint64_t* full = bars;            // [4]
  uint64_t* empty = bars + 4;       // [4]
  uint64_t* tfull = bars + 8;       // [2]
  uint64_t* tempty = bars + 10;     // [2]
  uint64_t* efull = bars + 12;      // [2]
  uint64_t* eempty = bars + 14;     // [2]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 16);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nchunk = (BN + CH - 1) / CH;

  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) { mbar_init(su32(&full[s]), 1); mbar_init(su32(&empty[s]), 1); }
    for (int b = 0; b < 2; ++b) {
      mbar_init(su32(&tfull[b]), 1);
      mbar_init(su32(&tempty[b]), 128);
      mbar_init(su32(&efull[b]), 1);
      mbar_init(su32(&eempty[b]), 128);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 1) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(su32(tmem_slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = *tmem_slot;
  int total_kb = 0;
  for (int i = 0; i < p.nparts; ++i) total_kb += p.kblocks[i];

  if (warp == 0) {
    if (lane == 0) {
      // ------------------------------------------------ TMA producer
      const uint32_t tx = A_STAGE + b_stage;
      int s = 0;
      uint32_t ph = 0;
      for (int64_t t = blockIdx.x; t < p.num_tiles; t += gridDim.x) {
        const int m0 = (int)((t / p.n_tiles) * BM), n0 = (int)((t % p.n_tiles) * BN);
        int part = 0, kk = 0;
        for (int kb = 0; kb < total_kb; ++kb) {
          mbar_wait(su32(&empty[s]), ph ^ 1);
          mbar_expect_tx(su32(&full[s]), tx);
          const CUtensorMap* ta = part == 0 ? &tA0 : (part == 1 ? &tA1 : &tA2);
          const CUtensorMap* tb = part == 0 ? &tB0 : (part == 1 ? &tB1 : &tB2);
          tma_load(su32(a_sm + s * A_STAGE), ta, kk * BK, m0, su32(&full[s]));
          tma_load(su32(b_sm + s * b_stage), tb, kk * BK, n0, su32(&full[s]));
          if (++kk == p.kblocks[part]) { kk = 0; ++part; }
          if (++s == S) { s = 0; ph ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      // ------------------------------------------------ MMA issuer
      const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(BN >> 3) << 17) |
                             ((uint32_t)(BM >> 4) << 24);
      int s = 0;
      uint32_t ph = 0;
      int j = 0;
      for (int64_t t = blockIdx.x; t < p.num_tiles; t += gridDim.x, ++j) {
        const int buf = j & 1;
        mbar_wait(su32(&tempty[buf]), ((j >> 1) & 1) ^ 1);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        const uint32_t acc = tmem + (uint32_t)(buf * 256);
        for (int kb = 0; kb < total_kb; ++kb) {
          mbar_wait(su32(&full[s]), ph);
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
          const uint32_t ad = su32(a_sm + s * A_STAGE), bd = su32(b_sm + s * b_stage);
#pragma unroll
          for (int k = 0; k < BK / 16; ++k)
            mma(acc, desc_sw128(ad + k * 32), desc_sw128(bd + k * 32), idesc, (kb | k) != 0 ? 1u : 0u);
          mma_commit(su32(&empty[s]));
          if (++s == S) { s = 0; ph ^= 1; }
        }
        mma_commit(su32(&tfull[buf]));
      }
    }
  } else if (warp == 6) {
    if (lane == 0 && (p.has_add || p.has_mask)) {
      // ------------------------------------------------ epilogue loader
      const uint32_t tx = (p.has_add ? CHUNK_BYTES : 0) + (p.has_mask ? CHUNK_BYTES : 0);
      int g = 0;
      for (int64_t t = blockIdx.x; t < p.num_tiles; t += gridDim.x) {
        const int m0 = (int)((t / p.n_tiles) * BM), n0 = (int)((t % p.n_tiles) * BN);
        for (int c = 0; c < nchunk; ++c, ++g) {
          const int b = g & 1;
          mbar_wait(su32(&eempty[b]), ((g >> 1) & 1) ^ 1);
          mbar_expect_tx(su32(&efull[b]), tx);
          if (p.has_add) tma_load(su32(ad_sm + b * CHUNK_BYTES), &tAdd, n0 + c * CH, m0, su32(&efull[b]));
          if (p.has_mask) tma_load(su32(mk_sm + b * CHUNK_BYTES), &tMask, n0 + c * CH, m0, su32(&efull[b]));
        }
      }
    }
  } else {
    // ------------------------------------------------ epilogue (warps 2..5)
    const int et = threadIdx.x - 64;               // 0..127
    const int quarter = warp & 3;                  // TMEM lane quarter this warp may access
    const int r = quarter * 32 + lane;             // tile row
    const bool epi_loads = p.has_add || p.has_mask;
    int j = 0, g = 0;
    for (int64_t t = blockIdx.x; t < p.num_tiles; t += gridDim.x, ++j) {
      const int m0 = (int)((t / p.n_tiles) * BM), n0 = (int)((t % p.n_tiles) * BN);
      const int buf = j & 1;
      const bool second = p.n_split > 0 && n0 >= p.n_split;
      const CUtensorMap* td = second ? &tD2 : &tD;
      const int ncol0 = second ? n0 - p.n_split : n0;
      const int64_t m = (int64_t)m0 + r;
      const float rs = (p.rscale && m < p.M) ? p.rscale[m] : 1.f;
      mbar_wait(su32(&tfull[buf]), (j >> 1) & 1);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      for (int c = 0; c < nchunk; ++c, ++g) {
        const int b = g & 1;
        uint32_t u[64];
        const uint32_t taddr = tmem + ((uint32_t)(quarter * 32) << 16) + (uint32_t)(buf * 256 + c * CH);
        tmem_ld16(taddr, u);
        tmem_ld16(taddr + 16, u + 16);
        tmem_ld16(taddr + 32, u + 32);
        tmem_ld16(taddr + 48, u + 48);
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        if (epi_loads) mbar_wait(su32(&efull[b]), (g >> 1) & 1);
        // the staging buffer b was last read by the TMA store issued two chunks ago
        if (et == 0) bulk_wait_read<1>();
        epi_bar();
        uint8_t* stg = st_sm + b * CHUNK_BYTES;
        const uint8_t* adp = ad_sm + b * CHUNK_BYTES;
        const uint8_t* mkp = mk_sm + b * CHUNK_BYTES;
#pragma unroll
        for (int k = 0; k < 8; ++k) {           // 8 columns (one 16-byte chunk) at a time
          float f[8];
          const int nc = n0 + c * CH + k * 8;
#pragma unroll
          for (int i = 0; i < 8; ++i) f[i] = rs * __uint_as_float(u[k * 8 + i]);
          if (p.has_add) {
            const int4 q = *reinterpret_cast<const int4*>(adp + sw_off(r, k * 8));
            const uint32_t w[4] = {(uint32_t)q.x, (uint32_t)q.y, (uint32_t)q.z, (uint32_t)q.w};
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              f[2 * i] += __uint_as_float(w[i] << 16);
              f[2 * i + 1] += __uint_as_float(w[i] & 0xffff0000u);
            }
          }
          if (p.bias) {
#pragma unroll
            for (int i = 0; i < 8; ++i) f[i] += (nc + i < p.N) ? p.bias[nc + i] : 0.f;
          }
          if (p.relu) {
#pragma unroll
            for (int i = 0; i < 8; ++i) f[i] = fmaxf(f[i], 0.f);
          }
          if (p.has_mask) {
            const int4 q = *reinterpret_cast<const int4*>(mkp + sw_off(r, k * 8));
            const uint32_t w[4] = {(uint32_t)q.x, (uint32_t)q.y, (uint32_t)q.z, (uint32_t)q.w};
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              if (!(__uint_as_float(w[i] << 16) > 0.f)) f[2 * i] = 0.f;
              if (!(__uint_as_float(w[i] & 0xffff0000u) > 0.f)) f[2 * i + 1] = 0.f;
            }
          }
#pragma unroll
          for (int i = 0; i < 8; ++i) if (nc + i >= p.N) f[i] = 0.f;
          uint32_t pk[4];
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            __nv_bfloat162 h = __floats2bfloat162_rn(f[2 * i], f[2 * i + 1]);
            pk[i] = *reinterpret_cast<uint32_t*>(&h);
          }
          *reinterpret_cast<int4*>(stg + sw_off(r, k * 8)) = make_int4((int)pk[0], (int)pk[1], (int)pk[2], (int)pk[3]);
        }
        if (epi_loads) mbar_arrive(su32(&eempty[b]));
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        epi_bar();
        if (et == 0) {
          tma_store(td, ncol0 + c * CH, m0, su32(stg));
          bulk_commit();
        }
      }
      asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
      mbar_arrive(su32(&tempty[buf]));
    }
    if (et == 0) bulk_wait_all();
  }
  __syncthreads();
  if (warp == 1) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
}

int g_sms = 0;

}  // namespace

size_t gemm_nt_p_smem(int BN, int stages) {
  return 1024 + (size_t)stages * (A_STAGE + BN * 128) + 6 * CHUNK_BYTES + 256;
}

// returns false when the shape / epilogue is not handled (caller falls back)
bool tc_gemm_nt_persistent(int64_t M, int N, const GemmPart* parts, int n_parts, const GemmEpi& epi, cudaStream_t s,
                           wg_status* st) {
  static int disabled = -1;
  if (disabled < 0) {
    const char* e = getenv("WG_GEMM_V1");
    disabled = (e && e[0] == '1') ? 1 : 0;
  }
  if (disabled || epi.d_f32 || n_parts > 3 || M <= 0) return false;
  // several N tiles: BN = 256 so every 64-column store box stays inside its
  // tile (the ragged end is clipped by the tensor map); one tile: BN = N
  const int n_tiles = (int)cdiv(N, 256);
  const int BN = n_tiles > 1 ? 256 : (int)rup(N, 16);
  if (epi.D2 && (epi.n_split % BN != 0)) return false;   // split must fall on a tile boundary
  CUtensorMap maps[10];
  memset(maps, 0, sizeof(maps));
  P2 p{};
  p.M = M; p.N = N; p.BN = BN; p.n_tiles = n_tiles; p.nparts = n_parts;
  p.num_tiles = cdiv(M, BM) * n_tiles;
  for (int i = 0; i < n_parts; ++i) {
    const GemmPart& q = parts[i];
    if (q.tile_group) return false;
    if (!tc_make_map(&maps[2 * i], q.A, (uint64_t)q.K, (uint64_t)M, (uint64_t)q.lda * 2, BK, BM)) return false;
    if (!tc_make_map(&maps[2 * i + 1], q.B, (uint64_t)q.K, (uint64_t)q.nb, (uint64_t)q.ldb * 2, BK, BN)) return false;
    p.kblocks[i] = (int)cdiv(q.K, BK);
  }
  for (int i = n_parts; i < 3; ++i) { maps[2 * i] = maps[0]; maps[2 * i + 1] = maps[1]; }
  const int n1 = epi.D2 ? epi.n_split : N;
  if (!tc_make_map(&maps[6], epi.D, (uint64_t)n1, (uint64_t)M, (uint64_t)epi.ldd * 2, CH, BM)) return false;
  maps[7] = maps[6];
  if (epi.D2) {
    p.n_split = epi.n_split;
    if (!tc_make_map(&maps[7], epi.D2, (uint64_t)(N - epi.n_split), (uint64_t)M, (uint64_t)epi.ldd2 * 2, CH, BM))
      return false;
  }
  maps[8] = maps[9] = maps[6];
  if (epi.addend) {
    if (!tc_make_map(&maps[8], epi.addend, (uint64_t)N, (uint64_t)M, (uint64_t)epi.ld_add * 2, CH, BM)) return false;
    p.has_add = 1;
  }
  if (epi.mask_ref) {
    if (!tc_make_map(&maps[9], epi.mask_ref, (uint64_t)N, (uint64_t)M, (uint64_t)epi.ld_mask * 2, CH, BM)) return false;
    p.has_mask = 1;
  }
  p.rscale = epi.rscale;
  p.bias = epi.bias;
  p.relu = epi.relu;
  int stages = 4;
  while (stages > 2 && gemm_nt_p_smem(BN, stages) > 227 * 1024) --stages;
  if (gemm_nt_p_smem(BN, stages) > 227 * 1024) return false;
  p.stages = stages;
  if (!g_sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&g_sms, cudaDevAttrMultiProcessorCount, dev);
  }
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(k_gemm_nt_p, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    attr = true;
  }
  const unsigned grid = (unsigned)std::min<int64_t>(p.num_tiles, g_sms);
  double kt = 0;
  for (int i = 0; i < n_parts; ++i) kt += parts[i].K;
  ProfScope ps(PK_TC_NT, s, (double)M * (kt + N + (epi.addend ? N : 0) + (epi.mask_ref ? N : 0)) * 2.0,
               2.0 * M * N * kt);
  k_gemm_nt_p<<<grid, NTHREADS, gemm_nt_p_smem(BN, stages), s>>>(maps[0], maps[1], maps[2], maps[3], maps[4],
                                                                 maps[5], maps[6], maps[7], maps[8], maps[9], p);
  ++launch_counter();
  cudaError_t e = cudaGetLastError();
  *st = e == cudaSuccess ? WG_OK : WG_ERR_CUDA;
  if (e != cudaSuccess) set_error(std::string("k_gemm_nt_p: ") + cudaGetErrorString(e));
  return true;
}

}  // namespace wg
