// tcgen05 / TMEM / TMA GEMMs for sm_100a (bf16 in, fp32 accumulate).
//
// The dense per-gTask / per-vertex transforms of the layer (a5, a7, a9, a11):
// "a batch of K src rows becomes a matrix-matrix product on tensor cores"
// (Fig 10c).  Two variants share one pipeline:
//   NT  D[M x N] = sum_p A_p[M x K_p] B_p[N x K_p]^T   (A, B K-major)
//       + epilogue (row scale, bias, addend, ReLU, ReLU-mask, RNE cast)
//   TN  D[M x N] = A[K x M]^T B[K x N]                   (A, B MN-major)
//       split-K over K (= vertices) with fp32 partials reduced in a fixed
//       order (deterministic weight gradients, a11).
// Structure: one CTA = 128 threads computes a 128 x BN tile.  Thread 0
// issues TMA loads (128-byte swizzle) into a STAGES-deep smem ring guarded by
// full/empty mbarriers; thread 32 issues tcgen05.mma (M=128, N=BN, K=16)
// into a TMEM accumulator and releases ring slots with tcgen05.commit; all
// four warps then drain TMEM with tcgen05.ld (warp w owns lanes 32w..32w+31)
// and run the epilogue.
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <mutex>

#include "wg_internal.cuh"

namespace wg {

namespace {

constexpr int BM = 128, BK = 64;
constexpr int TC_CONV = 256;            // 3xTF32 converter threads (warps 4..11)
constexpr int TC_LO = 3;                // TN 3xTF32: separate lo buffers
constexpr int A_STAGE = BM * BK * 2;   // 16 KB

struct TcParams {
  int64_t M;
  int N;          // columns written (NT) / real N (TN)
  int BN;         // MMA N (multiple of 16, <= 256)
  int stages;
  int nparts;
  int n_tiles;
  int kblocks[3];
  int64_t k_base; // TN: first K row of split z = blockIdx.z * k_span
  int64_t k_span;
  int64_t K;      // TN total K
  const int4* units;  // grouped TN: per blockIdx.z {first K row, k-blocks, -, -}
  int a_stage;        // TN: bytes of the A part of a stage (the real M chunks only)
  int fold;           // TN fp32, M <= 64: A_lo in A's MMA rows 64..127 (2 MMAs per k-step, see the kernel)
  GemmEpi epi;
  float* part;    // TN partial output [splits x M x N]
};

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count));
}

__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}

__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(bar),
      "r"(parity)
      : "memory");
}

__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap* map, int c0, int c1, uint32_t bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(bar)
      : "memory");
}

// UMMA shared-memory descriptor (sm100): start>>4 [0,14), LBO>>4 [16,30),
// SBO>>4 [32,46), version 1 [46,48), layout [61,64): SWIZZLE_128B = 2,
// SWIZZLE_128B_BASE32B = 1 (the only MN-major layout for 32-bit operands:
// 32-byte granules, 4-row atoms; TMA CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B)
__device__ __forceinline__ uint64_t umma_desc(uint32_t addr, uint32_t lbo, uint32_t sbo, uint32_t layout = 2) {
  uint64_t d = 0;
  d |= (uint64_t)((addr >> 4) & 0x3FFF);
  d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)layout << 61;
  return d;
}

__device__ __forceinline__ void umma_bf16(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                          uint32_t accumulate) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n"
      "}\n" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate));
}

__device__ __forceinline__ void umma_commit(uint32_t bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(bar) : "memory");
}

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, float* v) {
  uint32_t r[16];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
}

__device__ __forceinline__ void bf16x8_unpack(const int4& q, float* f) {
  const uint32_t w[4] = {(uint32_t)q.x, (uint32_t)q.y, (uint32_t)q.z, (uint32_t)q.w};
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    f[2 * i] = __uint_as_float(w[i] << 16);
    f[2 * i + 1] = __uint_as_float(w[i] & 0xffff0000u);
  }
}

__device__ __forceinline__ int4 bf16x8_pack(const float* f) {
  uint32_t w[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    __nv_bfloat162 h = __floats2bfloat162_rn(f[2 * i], f[2 * i + 1]);
    w[i] = *reinterpret_cast<uint32_t*>(&h);
  }
  return make_int4((int)w[0], (int)w[1], (int)w[2], (int)w[3]);
}

__device__ __forceinline__ void umma_tf32(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                          uint32_t accumulate) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n"
      "}\n" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate));
}

__device__ __forceinline__ void mbar_arrive1(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}

// 3xTF32 split of one operand region: the lo parts of n16 16-byte units at
// `base` go to `lo` (x itself is the hi operand, see tf32_split_stage);
// 4 units in flight per thread (the converters are the TN's critical stage:
// ncu shows the MMA issuer waiting on them and the TMA producer on free slots)
__device__ __forceinline__ void tf32_split_range(uint32_t base, uint32_t lo, int n16, int ct, int nct) {
  int i = ct;
  for (; i + 3 * nct < n16; i += 4 * nct) {
    uint32_t v[4][4];
#pragma unroll
    for (int u = 0; u < 4; ++u)
      asm volatile("ld.shared.v4.b32 {%0,%1,%2,%3}, [%4];"
                   : "=r"(v[u][0]), "=r"(v[u][1]), "=r"(v[u][2]), "=r"(v[u][3])
                   : "r"(base + (uint32_t)(i + u * nct) * 16u));
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      uint32_t l[4];
#pragma unroll
      for (int k = 0; k < 4; ++k)
        l[k] = __float_as_uint(__uint_as_float(v[u][k]) - __uint_as_float(v[u][k] & 0xffffe000u));
      asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};" ::"r"(lo + (uint32_t)(i + u * nct) * 16u), "r"(l[0]),
                   "r"(l[1]), "r"(l[2]), "r"(l[3]) : "memory");
    }
  }
  for (; i < n16; i += nct) {
    uint32_t v[4], l[4];
    asm volatile("ld.shared.v4.b32 {%0,%1,%2,%3}, [%4];" : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3])
                 : "r"(base + (uint32_t)i * 16u));
#pragma unroll
    for (int k = 0; k < 4; ++k) l[k] = __float_as_uint(__uint_as_float(v[k]) - __uint_as_float(v[k] & 0xffffe000u));
    asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};" ::"r"(lo + (uint32_t)i * 16u), "r"(l[0]), "r"(l[1]), "r"(l[2]),
                 "r"(l[3]) : "memory");
  }
}

// 3xTF32 stage split in shared memory: the lo parts of n16 16-byte units at
// `base` go to base + n16 * 16.  hi needs no rewrite: kind::tf32 reads only
// the top 19 bits of each fp32 operand (truncation -- scripts/tf32_probe.py:
// identical 1e-6 layer errors with and without the masked hi stored), so x
// itself is the hi operand; threads ct = 0..nct-1, explicit
// shared-space vector loads / stores, 4 units in flight per thread
__device__ __forceinline__ void tf32_split_stage(uint32_t base, int n16, int ct, int nct) {
  const uint32_t lo = base + (uint32_t)n16 * 16u;
  int i = ct;
  for (; i + 3 * nct < n16; i += 4 * nct) {
    uint32_t v[4][4];
#pragma unroll
    for (int u = 0; u < 4; ++u)
      asm volatile("ld.shared.v4.b32 {%0,%1,%2,%3}, [%4];"
                   : "=r"(v[u][0]), "=r"(v[u][1]), "=r"(v[u][2]), "=r"(v[u][3])
                   : "r"(base + (uint32_t)(i + u * nct) * 16u));
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      uint32_t h[4], l[4];
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        h[k] = v[u][k] & 0xffffe000u;
        l[k] = __float_as_uint(__uint_as_float(v[u][k]) - __uint_as_float(h[k]));
      }
      const uint32_t off = (uint32_t)(i + u * nct) * 16u;
      asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};" ::"r"(lo + off), "r"(l[0]), "r"(l[1]), "r"(l[2]), "r"(l[3])
                   : "memory");
    }
  }
  for (; i < n16; i += nct) {
    uint32_t v[4], h[4], l[4];
    asm volatile("ld.shared.v4.b32 {%0,%1,%2,%3}, [%4];" : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3])
                 : "r"(base + (uint32_t)i * 16u));
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      h[k] = v[k] & 0xffffe000u;
      l[k] = __float_as_uint(__uint_as_float(v[k]) - __uint_as_float(h[k]));
    }
    asm volatile("st.shared.v4.b32 [%0], {%1,%2,%3,%4};" ::"r"(lo + (uint32_t)i * 16u), "r"(l[0]), "r"(l[1]), "r"(l[2]),
                 "r"(l[3]) : "memory");
  }
}

// MN: TN variant (both operands MN-major, fp32 partial output).  T = float:
// 3xTF32 with eight extra converter warps (threads 128..383) that split each
// landed stage into hi (the landed fp32 itself: kind::tf32 reads its top 19
// bits) and lo.  TN: lo goes to one of TC_LO separate lo buffers (released by
// the MMA commit), so the TMA ring holds raw stages only (5 stages + 3 lo
// buffers instead of 4 stages with in-stage lo twins).
// Stage depth: 128 / sizeof(T) K elements (one 128-byte swizzle row).
template <bool MN, typename T>
__global__ void __launch_bounds__(sizeof(T) == 4 ? 128 + TC_CONV : 128, 1)
    k_tc_gemm(const __grid_constant__ CUtensorMap tA0, const __grid_constant__ CUtensorMap tB0,
              const __grid_constant__ CUtensorMap tA1, const __grid_constant__ CUtensorMap tB1,
              const __grid_constant__ CUtensorMap tA2, const __grid_constant__ CUtensorMap tB2, TcParams p) {
  constexpr bool TF32 = sizeof(T) == 4;
  constexpr int BKE = 128 / sizeof(T);      // K elements per stage
  constexpr int CHE = 128 / sizeof(T);      // MN elements per 128-byte chunk
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int BN = p.BN, S = p.stages;
  const int b_stage = MN ? ((BN + CHE - 1) / CHE) * BKE * 128 : BN * 128;
  // TN stages hold only the A chunks with real M columns (M = f_in = 64: 8 KB
  // of A per fp32 stage, so twice the stages fit -- the TN ring is latency-bound)
  const int a_stage = MN ? p.a_stage : A_STAGE;
  constexpr bool LOBUF = TF32 && MN;            // lo in separate buffers
  const int raw = a_stage + b_stage;
  const int stage = (TF32 && !MN) ? 2 * raw : raw;
  // M fold (TN fp32, M <= 64): the converters write A_lo into the stage's
  // MMA rows 64..127 (A chunks 2, 3), so one M = 128 MMA computes
  // [A_hi; A_lo]^T B and a k-step needs 2 MMAs (B_hi, B_lo) instead of 3 --
  // the 3xTF32 GEMMs are bound by shared-memory operand reads
  // (profiles/r02/tn_bound_experiment.md); the epilogue adds rows m and m + 64.
  // The lo buffers then hold B_lo only.
  const bool fold = LOBUF && p.fold;
  const int lo_stride = fold ? b_stage : raw;
  uint8_t* ring = smem;
  uint8_t* lo_buf = ring + S * stage;           // LOBUF: [TC_LO][A_lo | B_lo] (fold: [TC_LO][B_lo])
  uint64_t* bars = reinterpret_cast<uint64_t*>(lo_buf + (LOBUF ? TC_LO * lo_stride : 0));
  uint64_t* full = bars;                        // [S <= 8]
  uint64_t* empty = bars + 8;
  uint64_t* conv = bars + 16;
  uint64_t* lo_empty = bars + 24;               // [TC_LO <= 4]
  uint64_t* accf = bars + 28;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 29);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  uint32_t tcols = 32;
  while ((int)tcols < BN) tcols <<= 1;

  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(smem_u32(&full[s]), 1);
      mbar_init(smem_u32(&empty[s]), 1);
      mbar_init(smem_u32(&conv[s]), TC_CONV);
    }
    for (int j = 0; j < TC_LO; ++j) mbar_init(smem_u32(&lo_empty[j]), 1);
    mbar_init(smem_u32(accf), 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(tmem_slot)),
                 "r"(tcols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
  const uint32_t tmem = *tmem_slot;

  // NT: 1-D grid, N tiles of one M tile adjacent (the A tile is re-read from L2)
  const int64_t m0 = MN ? (int64_t)blockIdx.x * BM : (int64_t)(blockIdx.x / p.n_tiles) * BM;
  const int n0 = MN ? blockIdx.y * BN : (int)(blockIdx.x % p.n_tiles) * BN;
  int total_kb = 0;
  for (int i = 0; i < p.nparts; ++i) total_kb += p.kblocks[i];
  int64_t kz = MN ? p.k_base + (int64_t)blockIdx.z * p.k_span : 0;
  if (MN && p.units) {          // grouped TN: unit z = {first K row, k-blocks}
    const int4 u = p.units[blockIdx.z];
    kz = u.x;
    total_kb = u.y;
  }

  if (threadIdx.x == 0) {
    // ---------------- TMA producer
    // TN: only the A chunks holding real M columns are loaded (M = f_in may
    // be 64: rows >= M of the M=128 MMA read stale shared memory and only
    // feed accumulator rows the epilogue never stores)
    const int a_chunks = MN ? (int)min((int64_t)(BM / CHE), (p.M - m0 + CHE - 1) / CHE) : 0;
    const uint32_t tx = MN ? (uint32_t)(a_chunks * BKE * 128 + b_stage) : (uint32_t)(A_STAGE + b_stage);
    int part = 0, kk = 0;
    for (int kb = 0; kb < total_kb; ++kb) {
      const int s = kb % S;
      const uint32_t ph = (kb / S) & 1;
      mbar_wait(smem_u32(&empty[s]), ph ^ 1);
      mbar_expect_tx(smem_u32(&full[s]), tx);
      const uint32_t fb = smem_u32(&full[s]);
      const uint32_t ad = smem_u32(ring + s * stage), bd = ad + a_stage;
      if (MN) {
        const int krow = (int)(kz + (int64_t)kb * BKE);
#pragma unroll
        for (int j = 0; j < a_chunks; ++j) tma_load_2d(ad + j * BKE * 128, &tA0, (int)m0 + CHE * j, krow, fb);
        for (int j = 0; j * CHE < BN; ++j) tma_load_2d(bd + j * BKE * 128, &tB0, n0 + CHE * j, krow, fb);
      } else {
        const CUtensorMap* ta = part == 0 ? &tA0 : (part == 1 ? &tA1 : &tA2);
        const CUtensorMap* tb = part == 0 ? &tB0 : (part == 1 ? &tB1 : &tB2);
        tma_load_2d(ad, ta, kk * BKE, (int)m0, fb);
        tma_load_2d(bd, tb, kk * BKE, n0, fb);
        if (++kk == p.kblocks[part]) { kk = 0; ++part; }
      }
    }
  } else if (threadIdx.x == 32) {
    // ---------------- MMA issuer
    // instruction descriptor: D f32 [4,6)=1, A / B format [7,10) / [10,13)
    // (bf16 = 1, tf32 = 2), A/B major [15],[16], N>>3 [17,23), M>>4 [24,29)
    const uint32_t fmt = TF32 ? 2u : 1u;
    const uint32_t idesc = (1u << 4) | (fmt << 7) | (fmt << 10) | ((MN ? 1u : 0u) << 15) | ((MN ? 1u : 0u) << 16) |
                           ((uint32_t)(BN >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
    for (int kb = 0; kb < total_kb; ++kb) {
      const int s = kb % S;
      const uint32_t ph = (kb / S) & 1;
      mbar_wait(smem_u32(TF32 ? &conv[s] : &full[s]), ph);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      const uint32_t ad = smem_u32(ring + s * stage), bd = ad + a_stage;
      const uint32_t al = LOBUF ? smem_u32(lo_buf + (kb % TC_LO) * lo_stride) : bd + b_stage;
      const uint32_t bl = fold ? al : al + a_stage;
#pragma unroll
      for (int k = 0; k < 4; ++k) {   // 4 MMAs of 32 bytes of K (16 bf16 / 8 tf32)
        // MN-major: LBO = next 128-byte MN chunk, SBO = next K atom (8 rows
        // SW128 / 4 rows SW128_BASE32B for tf32); K-major SW128: K step =
        // +32 bytes inside the atom
        const uint32_t step = MN ? (uint32_t)(k * (32 / sizeof(T)) * 128) : (uint32_t)(k * 32);
        const uint32_t lbo = MN ? BKE * 128 : 16;
        const uint32_t sbo = (MN && TF32) ? 512 : 1024;
        const uint32_t lay = (MN && TF32) ? 1 : 2;
        const uint32_t on = (kb | k) != 0 ? 1u : 0u;
        if constexpr (TF32) {
          umma_tf32(tmem, umma_desc(ad + step, lbo, sbo, lay), umma_desc(bd + step, lbo, sbo, lay), idesc, on);
          umma_tf32(tmem, umma_desc(ad + step, lbo, sbo, lay), umma_desc(bl + step, lbo, sbo, lay), idesc, 1u);
          if (!fold)
            umma_tf32(tmem, umma_desc(al + step, lbo, sbo, lay), umma_desc(bd + step, lbo, sbo, lay), idesc, 1u);
        } else {
          umma_bf16(tmem, umma_desc(ad + step, lbo, sbo, lay), umma_desc(bd + step, lbo, sbo, lay), idesc, on);
        }
      }
      umma_commit(smem_u32(&empty[s]));
      if (LOBUF) umma_commit(smem_u32(&lo_empty[kb % TC_LO]));
    }
    umma_commit(smem_u32(accf));
  } else if (TF32 && warp >= 4) {
    // ---------------- hi / lo converters
    const int ct = threadIdx.x - 128;
    const int n16 = (a_stage + b_stage) / 16;
    const int a16 = MN ? (int)min((int64_t)(BM / CHE), (p.M - m0 + CHE - 1) / CHE) * BKE * 8 : 0;
    for (int kb = 0; kb < total_kb; ++kb) {
      const int s = kb % S;
      mbar_wait(smem_u32(&full[s]), (kb / S) & 1);
      if (MN) {   // stage [A | B] -> lo buffer kb % TC_LO [A_lo | B_lo], once the MMAs of kb - TC_LO released it
        mbar_wait(smem_u32(&lo_empty[kb % TC_LO]), ((kb / TC_LO) & 1) ^ 1);
        const uint32_t ad = smem_u32(ring + s * stage), bd = ad + a_stage;
        const uint32_t lb = smem_u32(lo_buf + (kb % TC_LO) * lo_stride);
        if (fold) {
          tf32_split_range(ad, ad + 2 * BKE * 128, a16, ct, TC_CONV);   // A_lo -> MMA rows 64..127
          tf32_split_range(bd, lb, b_stage / 16, ct, TC_CONV);
        } else {
          tf32_split_range(ad, lb, a16, ct, TC_CONV);
          tf32_split_range(bd, lb + a_stage, b_stage / 16, ct, TC_CONV);
        }
      } else {
        tf32_split_stage(smem_u32(ring + s * stage), n16, ct, TC_CONV);
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      mbar_arrive1(smem_u32(&conv[s]));
    }
  }
  __syncwarp();
  if (warp < 4) {
    // ---------------- epilogue: warp w owns TMEM lanes / tile rows 32w..32w+31
    mbar_wait(smem_u32(accf), 0);
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const int r = warp * 32 + lane;
    const int64_t m = m0 + r;
    const GemmEpi& e = p.epi;
    const float rs = (!MN && e.rscale && m < p.M) ? e.rscale[m] : 1.f;
    float* fb = reinterpret_cast<float*>(ring);   // fold: rows 64..127 (the ring is idle after accf)
    const int ldf = BN + 1;
    if (fold) {
      if (warp >= 2) {
        for (int c0 = 0; c0 < BN; c0 += 16) {
          float v[16];
          tmem_ld16(tmem + ((uint32_t)(warp * 32) << 16) + (uint32_t)c0, v);
#pragma unroll
          for (int i = 0; i < 16; ++i) fb[(r - 64) * ldf + c0 + i] = v[i];
        }
      }
      asm volatile("bar.sync 1, 128;" ::: "memory");   // the four epilogue warps
    }
    for (int c0 = 0; c0 < BN; c0 += 16) {
      if (fold && warp >= 2) break;
      float v[16];
      tmem_ld16(tmem + ((uint32_t)(warp * 32) << 16) + (uint32_t)c0, v);
      if (m >= p.M) continue;
      if (fold) {
#pragma unroll
        for (int i = 0; i < 16; ++i) v[i] += fb[r * ldf + c0 + i];   // A_hi^T B + A_lo^T B
      }
      if (MN) {
        float* out = p.part + (int64_t)blockIdx.z * p.M * p.N + m * p.N;
#pragma unroll
        for (int i = 0; i < 16; ++i) {
          const int n = n0 + c0 + i;
          if (n < p.N) out[n] = v[i];
        }
        continue;
      }
      if constexpr (!TF32) {
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int n = n0 + c0 + 8 * h;
          if (n >= p.N) continue;
          float* f = v + 8 * h;
#pragma unroll
          for (int i = 0; i < 8; ++i) f[i] *= (e.D2 && n >= e.n_split) ? 1.f : rs;
          if (e.addend) {
            float t[8];
            bf16x8_unpack(*reinterpret_cast<const int4*>(static_cast<const __nv_bfloat16*>(e.addend) + m * e.ld_add + n), t);
#pragma unroll
            for (int i = 0; i < 8; ++i) f[i] += t[i];
          }
          if (e.bias) {
#pragma unroll
            for (int i = 0; i < 8; ++i) f[i] += (n + i < p.N) ? e.bias[n + i] : 0.f;
          }
          if (e.relu) {
#pragma unroll
            for (int i = 0; i < 8; ++i) f[i] = fmaxf(f[i], 0.f);
          }
          if (e.mask_ref) {
            float t[8];
            bf16x8_unpack(*reinterpret_cast<const int4*>(static_cast<const __nv_bfloat16*>(e.mask_ref) + m * e.ld_mask + n), t);
#pragma unroll
            for (int i = 0; i < 8; ++i) f[i] = t[i] > 0.f ? f[i] : 0.f;
          }
          void* Dp = e.D;
          int64_t ld = e.ldd, nn = n;
          if (e.D2 && n >= e.n_split) { Dp = e.D2; ld = e.ldd2; nn = n - e.n_split; }
          if (e.d_f32) {
            float* o = static_cast<float*>(Dp) + m * ld + nn;
#pragma unroll
            for (int i = 0; i < 8; ++i) o[i] = f[i];
          } else {
            *reinterpret_cast<int4*>(static_cast<__nv_bfloat16*>(Dp) + m * ld + nn) = bf16x8_pack(f);
          }
        }
      }
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(tcols));
}

__global__ void k_split_reduce_tc(const float* part, int splits, int64_t MN, float* D, int acc) {
  int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= MN) return;
  float s = 0.f;
#pragma unroll 8
  for (int z = 0; z < splits; ++z) s += part[z * MN + i];   // 8 loads in flight, split order
  D[i] = acc ? D[i] + s : s;
}

PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  });
  return fn;
}

// 2-D tensor map, 128-byte swizzle; dims {inner, outer}, row pitch ld_bytes
bool make_map_t(CUtensorMap* m, CUtensorMapDataType ty, const void* ptr, uint64_t inner, uint64_t outer,
                uint64_t ld_bytes, uint32_t box_in, uint32_t box_out,
                CUtensorMapSwizzle swz = CU_TENSOR_MAP_SWIZZLE_128B) {
  auto fn = encode_fn();
  if (!fn) return false;
  if ((reinterpret_cast<uintptr_t>(ptr) & 15) || (ld_bytes & 15)) return false;
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {ld_bytes};
  cuuint32_t box[2] = {box_in, box_out};
  cuuint32_t estr[2] = {1, 1};
  return fn(m, ty, 2, const_cast<void*>(ptr), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, swz,
            CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}
bool make_map(CUtensorMap* m, const void* ptr, uint64_t inner, uint64_t outer, uint64_t ld_bytes, uint32_t box_in,
              uint32_t box_out) {
  return make_map_t(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, ptr, inner, outer, ld_bytes, box_in, box_out);
}

int g_tc_disabled = -1;
bool tc_enabled() {
  if (g_tc_disabled < 0) {
    const char* e = getenv("WG_DISABLE_TC");
    g_tc_disabled = (e && e[0] == '1') ? 1 : 0;
  }
  return !g_tc_disabled;
}

size_t smem_bytes(bool mn, int BN, int stages, int es = 2, int a_stage = A_STAGE, bool fold = false) {
  const int che = 128 / es, bke = 128 / es;
  const int b_stage = mn ? ((BN + che - 1) / che) * bke * 128 : BN * 128;
  const size_t raw = (mn ? a_stage : A_STAGE) + b_stage;
  const size_t lo = fold ? (size_t)b_stage : raw;   // fold: the lo buffers hold B_lo only
  // the M = 128 MMA reads 16 KB of A from every stage / lo buffer start: slack
  // keeps the rows past a short A part (never stored) inside the allocation
  const size_t slack = mn ? (size_t)(A_STAGE - a_stage) : 0;
  if (es == 4 && mn) return 1024 + (size_t)stages * raw + TC_LO * lo + 256 + slack;   // raw ring + lo buffers
  return 1024 + (size_t)stages * raw * (es == 4 ? 2 : 1) + 256 + slack;
}

template <bool MN, typename T>
wg_status launch(dim3 grid, size_t smem, const CUtensorMap* maps, const TcParams& p, cudaStream_t s) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(k_tc_gemm<MN, T>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    attr = true;
  }
  WG_LAUNCH((k_tc_gemm<MN, T>), grid, sizeof(T) == 4 ? 128 + TC_CONV : 128, smem, s, maps[0], maps[1], maps[2], maps[3], maps[4],
            maps[5], p);
  return WG_OK;
}

}  // namespace

bool tc_make_map_t(CUtensorMap* m, CUtensorMapDataType ty, const void* ptr, uint64_t inner, uint64_t outer,
                   uint64_t ld_bytes, uint32_t box_in, uint32_t box_out) {
  return make_map_t(m, ty, ptr, inner, outer, ld_bytes, box_in, box_out);
}

// 3-D tensor map {inner, outer, chunks} (128-byte swizzle): a column-chunked
// output table [chunks][outer][inner]; chunk_bytes = 0 when chunks == 1
bool tc_make_map3_t(CUtensorMap* m, CUtensorMapDataType ty, const void* ptr, uint64_t inner, uint64_t outer,
                    uint64_t chunks, uint64_t ld_bytes, uint64_t chunk_bytes, uint32_t box_in, uint32_t box_out) {
  auto fn = encode_fn();
  if (!fn) return false;
  if (chunks <= 1) chunk_bytes = ld_bytes * std::max<uint64_t>(outer, 1);
  if ((reinterpret_cast<uintptr_t>(ptr) & 15) || (ld_bytes & 15) || (chunk_bytes & 15)) return false;
  cuuint64_t dims[3] = {inner, outer, std::max<uint64_t>(chunks, 1)};
  cuuint64_t strides[2] = {ld_bytes, chunk_bytes};
  cuuint32_t box[3] = {box_in, box_out, 1};
  cuuint32_t estr[3] = {1, 1, 1};
  return fn(m, ty, 3, const_cast<void*>(ptr), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
            CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

bool tc_gemm_nt_persistent(wg_dtype dt, int64_t M, int N, const GemmPart* parts, int n_parts, const GemmEpi& epi,
                           cudaStream_t s, wg_status* st);

bool tc_gemm_nt(wg_dtype dt, int64_t M, int N, const GemmPart* parts, int n_parts, const GemmEpi& epi,
                cudaStream_t s, wg_status* st) {
  if (!tc_enabled() || n_parts > 3 || M <= 0) return false;
  if (tc_gemm_nt_persistent(dt, M, N, parts, n_parts, epi, s, st)) return true;
  if (dt != WG_BF16 || epi.d_chunk_cols > 0) return false;
  for (int i = 0; i < n_parts; ++i)
    if (parts[i].tile_group || parts[i].a_rows) return false;   // grouped B / gathered A: persistent kernel only
  const int n_tiles = (int)cdiv(N, 256);
  const int BN = (int)rup(cdiv(N, n_tiles), 16);
  if (BN > 256) return false;
  CUtensorMap maps[6];
  memset(maps, 0, sizeof(maps));
  TcParams p{};
  p.M = M; p.N = N; p.BN = BN; p.nparts = n_parts; p.epi = epi; p.n_tiles = n_tiles;
  for (int i = 0; i < n_parts; ++i) {
    const GemmPart& q = parts[i];
    if (!make_map(&maps[2 * i], q.A, (uint64_t)q.K, (uint64_t)M, (uint64_t)q.lda * 2, BK, BM)) return false;
    if (!make_map(&maps[2 * i + 1], q.B, (uint64_t)q.K, (uint64_t)q.nb, (uint64_t)q.ldb * 2, BK, BN))
      return false;
    p.kblocks[i] = (int)cdiv(q.K, BK);
  }
  for (int i = n_parts; i < 3; ++i) { maps[2 * i] = maps[0]; maps[2 * i + 1] = maps[1]; }
  if ((epi.addend && ((uintptr_t)epi.addend & 15)) || ((uintptr_t)epi.D & 15)) return false;
  int stages = 4;
  while (stages > 2 && smem_bytes(false, BN, stages) > 110 * 1024) --stages;
  p.stages = stages;
  dim3 grid((unsigned)(cdiv(M, BM) * n_tiles), 1, 1);
  double kt = 0;
  for (int i = 0; i < n_parts; ++i) kt += parts[i].K;
  ProfScope ps(PK_TC_NT, s, (double)M * (kt + N + (epi.addend ? N : 0) + (epi.mask_ref ? N : 0)) * 2.0,
               2.0 * M * N * kt);
  *st = launch<false, __nv_bfloat16>(grid, smem_bytes(false, BN, stages), maps, p, s);
  return true;
}

namespace {
// TN map pair + launch geometry shared by the plain and grouped TN GEMMs
struct TnSetup {
  CUtensorMap maps[6];
  int BN, n_tiles, m_tiles, stages, es, a_stage, fold;
  size_t smem;
};

bool tn_setup(wg_dtype dt, int64_t K, int M, int N, const void* A, int64_t lda, const void* B, int64_t ldb,
              TnSetup* t) {
  t->es = dt == WG_F32 ? 4 : 2;
  const CUtensorMapDataType ty = dt == WG_F32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16;
  const int che = 128 / t->es, bke = 128 / t->es;
  const int bn_max = dt == WG_F32 ? 128 : 256;
  t->n_tiles = (int)cdiv(N, bn_max);
  t->BN = (int)rup(cdiv(N, t->n_tiles), 16);
  t->m_tiles = (int)cdiv(M, BM);
  memset(t->maps, 0, sizeof(t->maps));
  // MN-major 32-bit operands: the 32-byte-granule 128-byte swizzle (see umma_desc)
  const CUtensorMapSwizzle swz = dt == WG_F32 ? CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B : CU_TENSOR_MAP_SWIZZLE_128B;
  if (!make_map_t(&t->maps[0], ty, A, (uint64_t)M, (uint64_t)K, (uint64_t)lda * t->es, che, bke, swz)) return false;
  if (!make_map_t(&t->maps[1], ty, B, (uint64_t)N, (uint64_t)K, (uint64_t)ldb * t->es, che, bke, swz)) return false;
  for (int i = 2; i < 6; ++i) t->maps[i] = t->maps[i & 1];
  // fp32 with M <= 64: fold A_lo into the M = 128 MMA's idle rows (kernel comment)
  static int fold_env = -1;
  if (fold_env < 0) {
    const char* e = getenv("WG_TN_FOLD");
    fold_env = (e && e[0] == '0') ? 0 : 1;
  }
  t->fold = (t->es == 4 && M <= 64 && fold_env) ? 1 : 0;
  t->a_stage = t->fold ? A_STAGE : (int)std::min<int64_t>(BM / che, cdiv(M, che)) * bke * 128;
  t->stages = t->es == 4 ? 8 : 4;
  while (t->stages > 2 && smem_bytes(true, t->BN, t->stages, t->es, t->a_stage, t->fold) > 200 * 1024) --t->stages;
  t->smem = smem_bytes(true, t->BN, t->stages, t->es, t->a_stage, t->fold);
  return t->smem <= 227 * 1024;
}

wg_status tn_launch(wg_dtype dt, const TnSetup& t, dim3 grid, const TcParams& p, cudaStream_t s) {
  return dt == WG_F32 ? launch<true, float>(grid, t.smem, t.maps, p, s)
                      : launch<true, __nv_bfloat16>(grid, t.smem, t.maps, p, s);
}

}  // namespace

bool tc_gemm_tn(wg_dtype dt, int64_t K, int M, int N, const void* A, int64_t lda, const void* B, int64_t ldb,
                float* D, float* part, cudaStream_t s, wg_status* st, int acc) {
  if (!tc_enabled() || K <= 0) return false;
  TnSetup t;
  if (!tn_setup(dt, K, M, N, A, lda, B, ldb, &t)) return false;
  const int bke = 128 / t.es;
  // split K so that the grid is one full wave (one CTA per SM: the 3-4-stage
  // ring takes most of shared memory).  A 160-split grid ran as 148 + 12
  // CTAs, i.e. two waves (C3 dW_0: 0.64 ms at 2.3 TB/s)
  const int tiles = t.m_tiles * t.n_tiles;
  int64_t splits = std::max<int64_t>(1, 148 / tiles);
  splits = std::min<int64_t>(splits, cdiv(K, bke));
  splits = std::min<int64_t>(splits, 160);
  const int64_t span = rup(cdiv(K, splits), bke);
  splits = cdiv(K, span);
  TcParams p{};
  p.M = M; p.N = N; p.BN = t.BN; p.nparts = 1; p.kblocks[0] = (int)(span / bke);
  p.k_base = 0; p.k_span = span; p.K = K; p.part = part; p.stages = t.stages; p.a_stage = t.a_stage;
  p.fold = t.fold;
  dim3 grid((unsigned)t.m_tiles, (unsigned)t.n_tiles, (unsigned)splits);
  ProfScope ps(PK_TC_TN, s, (double)K * (M + N) * t.es + (double)M * N * 4.0, 2.0 * K * M * N);
  *st = tn_launch(dt, t, grid, p, s);
  if (*st != WG_OK) return true;
  const int64_t MN = (int64_t)M * N;
  k_split_reduce_tc<<<(unsigned)cdiv(MN, 256), 256, 0, s>>>(part, (int)splits, MN, D, acc);
  ++launch_counter();
  if (cudaGetLastError() != cudaSuccess) *st = WG_ERR_CUDA;
  return true;
}

namespace {
// D[g] = sum of the partials of group g's units, in unit order (deterministic)
__global__ void k_unit_reduce(const float* part, const int32_t* unit_off, int groups, int64_t MN, float* D) {
  const int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
  if (i >= MN * groups) return;
  const int64_t g = i / MN, e = i % MN;
  float s = 0.f;
#pragma unroll 8
  for (int u = unit_off[g]; u < unit_off[g + 1]; ++u) s += part[(int64_t)u * MN + e];
  D[i] = s;
}
}  // namespace

bool tc_gemm_tn_grouped(wg_dtype dt, const TnUnits& U, int M, int N, const void* A, int64_t lda, const void* B,
                        int64_t ldb, float* D, float* part, cudaStream_t s, wg_status* st) {
  if (!tc_enabled() || U.n_units <= 0 || U.align % (128 / (dt == WG_F32 ? 4 : 2)) != 0) return false;
  TnSetup t;
  if (!tn_setup(dt, U.k_total, M, N, A, lda, B, ldb, &t)) return false;
  TcParams p{};
  p.M = M; p.N = N; p.BN = t.BN; p.nparts = 1; p.K = U.k_total; p.part = part; p.stages = t.stages;
  p.a_stage = t.a_stage;
  p.fold = t.fold;
  p.units = U.units;
  dim3 grid((unsigned)t.m_tiles, (unsigned)t.n_tiles, (unsigned)U.n_units);
  ProfScope ps(PK_TC_TN, s, (double)U.k_total * (M + N) * t.es + (double)U.n_units * M * N * 4.0,
               2.0 * U.k_total * M * N);
  *st = tn_launch(dt, t, grid, p, s);
  if (*st != WG_OK) return true;
  const int64_t MN = (int64_t)M * N;
  k_unit_reduce<<<(unsigned)cdiv(MN * U.groups, 256), 256, 0, s>>>(part, U.unit_off, U.groups, MN, D);
  ++launch_counter();
  if (cudaGetLastError() != cudaSuccess) *st = WG_ERR_CUDA;
  return true;
}

}  // namespace wg
