// Persistent, warp-specialized tcgen05 GEMM (NT) with a TMA epilogue.
//
//   D[M x N] = sum_p A_p[M x K_p] B_p[N x K_p]^T  (+ row scale, bias, addend, ReLU, ReLU-mask)
//
// bf16: kind::f16.  fp32: 3xTF32 (kind::tf32): every operand x = hi + lo with
// hi = x with its 13 low mantissa bits cleared and lo = x - hi (exact), and
// D += A_hi B_hi + A_hi B_lo + A_lo B_hi (the dropped lo*lo term is ~2^-22
// relative), so fp32 layers keep fp32-level accuracy on tensor cores.  The
// split runs in shared memory: four converter warps write the lo part of each
// landed stage into a twin buffer before the MMA warp consumes it; the landed
// x is the hi operand as is (kind::tf32 truncates to the top 19 bits).
//
// Grouped B (RGCN relation weights, GemmPart::tile_group): the B rows of
// 128-row tile t start at tile_group[t] * group_rows.
//
// These layer transforms are HBM-bound (K <= 512), so what matters is keeping
// loads, MMAs and the output stream overlapped across tiles:
//   warp 0      TMA producer: A/B k-blocks of all of this CTA's tiles into an
//               S-stage shared-memory ring (full / empty mbarriers);
//   warp 1      TMEM allocator + MMA issuer: tcgen05.mma (M=128, N=BN, K=16)
//               into one of TWO accumulator buffers (2 x BN TMEM columns), so
//               tile i+1's MMAs run while tile i is drained;
//   warps 2-9   epilogue, two groups of four warps (one warp per TMEM lane
//               quarter in each group; warp w drains lanes 32*(w%4)..): the
//               groups take alternate 128-byte-wide output chunks, so one
//               group's tcgen05.ld / math overlaps the other's staging and TMA
//               store.  Per chunk: tcgen05.ld, fused epilogue math, pack into
//               a 128-byte-swizzled staging tile, TMA store (bulk_group) --
//               coalesced writes;
//   warp 10     epilogue loader: TMA loads of the addend / mask chunks into a
//               2-deep buffer (buffer b feeds epilogue group b);
//   warps 11-14 (fp32 only) hi / lo converters.
// One CTA per SM loops over 128 x BN tiles (N fastest, so A tiles of the N
// tiles of one row block are adjacent in time).
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstring>
#include <mutex>
#include <type_traits>

#include "wg_internal.cuh"

namespace wg {

bool tc_make_map_t(CUtensorMap* m, CUtensorMapDataType ty, const void* ptr, uint64_t inner, uint64_t outer,
                   uint64_t ld_bytes, uint32_t box_in, uint32_t box_out);
bool tc_make_map3_t(CUtensorMap* m, CUtensorMapDataType ty, const void* ptr, uint64_t inner, uint64_t outer,
                    uint64_t chunks, uint64_t ld_bytes, uint64_t chunk_bytes, uint32_t box_in, uint32_t box_out);

namespace {

// Every stage row and every epilogue chunk row is one 128-byte swizzle span:
// BKE = 128 / sizeof(T) K elements per stage, CHE = 128 / sizeof(T) columns
// per epilogue chunk.
constexpr int BM = 128;
constexpr int A_STAGE = BM * 128;                  // 16 KB
constexpr int CHUNK_BYTES = BM * 128;              // 16 KB

template <typename T> struct Cfg {
  static constexpr bool TF32 = sizeof(T) == 4;
  static constexpr int ES = sizeof(T);
  static constexpr int BKE = 128 / ES;
  static constexpr int CHE = 128 / ES;
  static constexpr int EPV = 16 / ES;              // elements per 16-byte unit
  static constexpr int NTHREADS = TF32 ? 480 : 352;   // fp32: + 4 converter warps
  static constexpr int CONV0 = 352;                   // first converter thread
};

struct P2 {
  int64_t M;
  int N, BN, n_tiles, stages, nparts, n_split;
  int64_t num_tiles;
  int kblocks[3];
  const int32_t* tile_group[3];
  int group_rows[3];
  const int32_t* a_rows[3];
  const float* rscale;
  const float* bias;
  int relu, has_add, has_mask, bias_vec;
  int cpg;          // fp32 row-gathered A by per-lane cp.async (see the producer)
  int fc_d, fc_d2;  // columns per chunk of the (column-chunked) D / D2 output maps
  int bres;         // B resident: every k-block of B loaded once per CTA (one N tile, no grouped B)
  // direct stores of a chunk that straddles the D / D2 split (n_split not a
  // multiple of the 128-byte chunk: C5's 32-wide [Y | S])
  void* d_ptr; int64_t ldd, d_cstride; void* d2_ptr; int64_t ldd2;
  const void* a_tab; int64_t lda_tab; int k_a;   // cpg: table, its row pitch (elements), K
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
// TMA tile::gather4: rows r0..r3 of a 2-D map (box {inner, 1}) at column c0 -> 4 consecutive smem rows
__device__ __forceinline__ void tma_gather4(uint32_t dst, const CUtensorMap* m, int c0, int r0, int r1, int r2, int r3,
                                            uint32_t bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, "
      "%4, %5, %6}], [%7];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(m)), "r"(c0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(bar)
      : "memory");
}
// output maps are 3-D {columns of a chunk, rows, chunks}: a column-chunked
// table [C][rows][Fc] (the exchange layout of DESIGN.md §9); C = 1 is the
// plain row-major matrix.  A 128-byte store box never straddles a chunk
// (Fc is a multiple of 128 bytes when C > 1).
__device__ __forceinline__ void tma_store3(const CUtensorMap* m, int c0, int c1, int c2, uint32_t src) {
  asm volatile("cp.async.bulk.tensor.3d.global.shared::cta.bulk_group [%0, {%1, %2, %3}], [%4];" ::"l"(
                   reinterpret_cast<uint64_t>(m)),
               "r"(c0), "r"(c1), "r"(c2), "r"(src)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void epi_bar(int grp) { asm volatile("bar.sync %0, 128;" ::"r"(grp + 1) : "memory"); }

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
__device__ __forceinline__ void mma_tf32(uint32_t tmem, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n}\n" ::"r"(tmem),
      "l"(a), "l"(b), "r"(idesc), "r"(acc));
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

// byte offset of 16-byte unit k of row r inside a [128 x 128 B] tile with 128-byte swizzle
__device__ __forceinline__ uint32_t sw_off(int r, int k) { return (uint32_t)(r * 128 + ((k ^ (r & 7)) << 4)); }

template <typename T> __device__ __forceinline__ void unpack16(const int4& q, float* f);
template <> __device__ __forceinline__ void unpack16<__nv_bfloat16>(const int4& q, float* f) {
  const uint32_t w[4] = {(uint32_t)q.x, (uint32_t)q.y, (uint32_t)q.z, (uint32_t)q.w};
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    f[2 * i] = __uint_as_float(w[i] << 16);
    f[2 * i + 1] = __uint_as_float(w[i] & 0xffff0000u);
  }
}
template <> __device__ __forceinline__ void unpack16<float>(const int4& q, float* f) {
  f[0] = __int_as_float(q.x); f[1] = __int_as_float(q.y); f[2] = __int_as_float(q.z); f[3] = __int_as_float(q.w);
}
template <typename T> __device__ __forceinline__ int4 pack16(const float* f);
template <> __device__ __forceinline__ int4 pack16<__nv_bfloat16>(const float* f) {
  uint32_t pk[4];
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    __nv_bfloat162 h = __floats2bfloat162_rn(f[2 * i], f[2 * i + 1]);
    pk[i] = *reinterpret_cast<uint32_t*>(&h);
  }
  return make_int4((int)pk[0], (int)pk[1], (int)pk[2], (int)pk[3]);
}
template <> __device__ __forceinline__ int4 pack16<float>(const float* f) {
  return make_int4(__float_as_int(f[0]), __float_as_int(f[1]), __float_as_int(f[2]), __float_as_int(f[3]));
}

// shared-memory plan (bytes from the 1024-aligned base), identical on host and device
struct SmemPlan {
  int stage, ring, bres, stg, add, mask, ids, bars, total;
};
// bres_kb > 0: B resident (bf16 only) -- the ring holds A only and the
// bres_kb k-blocks of B (BN rows x 128 B each) sit after it for the whole kernel
__host__ __device__ inline SmemPlan smem_plan(bool tf32, int BN, int S, bool has_add, bool has_mask, bool cpg,
                                              int bres_kb = 0) {
  SmemPlan q;
  q.stage = bres_kb ? A_STAGE : (A_STAGE + BN * 128) * (tf32 ? 2 : 1);   // [A | B] (+ [A_lo | B_lo])
  q.ring = S * q.stage;
  q.bres = q.ring;
  q.stg = q.ring + bres_kb * BN * 128;
  q.add = q.stg + 2 * CHUNK_BYTES;
  q.mask = q.add + (has_add ? 2 * CHUNK_BYTES : 0);
  q.ids = q.mask + (has_mask ? 2 * CHUNK_BYTES : 0);
  q.bars = q.ids + (cpg ? BM * 4 : 0);               // cpg: the tile's 128 gather row ids
  q.total = q.bars + 512;
  return q;
}

// FL: compile-time epilogue operands (EP_ADD addend, EP_MASK ReLU mask, EP_BIAS
// bias), so the per-chunk epilogue code carries no predicated dead paths
constexpr int EP_ADD = 1, EP_MASK = 2, EP_BIAS = 4;

template <typename T, int FL>
__global__ void __launch_bounds__(Cfg<T>::NTHREADS, 1)
    k_gemm_nt_p(const __grid_constant__ CUtensorMap tA0, const __grid_constant__ CUtensorMap tB0,
                const __grid_constant__ CUtensorMap tA1, const __grid_constant__ CUtensorMap tB1,
                const __grid_constant__ CUtensorMap tA2, const __grid_constant__ CUtensorMap tB2,
                const __grid_constant__ CUtensorMap tD, const __grid_constant__ CUtensorMap tD2,
                const __grid_constant__ CUtensorMap tAdd, const __grid_constant__ CUtensorMap tMask, P2 p) {
  using C = Cfg<T>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int BN = p.BN, S = p.stages;
  const int b_bytes = BN * 128;
  int total_kb0 = 0;
  for (int i = 0; i < p.nparts; ++i) total_kb0 += p.kblocks[i];
  const SmemPlan L = smem_plan(C::TF32, BN, S, p.has_add, p.has_mask, p.cpg != 0, p.bres ? total_kb0 : 0);
  // stage s: A at s*stage, B at +A_STAGE; fp32: A_lo at +A_STAGE+b_bytes, B_lo after it
  uint8_t* ring = smem;
  uint8_t* st_sm = smem + L.stg;                   // 2 x 16 KB output staging
  uint8_t* ad_sm = smem + L.add;                   // 2 x 16 KB addend
  uint8_t* mk_sm = smem + L.mask;                  // 2 x 16 KB mask
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + L.bars);
  uint64_t* full = bars;            // [8] TMA landed
  uint64_t* empty = bars + 8;       // [8] MMA done with the stage
  uint64_t* tfull = bars + 16;      // [2]
  uint64_t* tempty = bars + 18;     // [2]
  uint64_t* efull = bars + 20;      // [2]
  uint64_t* eempty = bars + 22;     // [2]
  uint64_t* conv = bars + 24;       // [8] fp32: hi / lo split done
  uint64_t* bfull = bars + 32;      // resident B landed
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + 33);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nchunk = (BN + C::CHE - 1) / C::CHE;

  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(su32(&full[s]), p.cpg ? 33 : 1);   // cpg: + one cp.async arrive per producer lane
      mbar_init(su32(&empty[s]), 1);
      mbar_init(su32(&conv[s]), 128);
    }
    mbar_init(su32(bfull), 1);
    for (int b = 0; b < 2; ++b) {
      mbar_init(su32(&tfull[b]), 1);
      mbar_init(su32(&tempty[b]), 256);
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
    // ------------------------------------------------ TMA producer (lane 0;
    // row-gathered A parts: every lane issues the gather4 of its 4 tile rows)
    const uint32_t tx = p.bres ? (uint32_t)A_STAGE : (uint32_t)(A_STAGE + b_bytes);
    int s = 0;
    uint32_t ph = 0;
    if (p.bres && lane == 0 && blockIdx.x < p.num_tiles) {   // every k-block of B, once
      mbar_expect_tx(su32(bfull), (uint32_t)(total_kb0 * b_bytes));
      int kb = 0;
      for (int part = 0; part < p.nparts; ++part) {
        const CUtensorMap* tb = part == 0 ? &tB0 : (part == 1 ? &tB1 : &tB2);
        for (int kk = 0; kk < p.kblocks[part]; ++kk, ++kb)
          tma_load(su32(smem + L.bres + kb * b_bytes), tb, kk * C::BKE, 0, su32(bfull));
      }
    }
    // the next tile's gather row ids and relation are loaded one tile ahead,
    // so their latency never stalls the producer between tiles
    auto tile_meta = [&](int64_t t, int4& gi, int& grp) {
      gi = make_int4(0, 0, 0, 0);
      grp = 0;
      if (t >= p.num_tiles) return;
      const int64_t mt = t / p.n_tiles;
      if (p.a_rows[0]) gi = __ldg(reinterpret_cast<const int4*>(p.a_rows[0] + mt * BM) + lane);
      if (p.tile_group[0]) grp = __ldg(p.tile_group[0] + mt);
    };
    int4 gi_next;
    int grp_next;
    tile_meta(blockIdx.x, gi_next, grp_next);
    // cpg: lane l copies 16-byte unit (l & 7) of rows 4j + (l >> 3), j < 32:
    // each instruction moves four whole 128-byte row pieces (coalesced); the
    // lane's cp.async completions arrive on full[s] (noinc; count 33)
    int* ids = reinterpret_cast<int*>(smem + L.ids);
    const int cu = lane & 7, csub = lane >> 3;
    for (int64_t t = blockIdx.x; t < p.num_tiles; t += gridDim.x) {
      const int64_t mt = t / p.n_tiles;
      const int m0 = (int)(mt * BM), n0 = (int)((t % p.n_tiles) * BN);
      int part = 0, kk = 0;
      int4 gi = gi_next;
      int brow = n0 + grp_next * p.group_rows[0];
      if constexpr (C::TF32) {
        if (p.cpg) {
          __syncwarp();                       // previous tile's ids fully consumed
          ids[4 * lane + 0] = gi.x; ids[4 * lane + 1] = gi.y; ids[4 * lane + 2] = gi.z; ids[4 * lane + 3] = gi.w;
          __syncwarp();
        }
      }
      tile_meta(t + gridDim.x, gi_next, grp_next);
      for (int kb = 0; kb < total_kb; ++kb) {
        const CUtensorMap* ta = part == 0 ? &tA0 : (part == 1 ? &tA1 : &tA2);
        const CUtensorMap* tb = part == 0 ? &tB0 : (part == 1 ? &tB1 : &tB2);
        uint8_t* st = ring + s * L.stage;
        if (lane == 0) {
          mbar_wait(su32(&empty[s]), ph ^ 1);
          mbar_expect_tx(su32(&full[s]), p.cpg ? (uint32_t)b_bytes : tx);
        }
        __syncwarp();
        if (C::TF32 && p.cpg) {
          const float* tab = static_cast<const float*>(p.a_tab);
          const int col = kk * C::BKE + cu * 4;
          const bool ok = col < p.k_a;
          const uint32_t sb = su32(st);
#pragma unroll 8
          for (int j = 0; j < 32; ++j) {
            const int r = 4 * j + csub;
            const float* src = tab + (int64_t)ids[r] * p.lda_tab + (ok ? col : 0);
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(sb + sw_off(r, cu)), "l"(src),
                         "r"(ok ? 16 : 0) : "memory");
          }
          asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(su32(&full[s])) : "memory");
        } else if (p.a_rows[part]) {
          tma_gather4(su32(st) + lane * 512, ta, kk * C::BKE, gi.x, gi.y, gi.z, gi.w, su32(&full[s]));
        } else if (lane == 0) {
          tma_load(su32(st), ta, kk * C::BKE, m0, su32(&full[s]));
        }
        if (lane == 0 && !p.bres) tma_load(su32(st + A_STAGE), tb, kk * C::BKE, brow, su32(&full[s]));
        if (++kk == p.kblocks[part]) {
          kk = 0;
          ++part;
          if (part < p.nparts) {
            brow = n0 + (p.tile_group[part] ? p.tile_group[part][mt] * p.group_rows[part] : 0);
            if (p.a_rows[part]) gi = __ldg(reinterpret_cast<const int4*>(p.a_rows[part] + m0) + lane);
          }
        }
        if (++s == S) { s = 0; ph ^= 1; }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      // ------------------------------------------------ MMA issuer
      // idesc: D f32 [4,6), A / B format [7,10) / [10,13) (bf16 = 1, tf32 = 2), N>>3, M>>4
      const uint32_t fmt = C::TF32 ? 2u : 1u;
      const uint32_t idesc = (1u << 4) | (fmt << 7) | (fmt << 10) | ((uint32_t)(BN >> 3) << 17) |
                             ((uint32_t)(BM >> 4) << 24);
      int s = 0;
      uint32_t ph = 0;
      int j = 0;
      if (p.bres && blockIdx.x < p.num_tiles) mbar_wait(su32(bfull), 0);
      for (int64_t t = blockIdx.x; t < p.num_tiles; t += gridDim.x, ++j) {
        const int buf = j & 1;
        mbar_wait(su32(&tempty[buf]), ((j >> 1) & 1) ^ 1);
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        const uint32_t acc = tmem + (uint32_t)(buf * 256);
        for (int kb = 0; kb < total_kb; ++kb) {
          mbar_wait(su32(C::TF32 ? &conv[s] : &full[s]), ph);
          asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
          const uint32_t ad = su32(ring + s * L.stage);
          const uint32_t bd = p.bres ? su32(smem + L.bres + kb * b_bytes) : ad + A_STAGE;
#pragma unroll
          for (int k = 0; k < 4; ++k) {     // 4 MMAs of 32 bytes of K (16 bf16 / 8 tf32)
            const uint32_t on = (kb | k) != 0 ? 1u : 0u;
            if constexpr (C::TF32) {
              const uint32_t al = bd + b_bytes, bl = al + A_STAGE;
              mma_tf32(acc, desc_sw128(ad + k * 32), desc_sw128(bd + k * 32), idesc, on);
              mma_tf32(acc, desc_sw128(ad + k * 32), desc_sw128(bl + k * 32), idesc, 1u);
              mma_tf32(acc, desc_sw128(al + k * 32), desc_sw128(bd + k * 32), idesc, 1u);
            } else {
              mma(acc, desc_sw128(ad + k * 32), desc_sw128(bd + k * 32), idesc, on);
            }
          }
          mma_commit(su32(&empty[s]));
          if (++s == S) { s = 0; ph ^= 1; }
        }
        mma_commit(su32(&tfull[buf]));
      }
    }
  } else if (warp == 10) {
    if (lane == 0 && (FL & (EP_ADD | EP_MASK)) != 0) {
      // ------------------------------------------------ epilogue loader
      const uint32_t tx = (p.has_add ? CHUNK_BYTES : 0) + (p.has_mask ? CHUNK_BYTES : 0);
      int g = 0;
      for (int64_t t = blockIdx.x; t < p.num_tiles; t += gridDim.x) {
        const int m0 = (int)((t / p.n_tiles) * BM), n0 = (int)((t % p.n_tiles) * BN);
        for (int c = 0; c < nchunk; ++c, ++g) {
          const int b = g & 1;
          mbar_wait(su32(&eempty[b]), ((g >> 1) & 1) ^ 1);
          mbar_expect_tx(su32(&efull[b]), tx);
          if (p.has_add) tma_load(su32(ad_sm + b * CHUNK_BYTES), &tAdd, n0 + c * C::CHE, m0, su32(&efull[b]));
          if (p.has_mask) tma_load(su32(mk_sm + b * CHUNK_BYTES), &tMask, n0 + c * C::CHE, m0, su32(&efull[b]));
        }
      }
    }
  } else if (warp >= 11) {
    if constexpr (C::TF32) {
      // ------------------------------------------------ hi / lo converters (128 threads)
      const int ct = threadIdx.x - C::CONV0;
      const int n16 = (A_STAGE + b_bytes) / 16;
      int s = 0;
      uint32_t ph = 0;
      for (int64_t t = blockIdx.x; t < p.num_tiles; t += gridDim.x) {
        for (int kb = 0; kb < total_kb; ++kb) {
          mbar_wait(su32(&full[s]), ph);
          tf32_split_stage(su32(ring + s * L.stage), n16, ct, 128);
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          mbar_arrive(su32(&conv[s]));
          if (++s == S) { s = 0; ph ^= 1; }
        }
      }
    }
  } else {
    // ------------------------------------------------ epilogue (warps 2..9)
    const int grp = (warp - 2) >> 2;               // epilogue group: chunks g with g % 2 == grp
    const int et = (threadIdx.x - 64) & 127;       // 0..127 inside the group
    const int quarter = warp & 3;                  // TMEM lane quarter this warp may access
    const int r = quarter * 32 + lane;             // tile row
    constexpr bool epi_loads = (FL & (EP_ADD | EP_MASK)) != 0;
    const float lo_clamp = p.relu ? 0.f : -INFINITY;
    uint8_t* stg = st_sm + grp * CHUNK_BYTES;      // this group's staging tile
    const uint8_t* adp = ad_sm + grp * CHUNK_BYTES;
    const uint8_t* mkp = mk_sm + grp * CHUNK_BYTES;
    int j = 0, g = 0;
    for (int64_t t = blockIdx.x; t < p.num_tiles; t += gridDim.x, ++j) {
      const int m0 = (int)((t / p.n_tiles) * BM), n0 = (int)((t % p.n_tiles) * BN);
      const int buf = j & 1;
      const int64_t m = (int64_t)m0 + r;
      const float rs_d = (p.rscale && m < p.M) ? p.rscale[m] : 1.f;   // D only (not the split output D2)
      mbar_wait(su32(&tfull[buf]), (j >> 1) & 1);
      asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
      for (int c = 0; c < nchunk; ++c, ++g) {
        if ((g & 1) != grp) continue;              // the other group's chunk
        uint32_t u[64];
        const uint32_t taddr = tmem + ((uint32_t)(quarter * 32) << 16) + (uint32_t)(buf * 256 + c * C::CHE);
#pragma unroll
        for (int q = 0; q < C::CHE / 16; ++q) tmem_ld16(taddr + 16 * q, u + 16 * q);
        asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
        if (epi_loads) mbar_wait(su32(&efull[grp]), (g >> 1) & 1);
        // the staging tile was last read by this group's previous TMA store
        if (et == 0) bulk_wait_read<0>();
        epi_bar(grp);
        const int nc0 = n0 + c * C::CHE;
        // split output: a 128-byte chunk belongs to D or to D2, or straddles
        // the split (stored directly from registers, 16 bytes at a time)
        const bool second = p.n_split > 0 && nc0 >= p.n_split;
        const bool strad = p.n_split > 0 && nc0 < p.n_split && nc0 + C::CHE > p.n_split;
        const float rs = second ? 1.f : rs_d;
        // one 16-byte output unit (EPV columns) at a time; FULL: every column < N
        auto units = [&](auto full_t) {
          constexpr bool FULL = decltype(full_t)::value;
#pragma unroll
          for (int k = 0; k < 8; ++k) {
            float f[C::EPV];
            const int nc = nc0 + k * C::EPV;
#pragma unroll
            const float rsu = (strad && nc >= p.n_split) ? 1.f : rs;   // the row scale is D's only
#pragma unroll
            for (int i = 0; i < C::EPV; ++i) f[i] = rsu * __uint_as_float(u[k * C::EPV + i]);
            if constexpr ((FL & EP_ADD) != 0) {
              float a[C::EPV];
              unpack16<T>(*reinterpret_cast<const int4*>(adp + sw_off(r, k)), a);
#pragma unroll
              for (int i = 0; i < C::EPV; ++i) f[i] += a[i];
            }
            if constexpr ((FL & EP_BIAS) != 0) {
              if constexpr (FULL) {
#pragma unroll
                for (int i = 0; i < C::EPV; i += 4) {
                  const float4 b4 = __ldg(reinterpret_cast<const float4*>(p.bias + nc + i));
                  f[i] += b4.x; f[i + 1] += b4.y; f[i + 2] += b4.z; f[i + 3] += b4.w;
                }
              } else {
#pragma unroll
                for (int i = 0; i < C::EPV; ++i) f[i] += (nc + i < p.N) ? p.bias[nc + i] : 0.f;
              }
            }
#pragma unroll
            for (int i = 0; i < C::EPV; ++i) f[i] = fmaxf(f[i], lo_clamp);   // ReLU (or -inf: none)
            if constexpr ((FL & EP_MASK) != 0) {
              float a[C::EPV];
              unpack16<T>(*reinterpret_cast<const int4*>(mkp + sw_off(r, k)), a);
#pragma unroll
              for (int i = 0; i < C::EPV; ++i) if (!(a[i] > 0.f)) f[i] = 0.f;
            }
            if constexpr (!FULL) {
#pragma unroll
              for (int i = 0; i < C::EPV; ++i) if (nc + i >= p.N) f[i] = 0.f;
            }
            if (strad) {
              if (m < p.M && nc < p.N) {
                T* dst = nc < p.n_split
                             ? static_cast<T*>(p.d_ptr) + (int64_t)(nc / p.fc_d) * p.d_cstride + m * p.ldd + nc % p.fc_d
                             : static_cast<T*>(p.d2_ptr) + m * p.ldd2 + (nc - p.n_split);
                *reinterpret_cast<int4*>(dst) = pack16<T>(f);
              }
            } else {
              *reinterpret_cast<int4*>(stg + sw_off(r, k)) = pack16<T>(f);
            }
          }
        };
        if (nc0 + C::CHE <= p.N && p.bias_vec) units(std::true_type{});
        else units(std::false_type{});
        if (epi_loads) mbar_arrive(su32(&eempty[grp]));
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        epi_bar(grp);
        if (et == 0 && !strad) {
          const CUtensorMap* td = second ? &tD2 : &tD;
          const int col = second ? nc0 - p.n_split : nc0, fc = second ? p.fc_d2 : p.fc_d;
          tma_store3(td, col % fc, m0, col / fc, su32(stg));
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

template <typename T, int FL>
void launch_p(unsigned grid, size_t smem, cudaStream_t s, const CUtensorMap* maps, const P2& p) {
  static bool attr = false;
  if (!attr) {
    cudaFuncSetAttribute(k_gemm_nt_p<T, FL>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    attr = true;
  }
  k_gemm_nt_p<T, FL><<<grid, Cfg<T>::NTHREADS, smem, s>>>(maps[0], maps[1], maps[2], maps[3], maps[4], maps[5],
                                                          maps[6], maps[7], maps[8], maps[9], p);
}

template <typename T>
void launch_fl(int fl, unsigned grid, size_t smem, cudaStream_t s, const CUtensorMap* maps, const P2& p) {
  switch (fl) {
    case 0: launch_p<T, 0>(grid, smem, s, maps, p); break;
    case 1: launch_p<T, 1>(grid, smem, s, maps, p); break;
    case 2: launch_p<T, 2>(grid, smem, s, maps, p); break;
    case 3: launch_p<T, 3>(grid, smem, s, maps, p); break;
    case 4: launch_p<T, 4>(grid, smem, s, maps, p); break;
    case 5: launch_p<T, 5>(grid, smem, s, maps, p); break;
    case 6: launch_p<T, 6>(grid, smem, s, maps, p); break;
    default: launch_p<T, 7>(grid, smem, s, maps, p); break;
  }
}

}  // namespace

// returns false when the shape / epilogue is not handled (caller falls back)
bool tc_gemm_nt_persistent(wg_dtype dt, int64_t M, int N, const GemmPart* parts, int n_parts, const GemmEpi& epi,
                           cudaStream_t s, wg_status* st) {
  static int disabled = -1;
  if (disabled < 0) {
    const char* e = getenv("WG_GEMM_V1");
    disabled = (e && e[0] == '1') ? 1 : 0;
  }
  const bool f32 = dt == WG_F32;
  if (disabled || (epi.d_f32 && !f32) || n_parts > 3 || M <= 0) return false;
  const int es = f32 ? 4 : 2, che = 128 / es;
  const CUtensorMapDataType ty = f32 ? CU_TENSOR_MAP_DATA_TYPE_FLOAT32 : CU_TENSOR_MAP_DATA_TYPE_BFLOAT16;
  // several N tiles: BN = 256 (bf16) / 128 (fp32, the lo twins double the
  // stage) so every store box stays inside its tile (the ragged end is
  // clipped by the tensor map); one tile: BN = N
  static int bn_env = -1;
  if (bn_env < 0) {
    const char* e = getenv("WG_NT_BNMAX");
    bn_env = e ? atoi(e) : 0;
  }
  const int bn_max = (bn_env >= 64 && bn_env <= 256 && bn_env % 64 == 0) ? bn_env : (f32 ? 128 : 256);
  const int n_tiles = (int)cdiv(N, bn_max);
  const int BN = n_tiles > 1 ? bn_max : (int)rup(N, 16);
  // a split off the 128-byte chunk grid is stored directly for the straddling chunk; 16-byte units
  if (epi.D2 && (epi.n_split % (16 / es) != 0 || (N - epi.n_split) % (16 / es) != 0)) return false;
  CUtensorMap maps[10];
  memset(maps, 0, sizeof(maps));
  P2 p{};
  p.M = M; p.N = N; p.BN = BN; p.n_tiles = n_tiles; p.nparts = n_parts;
  p.num_tiles = cdiv(M, BM) * n_tiles;
  for (int i = 0; i < n_parts; ++i) {
    const GemmPart& q = parts[i];
    const uint64_t brows = q.tile_group ? (uint64_t)q.groups * q.group_rows : (uint64_t)q.nb;
    if (q.tile_group && BN > q.group_rows) return false;
    if (q.a_rows) {   // gather4 map: box {che, 1} over the whole table
      if ((reinterpret_cast<uintptr_t>(q.a_rows) & 15) != 0) return false;
      if (!tc_make_map_t(&maps[2 * i], ty, q.A, (uint64_t)q.K, (uint64_t)q.a_table_rows, (uint64_t)q.lda * es, che, 1))
        return false;
    } else if (!tc_make_map_t(&maps[2 * i], ty, q.A, (uint64_t)q.K, (uint64_t)M, (uint64_t)q.lda * es, che, BM)) {
      return false;
    }
    p.a_rows[i] = q.a_rows;
    if (!tc_make_map_t(&maps[2 * i + 1], ty, q.B, (uint64_t)q.K, brows, (uint64_t)q.ldb * es, che, BN)) return false;
    p.kblocks[i] = (int)cdiv(q.K, che);
    p.tile_group[i] = q.tile_group;
    p.group_rows[i] = q.group_rows;
  }
  for (int i = n_parts; i < 3; ++i) { maps[2 * i] = maps[0]; maps[2 * i + 1] = maps[1]; }
  const int n1 = epi.D2 ? epi.n_split : N;
  // D: column-chunked when d_chunk_cols > 0 (chunks of d_chunk_cols columns,
  // d_chunk_stride elements apart); otherwise one chunk of n1 columns
  const int C1 = epi.d_chunk_cols > 0 ? (int)cdiv(n1, epi.d_chunk_cols) : 1;
  p.fc_d = C1 > 1 ? epi.d_chunk_cols : n1;
  if (C1 > 1 && (p.fc_d % che != 0 || (epi.d_chunk_stride * es) % 16 != 0)) return false;
  p.d_ptr = epi.D; p.ldd = epi.ldd; p.d_cstride = C1 > 1 ? epi.d_chunk_stride : 0;
  p.d2_ptr = epi.D2; p.ldd2 = epi.ldd2;
  if ((epi.D2 && (reinterpret_cast<uintptr_t>(epi.D2) % 16 || (epi.ldd2 * es) % 16)) ||
      reinterpret_cast<uintptr_t>(epi.D) % 16 || (epi.ldd * es) % 16)
    return false;
  if (!tc_make_map3_t(&maps[6], ty, epi.D, (uint64_t)p.fc_d, (uint64_t)M, (uint64_t)C1, (uint64_t)epi.ldd * es,
                      (uint64_t)(C1 > 1 ? epi.d_chunk_stride : 0) * es, che, BM))
    return false;
  maps[7] = maps[6];
  p.fc_d2 = p.fc_d;
  if (epi.D2) {
    p.n_split = epi.n_split;
    p.fc_d2 = N - epi.n_split;
    if (!tc_make_map3_t(&maps[7], ty, epi.D2, (uint64_t)(N - epi.n_split), (uint64_t)M, 1, (uint64_t)epi.ldd2 * es, 0,
                        che, BM))
      return false;
  }
  // addend / mask maps (2-D loads) need their own maps
  maps[8] = maps[9] = maps[0];
  if (epi.addend) {
    if (!tc_make_map_t(&maps[8], ty, epi.addend, (uint64_t)N, (uint64_t)M, (uint64_t)epi.ld_add * es, che, BM))
      return false;
    p.has_add = 1;
  }
  if (epi.mask_ref) {
    if (!tc_make_map_t(&maps[9], ty, epi.mask_ref, (uint64_t)N, (uint64_t)M, (uint64_t)epi.ld_mask * es, che, BM))
      return false;
    p.has_mask = 1;
  }
  // fp32 row-gathered A by per-lane cp.async instead of TMA gather4: opt-in
  // (WG_GATHER_CPASYNC=1) -- on C3 (128-byte row pieces, 4-stage ring) it
  // measured 6.45 ms vs 6.0 ms for gather4: both are bound by the ring's
  // bytes in flight, not by TMA issue
  static int gather_cp = -1;
  if (gather_cp < 0) {
    const char* e = getenv("WG_GATHER_CPASYNC");
    gather_cp = (e && e[0] == '1') ? 1 : 0;
  }
  if (f32 && n_parts == 1 && parts[0].a_rows && parts[0].K % 4 == 0 && (parts[0].lda % 4) == 0 && gather_cp) {
    p.cpg = 1;
    p.a_tab = parts[0].A;
    p.lda_tab = parts[0].lda;
    p.k_a = parts[0].K;
  }
  p.rscale = epi.rscale;
  p.bias = epi.bias;
  p.bias_vec = (reinterpret_cast<uintptr_t>(epi.bias) & 15) == 0;
  p.relu = epi.relu;
  const int limit = 227 * 1024 - 1024;
  // B resident (bf16, one N tile, no grouped B): B is read from L2 once per
  // CTA instead of once per tile, and the ring carries A only -- the HBM-bound
  // skinny-K GEMMs of the gTask layer then keep A, not B, in flight.  Needs
  // room for >= 3 A stages next to it.  WG_NT_BRES=0 disables.
  static int bres_env = -1;
  if (bres_env < 0) {
    const char* e = getenv("WG_NT_BRES");
    bres_env = (e && e[0] == '0') ? 0 : 1;
  }
  int total_kb = 0;
  bool grouped = false;
  for (int i = 0; i < n_parts; ++i) { total_kb += p.kblocks[i]; grouped = grouped || parts[i].tile_group; }
  int stages = 4;
  p.bres = 0;
  if (bres_env && !f32 && n_tiles == 1 && !grouped && !p.cpg) {
    int st2 = 8;
    while (st2 > 3 && smem_plan(f32, BN, st2, p.has_add, p.has_mask, false, total_kb).total > limit) --st2;
    if (smem_plan(f32, BN, st2, p.has_add, p.has_mask, false, total_kb).total <= limit) {
      p.bres = 1;
      stages = st2;
    }
  }
  const int bkb = p.bres ? total_kb : 0;
  if (!p.bres) {
    while (stages > 2 && smem_plan(f32, BN, stages, p.has_add, p.has_mask, p.cpg).total > limit) --stages;
    if (smem_plan(f32, BN, stages, p.has_add, p.has_mask, p.cpg).total > limit) return false;
  }
  p.stages = stages;
  if (!g_sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&g_sms, cudaDevAttrMultiProcessorCount, dev);
  }
  const unsigned grid = (unsigned)std::min<int64_t>(p.num_tiles, g_sms);
  const size_t smem = 1024 + (size_t)smem_plan(f32, BN, stages, p.has_add, p.has_mask, p.cpg, bkb).total;
  double kt = 0;
  for (int i = 0; i < n_parts; ++i) kt += parts[i].K;
  ProfScope ps(PK_TC_NT, s, (double)M * (kt + N + (epi.addend ? N : 0) + (epi.mask_ref ? N : 0)) * es,
               2.0 * M * N * kt);
  const int fl = (p.has_add ? EP_ADD : 0) | (p.has_mask ? EP_MASK : 0) | (p.bias ? EP_BIAS : 0);
  if (f32) launch_fl<float>(fl, grid, smem, s, maps, p);
  else launch_fl<__nv_bfloat16>(fl, grid, smem, s, maps, p);
  ++launch_counter();
  cudaError_t e = cudaGetLastError();
  *st = e == cudaSuccess ? WG_OK : WG_ERR_CUDA;
  if (e != cudaSuccess) set_error(std::string("k_gemm_nt_p: ") + cudaGetErrorString(e));
  return true;
}

}  // namespace wg
