// Internal declarations of the B200 gTask graph-convolution library (libwg.so).
// Product code: never includes or links anything under oracle/.
#pragma once
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>
#include <string>
#include <vector>

#include "../../include/wg.h"

namespace wg {

// ----------------------------------------------------------------- errors
void set_error(const std::string& msg);
int64_t& launch_counter();

#define WG_CK(call)                                                                    \
  do {                                                                                 \
    cudaError_t e_ = (call);                                                           \
    if (e_ != cudaSuccess) {                                                           \
      ::wg::set_error(std::string(#call) + ": " + cudaGetErrorString(e_) + " @" +      \
                      __FILE__ + ":" + std::to_string(__LINE__));                      \
      return WG_ERR_CUDA;                                                              \
    }                                                                                  \
  } while (0)

#define WG_REQ(cond, code, msg)                                                        \
  do {                                                                                 \
    if (!(cond)) {                                                                     \
      ::wg::set_error(msg);                                                            \
      return code;                                                                     \
    }                                                                                  \
  } while (0)

#define WG_TRY(expr)                                                                   \
  do {                                                                                 \
    wg_status s_ = (expr);                                                             \
    if (s_ != WG_OK) return s_;                                                        \
  } while (0)

// every kernel launch goes through this so wg_launch_count() is exact
#define WG_LAUNCH(kernel, grid, block, smem, stream, ...)                              \
  do {                                                                                 \
    kernel<<<(grid), (block), (smem), (stream)>>>(__VA_ARGS__);                        \
    ++::wg::launch_counter();                                                          \
    cudaError_t e_ = cudaGetLastError();                                               \
    if (e_ != cudaSuccess) {                                                           \
      ::wg::set_error(std::string("launch ") + #kernel + ": " + cudaGetErrorString(e_)); \
      return WG_ERR_CUDA;                                                              \
    }                                                                                  \
  } while (0)

// live per-kernel-class timing (wg_profile): events around each launch
enum ProfKind { PK_AGG = 0, PK_COMBINE = 1, PK_TC_NT = 2, PK_TC_TN = 3, PK_SIMT = 4, PK_MISC = 5, PK_GAT = 6,
                PK_RGCN = 7, PK_KINDS = 8 };
struct ProfScope {
  ProfScope(int kind, cudaStream_t s, double bytes, double flops);
  ~ProfScope();
  int rec_ = -1;
  cudaStream_t s_;
};

static inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }
static inline int64_t rup(int64_t a, int64_t b) { return cdiv(a, b) * b; }
static inline int dsize(wg_dtype t) { return t == WG_BF16 ? 2 : 4; }
// row pitch in elements of a table the gathers read: <= 32 / <= 64-byte rows
// padded to 32 / 64 bytes, longer rows to a multiple of 128 bytes, so a row
// touches the fewest 128-byte L2 lines (random row gathers are bound by line
// accesses: DESIGN.md §5, profiles/r02/gran_probe.md)
static inline int64_t pitch(int64_t F, wg_dtype t) {
  const int64_t b = F * dsize(t);
  return rup(b, b <= 32 ? 32 : b <= 64 ? 64 : 128) / dsize(t);
}

// ------------------------------------------------------------ work items
// A work item is the unit a CTA executes: the rows of one gTask (plus the
// empty rows next to it in the same tile), or one SPLIT chunk of a row.
struct WorkItem {
  int32_t row_lo, row_hi;   // local rows [row_lo, row_hi)
  int64_t e_lo, e_hi;       // SPLIT: edge positions of the chunk; regular: row_ptr range
  int32_t split_slot;       // >= 0: SPLIT chunk -> partial slot; -1: regular
  int32_t task;             // gTask index (for plans / debugging)
};
static_assert(sizeof(WorkItem) == 32, "WorkItem layout");

struct SplitRow {
  int32_t row;              // local row
  int32_t first_slot, n_slots;
  int32_t plan;
};

// --------------------------------------------------- one partition side
struct Side {
  int64_t E = 0;            // local edges (in-edges of owned rows, or out-edges)
  int64_t n_rows = 0;       // owned rows
  int32_t* perm = nullptr;  // [E] global edge ids in sorted order
  int32_t* idx = nullptr;   // [E] other endpoint (global vertex id) in sorted order
  int32_t* key = nullptr;   // [E] key vertex (global) in sorted order
  int32_t* type = nullptr;  // [E] edge type in sorted order (typed graphs)
  int64_t* row_ptr = nullptr;  // [n_rows+1] local CSR over key rows (untyped graphs)
  wg_task* tasks = nullptr; // device task table
  int64_t n_tasks = 0;
  std::vector<wg_task> h_tasks;  // host copy (plan building)
  std::vector<int64_t> h_row_ptr;
};

}  // namespace wg

struct wg_graph_s {
  int device = 0;
  int64_t V = 0, vb = 0, ve = 0, E_total = 0;
  int32_t T = 128, R = 1, by_type = 0;
  int64_t E_max = 0;
  int64_t max_in_deg = 0;
  int32_t* deg_in = nullptr;   // [V] global
  int32_t* deg_out = nullptr;  // [V]
  float* rs_in = nullptr;      // [V] 1/sqrt(max(1,deg_in))
  float* rs_out = nullptr;     // [V] 1/sqrt(max(1,deg_out))
  float* inv_in = nullptr;     // [V] 1/max(1,deg_in)
  wg::Side fwd, bwd;
  int64_t* fwdpos = nullptr;   // [E_T] (owning all rows)
  int32_t* etype_all = nullptr; // [E_total] types by global edge id (typed graphs)
  int32_t* rel_cnt = nullptr;   // [E_total] |in_r(dst_e)| by global edge id (typed graphs)
  std::vector<void*> allocs;
  int live_plans = 0;
  std::vector<int64_t> bounds;  // 1-D partition of every rank (wg_graph_create_dist), else empty
};

namespace wg {

// ------------------------------------------------------------- kernels
struct AggArgs {
  const WorkItem* items;
  int n_items;
  const int64_t* row_ptr;     // [n_rows+1]
  const int32_t* idx;         // gathered row id per position
  const int32_t* key;         // key (output) vertex per position, GLOBAL id
  const void* table;          // gathered table [.. x ld_tab]
  int64_t ld_tab;
  const float* gscale;        // per gathered row (nullable)
  const float* escale;        // per entry / edge position (nullable; not combined with gscale)
  const float* rscale;        // per output row, indexed by GLOBAL row (local + row_base) (nullable)
  int64_t row_base;           // local row -> global row offset (for rscale / self rows)
  const void* self_tab;       // self term rows (local row indexing) (nullable)
  int64_t ld_self;
  float self_coef;
  const float* bias;          // [F] (nullable)
  int relu;
  const void* mask_ref;       // relu mask reference (output row r kept where ref[r] > 0) (nullable)
  int64_t ld_mask;
  void* out;                  // [n_rows x ld_out]
  int64_t ld_out;
  void* zero_out;             // optional second output zeroed for the same rows
  int64_t ld_zero;
  int zero_cols;              // columns (elements) of zero_out to clear
  float* partial;             // SPLIT partials [slots x ld_part] fp32
  int64_t ld_part;
  int F;                      // real columns
  int64_t E_max;              // rows with deg > E_max belong to SPLIT items
  int64_t n_edges, n_rows;    // totals over the items (profiling: algorithmic bytes)
};

struct CombineArgs {
  const SplitRow* rows;
  int n_rows;
  const float* partial;
  int64_t ld_part;
  const float* rscale;
  int64_t row_base;
  const void* self_tab;
  int64_t ld_self;
  float self_coef;
  const float* bias;
  int relu;
  const void* mask_ref;
  int64_t ld_mask;
  void* out;
  int64_t ld_out;
  void* zero_out;
  int64_t ld_zero;
  int zero_cols;
  int F;
  int plan_filter;            // -1 all, else only rows with this plan
};

wg_status launch_agg(wg_dtype dt, const AggArgs& a, cudaStream_t s);
wg_status launch_combine(wg_dtype dt, const CombineArgs& a, cudaStream_t s);
// regular items + overfill rows: a cluster kernel per heavy row on a
// high-priority side stream (or, WG_HEAVY=0, SPLIT items + combine)
wg_status launch_agg_outliers(wg_dtype dt, const AggArgs& a, int n_split_items, const SplitRow* split_rows,
                              int n_split_rows, const CombineArgs& comb, cudaStream_t s);

// GEMM: D[M x N] = sum_p A_p[M x K_p] * B_p[N x K_p]^T  (+ epilogue)
struct GemmPart {
  const void* A; int64_t lda;   // row-major [M x K]
  const void* B; int64_t ldb;   // row-major [nb x K]; rows >= nb read as 0
  int K;
  int nb;
  // grouped GEMM (RGCN relation weights): 128-row tile t of A uses the B rows
  // [tile_group[t] * group_rows, +nb) of a stacked [groups x group_rows x ldb] B
  const int32_t* tile_group = nullptr;
  int group_rows = 0;
  int groups = 1;
  // row-gathered A (tcgen05 path only, TMA tile::gather4): row m of A is row
  // a_rows[m] of the [a_table_rows x lda] table A; a_rows holds rup(M, 128)
  // valid indices
  const int32_t* a_rows = nullptr;
  int64_t a_table_rows = 0;
};
struct GemmEpi {
  const float* rscale = nullptr;      // per row (split output: applies to D only, not D2)
  const float* bias = nullptr;        // per column [N]
  const void* addend = nullptr;       // add [M x N] (conv dtype), ld_add
  int64_t ld_add = 0;
  int relu = 0;
  const void* mask_ref = nullptr;     // keep where ref > 0 (conv dtype), ld_mask
  int64_t ld_mask = 0;
  void* D = nullptr; int64_t ldd = 0; // output (conv dtype unless d_f32)
  int d_f32 = 0;
  // split output: columns >= n_split go to D2 (column n - n_split); n_split % 16 == 0
  void* D2 = nullptr; int64_t ldd2 = 0; int n_split = 0;
  // column-chunked D (exchange layout [C][rows][Fc]): chunks of d_chunk_cols
  // columns, d_chunk_stride elements apart; ldd is then the chunk pitch Fc
  int d_chunk_cols = 0; int64_t d_chunk_stride = 0;
};
wg_status gemm_nt(wg_dtype dt, int64_t M, int N, const GemmPart* parts, int n_parts,
                  const GemmEpi& epi, void* scratch, size_t scratch_bytes, cudaStream_t s);
// Grouped TN work units (RGCN dW_r): group g owns K rows [off[g], off[g+1]),
// cut into units of <= span rows (multiples of `align`); unit u = {first K
// row, k-blocks of 128 / sizeof(dtype) rows, group, -}, units of a group are
// consecutive, unit_off[g] .. unit_off[g+1].  Built once per plan.
struct TnUnits {
  const int4* units = nullptr;
  const int32_t* unit_off = nullptr;
  int n_units = 0, groups = 0, align = 0;
  int64_t k_total = 0;
};
// host: unit table for group offsets h_off (size groups + 1); kb_rows = rows per k-block
void make_tn_units(const std::vector<int64_t>& h_off, int64_t target_units, int kb_rows, std::vector<int4>* units,
                   std::vector<int32_t>* unit_off);
// dW[M x N] (fp32, exact shape, ld = N) = A[K x M]^T * B[K x N] (split-K, deterministic)
size_t gemm_tn_scratch(int64_t K, int M, int N);
// acc != 0: D += A^T B (fixed order: the previous D is added after the split sums)
wg_status gemm_tn(wg_dtype dt, int64_t K, int M, int N, const void* A, int64_t lda,
                  const void* B, int64_t ldb, float* D, void* scratch, cudaStream_t s, int acc = 0);

// grouped weight gradient: D[g] (fp32 [M x N]) = sum_{k in [off[g], off[g+1])} A[k]^T B[k]
size_t gemm_tn_grouped_scratch(int n_units, int M, int N);
wg_status gemm_tn_grouped(wg_dtype dt, const TnUnits& U, int M, int N, const void* A, int64_t lda,
                          const void* B, int64_t ldb, float* D, void* scratch, cudaStream_t s);
// batched weight prep: `batch` matrices of [rows x cols] (fp32, contiguous) into
// consecutive [out_rows x ldo] blocks
wg_status prep_weight_batched(wg_dtype dt, const float* W, int batch, int rows, int cols, int transpose, void* out,
                              int64_t ldo, int out_rows, cudaStream_t s);
// weight prep: fp32 [rows x cols] -> dtype, optionally transposed, into [out_rows x ldo]
wg_status prep_weight(wg_dtype dt, const float* W, int rows, int cols, int transpose,
                      void* out, int64_t ldo, int out_rows, cudaStream_t s);
// column sums (deterministic) of dy (optionally relu-masked by ref, written to dt_out)
// dt2 (optional): the same rows scaled by rs2[row] (nullable: 1; the
// destination scale folded into an exchanged table), in a column-chunked
// layout when fc2 > 0 (chunks of fc2 columns, cs2 elements apart, pitch ldt2)
wg_status bias_grad_mask(wg_dtype dt, int64_t M, int N, const void* dy, int64_t lddy,
                         const void* ref, int64_t ldref, void* dt_out, int64_t ldt,
                         float* db, float* scratch, cudaStream_t s,
                         const float* rs2 = nullptr, void* dt2 = nullptr, int64_t ldt2 = 0, int fc2 = 0,
                         int64_t cs2 = 0);
size_t bias_grad_scratch(int64_t M, int N);

// cost-model constants (milli-femtoseconds per byte / per flop), from MEASURED_PEAKS
constexpr int64_t K_MEM = 152952;   // 1e6 / 6.538 GB/s-per-fs
constexpr int64_t K_LINK = 1428571; // 1e6 / 0.7 TB/s: NVLink 5 all-gather bandwidth per GPU (effective)
constexpr int64_t K_MMA_BF16 = 720; // 1e6 / 1389.2
constexpr int64_t K_MMA_F32 = 16000;

}  // namespace wg
