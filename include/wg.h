/*
 * wg.h -- C ABI of the B200-native gTask graph-convolution layer
 * (WiseGraph, Huang et al., EuroSys '24; this build's hot path is named by
 * BASELINE.json north_star and SURVEY.md §8).
 *
 * Every entry point returns a wg_status; nothing throws, aborts or exits, and
 * no CUDA or torch type appears in a signature (streams are passed as the
 * opaque value of a cudaStream_t).  There is no CPU fallback: a call that
 * cannot run on the GPU returns WG_ERR_UNSUPPORTED / WG_ERR_CUDA.
 *
 * Citations: "P:L<a>-<b>" = line range of the paper text and the
 * section / figure / equation it falls in; "Q<n>" = a reading listed in
 * DESIGN.md for a point the paper leaves open.
 *
 * Layout conventions (all calls):
 *   - Vertex tensors are row-major [rows x ld] in the conv dtype (fp32 or
 *     bf16); ld >= F and ld * sizeof(dtype) is a multiple of 16 bytes.
 *     Input columns >= F are never read into a result; output columns in
 *     [F, round_up(F, 16 B)) are written as 0, later pad columns untouched.
 *   - Weights and biases are fp32 (master copies), row-major, exact shapes;
 *     the library casts them to the conv dtype internally (RNE for bf16, Q23).
 *   - Weight gradients are fp32, exact shapes, OVERWRITTEN (not accumulated).
 *   - bf16 results are rounded to nearest even; accumulation is fp32.
 * Ownership: the caller owns every tensor passed in (x, y, params, grads,
 * saved, workspace, exchange).  The library owns graph / plan internals
 * (device memory allocated on the creation stream, freed by *_destroy).
 * Graphs and plans are immutable after creation; a plan must not outlive
 * its graph.
 * Errors: argument / range errors are detected synchronously in *_create
 * (WG_ERR_INVALID / WG_ERR_RANGE); kernel faults surface as WG_ERR_CUDA on a
 * later call.  wg_last_error() returns a thread-local message.
 */
#ifndef WG_H_
#define WG_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  WG_OK = 0,
  WG_ERR_INVALID = 1,      /* bad argument / descriptor                     */
  WG_ERR_RANGE = 2,        /* vertex id or type out of range                */
  WG_ERR_NOMEM = 3,        /* device allocation failed                      */
  WG_ERR_CUDA = 4,         /* CUDA runtime / kernel error                   */
  WG_ERR_UNSUPPORTED = 6,  /* valid but not implemented combination         */
  WG_ERR_STATE = 7         /* misuse of handles                             */
} wg_status;

/* WG_SAGE_LSTM: GraphSAGE with the LSTM aggregator (the paper's fifth model,
 * P:L3790-3814; reading Q26): fp32, full graphs.          */
typedef enum { WG_GCN = 0, WG_GIN = 1, WG_SAGE = 2, WG_GAT = 3, WG_RGCN = 4, WG_SAGE_LSTM = 5 } wg_model;
typedef enum { WG_F32 = 0, WG_BF16 = 1 } wg_dtype;
/* GCN [24] / RGCN [34] edge coefficient c_e (Q2, Q3):
 * NONE: 1; RIGHT: 1/deg_in(dst) (RGCN: 1/|in(dst) of type r|);
 * BOTH: deg_out(src)^-1/2 * deg_in(dst)^-1/2.  Degrees clamp to >= 1.    */
typedef enum { WG_NORM_NONE = 0, WG_NORM_RIGHT = 1, WG_NORM_BOTH = 2 } wg_norm;
/* Per-gTask operation plan (a4): EDGE = gather-then-transform, VERTEX =
 * transform-before-gather (T2 "indexing swapping").          */
typedef enum { WG_PLAN_AUTO = 0, WG_PLAN_ALL_EDGE = 1, WG_PLAN_ALL_VERTEX = 2,
               WG_PLAN_RANDOM = 3 } wg_plan_policy;

typedef void* wg_stream;                 /* a cudaStream_t value (0 = legacy) */
typedef struct wg_graph_s* wg_graph;
typedef struct wg_plan_s* wg_plan;

/* ------------------------------------------------------------------------ */
/* Graph ingest + gTask partition (a1-a3).                                  */
/* Edge attributes src-id / dst-id / edge-type (Fig 5a).      */
/* ------------------------------------------------------------------------ */
typedef struct {
  int64_t num_vertices;     /* V (global), 1 <= V < 2^31                          */
  int64_t num_edges;        /* E, 0 <= E < 2^31                                   */
  const int64_t* indptr;    /* CSR over dst, length V+1; NULL => COO (dst given)  */
  const int32_t* src;       /* length E                                           */
  const int32_t* dst;       /* length E (COO); ignored when indptr != NULL        */
  const int32_t* etype;     /* length E, in [0, num_types); NULL => one relation  */
  int32_t num_types;        /* R >= 1; gTasks are split by type iff R > 1 && etype */
  int32_t tile_rows;        /* T (dst-range restriction, Q11); 0 => 128           */
  int64_t max_task_edges;   /* E_max (uniq(edge-id) <= E_max, Q13); 0 => default  */
  int64_t v_begin, v_end;   /* owned vertex range for a 1-D partition (multiple of */
                            /* T, except v_end == V); both 0 => [0, V)            */
} wg_graph_desc;
/* Pointers may be host or device memory (detected with
 * cudaPointerGetAttributes); the call copies what it needs and returns after
 * the partition is complete (synchronous on `stream`).                      */

/* gTask record (D5).  Forward graph: key vertex = dst; transposed graph
 * (backward): key vertex = src.  e_begin/e_end are positions in this
 * graph's perm order; tile / d_lo / d_hi are GLOBAL vertex-derived ids.     */
typedef struct {
  int32_t tile, type;
  int64_t e_begin, e_end;
  int32_t d_lo, d_hi;       /* first / last key vertex                            */
  int32_t flags;            /* WG_TASK_SPLIT: chunk of a key segment > E_max      */
  int32_t n_uniq_src;       /* distinct other-endpoint ids in the task            */
} wg_task;
#define WG_TASK_SPLIT 1

wg_status wg_graph_create(const wg_graph_desc* desc, int device, wg_stream stream, wg_graph* out);
/* info[0..9]: V, owned rows, E_fwd (local in-edges), E_T (local out-edges),
 * n_tasks, n_tasks_T, T, E_max, by_type, max in-degree                      */
wg_status wg_graph_info(wg_graph g, int64_t info[10]);
/* Copies the partition to HOST memory.  transposed = 0: forward tables
 * (perm = GLOBAL edge ids in sorted order); 1: transposed tables.  fwdpos
 * (transposed only, may be NULL): fwdpos_of_T[j] = inv(perm)[perm_T[j]],
 * valid when the graph owns all rows.                                      */
wg_status wg_graph_export(wg_graph g, int transposed, int64_t* perm, wg_task* tasks, int64_t* fwdpos);
wg_status wg_graph_destroy(wg_graph g);

/* ------------------------------------------------------------------------ */
/* Plan (a4): per-gTask EDGE / VERTEX choice by an integer cost model of     */
/* FLOP + memory volume.             */
/* ------------------------------------------------------------------------ */
typedef struct {
  wg_model model;
  wg_dtype dtype;
  int32_t f_in, f_out;      /* GAT: f_out is per head                            */
  int32_t heads;            /* GAT only (>= 1)                                   */
  int32_t concat_heads;     /* GAT: 1 = concat heads, 0 = mean (last layer, Q6)  */
  wg_norm norm;             /* GCN / RGCN                                        */
  int32_t self_loop;        /* RGCN: add x[v] W_0                                */
  int32_t bias;             /* add a bias                                        */
  int32_t fuse_relu;        /* ReLU applied to the conv output (Q7)              */
  float gin_eps;            /* GIN epsilon (Q5: 0)                               */
  float neg_slope;          /* GAT LeakyReLU slope (Q6: 0.2)                     */
  wg_plan_policy policy;
  uint64_t policy_seed;     /* WG_PLAN_RANDOM                                    */
  int32_t need_dx;          /* backward produces dx (0 for the input layer)      */
  int32_t x_replicated;     /* 1-D partition: the layer's input rows are on every */
                            /* rank already (the input features); 0: exchanged  */
} wg_conv_desc;

/* Errors: WG_ERR_INVALID (bad sizes / model / dtype), WG_ERR_UNSUPPORTED
 * (typed graph with a non-RGCN model; GAT on a graph that owns only a row
 * block -- the 1-D partition covers GCN / SAGE / GIN / RGCN).  GAT also
 * needs f_out * sizeof(dtype) to be a multiple of 16 bytes (one head's row
 * slice is a whole number of 16-byte vectors); otherwise wg_conv_forward
 * returns WG_ERR_UNSUPPORTED.                                              */
wg_status wg_plan_create(wg_graph g, const wg_conv_desc* desc, wg_plan* out);
/* Bytes of the caller-owned `saved` (forward -> backward) and `workspace`
 * buffers; both 256-byte aligned device memory.                            */
wg_status wg_plan_sizes(wg_plan p, size_t* saved_bytes, size_t* workspace_bytes);
/* per_task_plan (host, n_tasks bytes, may be NULL): 0 = EDGE, 1 = VERTEX.
 * stats (host, may be NULL) [0..7]: n EDGE tasks, n VERTEX tasks, backward
 * path (0 = dAgg, 1 = G), exchange width fwd, exchange width bwd (columns
 * of the table the layer exchanges on a 1-D partition, 0 = none: an EDGE
 * layer's forward reads the activation itself), n work items fwd, n work
 * items T, n split rows fwd.                                               */
wg_status wg_plan_export(wg_plan p, uint8_t* per_task_plan, int64_t stats[8]);
/* Introspection (tests / tools): byte offset of a named sub-buffer of the
 * saved (which = 0) or workspace (which = 1) buffer, e.g. "agg" (the saved
 * aggregation, [owned rows x pitch(f_in)]) or "h" (GIN hidden activation,
 * [owned rows x pitch(f_out)]) or "xg" (RGCN on one partition with every
 * gTask VERTEX: x[src] of each (source, relation) row, grouped by relation,
 * gathered once by the forward for the Y GEMM and reused by the dW_r GEMM,
 * SURVEY §8(a) a5 / a11).  WG_ERR_INVALID if the plan has no such
 * buffer.  Row pitches: <= 32 / <= 64-byte rows padded to 32 / 64 bytes,
 * longer rows to a multiple of 128 bytes (one L2 line), in the conv dtype. */
wg_status wg_plan_buffer(wg_plan p, int which, const char* name, size_t* offset);
wg_status wg_plan_destroy(wg_plan p);

/* ------------------------------------------------------------------------ */
/* Forward / backward (a5-a11).  Parameters (fp32, device):                  */
/*   GCN : W [f_in x f_out], bias [f_out]                                   */
/*   SAGE: W = W_neigh, W_self [f_in x f_out], bias [f_out]                 */
/*   GIN : W = W1 [f_in x f_out], bias = b1, W2 [f_out x f_out], b2         */
/*   GAT : W [f_in x heads*f_out], attn_l / attn_r [heads x f_out],         */
/*         bias [heads*f_out] (concat) or [f_out] (mean)                    */
/*   RGCN: W [R x f_in x f_out], W_self = W_0 (self_loop), bias             */
/*   SAGE-LSTM: W = W_n [f_in x f_out], W_self = W_s, bias, Wih / Whh       */
/*         [f_in x 4 f_in] (gate column blocks i | f | g | o), bl [4 f_in]   */
/* ------------------------------------------------------------------------ */
typedef struct {
  const float *W, *W_self, *bias, *attn_l, *attn_r, *W2, *b2, *Wih, *Whh, *bl;
} wg_params;
typedef struct {
  float *W, *W_self, *bias, *attn_l, *attn_r, *W2, *b2, *Wih, *Whh, *bl;   /* NULL => skip */
} wg_grads;

/* Phases for the 1-D multi-GPU layer (§8(e)).  Single GPU: WG_PHASE_ALL.
 * PRE computes this rank's rows of the exchange table into
 * `xchg + row_offset * ld_xchg`; the caller all-gathers `xchg` (in place);
 * POST consumes the gathered table.  GCN / SAGE backward tables carry the
 * destination's normalisation already (dT * c_dst on the G path, dAgg * c_dst
 * on the dAgg path, c_dst = 1/deg_in or deg_in^-1/2), so POST reads no
 * per-edge scale; the table is opaque to the caller.  RGCN: the forward has no exchange
 * (x must hold all rows: PRE does nothing, POST = ALL); the backward
 * exchange table is dT = dy (masked by the fused ReLU), f_out wide.  GAT
 * plans accept only WG_PHASE_ALL (and only on a full graph, see
 * wg_plan_create): other phases return WG_ERR_UNSUPPORTED.                  */
typedef enum { WG_PHASE_ALL = 0, WG_PHASE_PRE = 1, WG_PHASE_POST = 2 } wg_phase;

typedef struct {
  int32_t phase;
  const void* x;            /* [V_global x ldx]: all rows (gathered when distributed) */
  int64_t ldx;
  void* y;                  /* [owned rows x ldy] output                          */
  int64_t ldy;
  void* saved;              /* wg_plan_sizes().saved bytes                        */
  void* workspace;          /* wg_plan_sizes().workspace bytes                    */
  void* xchg;               /* exchange table [V_global x ld_xchg] (or NULL)      */
  int64_t ld_xchg;
} wg_fwd_args;

typedef struct {
  int32_t phase;
  const void* dy;           /* [owned rows x lddy] gradient of the conv output    */
  int64_t lddy;
  const void* x;            /* forward input, as in wg_fwd_args                   */
  int64_t ldx;
  const void* y;            /* forward output (needed when fuse_relu)             */
  int64_t ldy;
  const void* saved;
  void* dx;                 /* [owned rows x lddx], written when need_dx          */
  int64_t lddx;
  void* workspace;
  void* xchg;
  int64_t ld_xchg;
  /* Fusion of adjacent layers (optional, NULL / 0 = off):
   * dx_mask: dx is written already multiplied by [dx_mask > 0] (the ReLU of
   *          the layer that produced x), row-major [owned rows x ld_dx_mask];
   * dy_masked: dy already carries this layer's fused-ReLU mask (as produced
   *          by the next layer's dx_mask), so y is not read.               */
  const void* dx_mask;
  int64_t ld_dx_mask;
  int32_t dy_masked;
} wg_bwd_args;

/* Forward: h^{l+1} of Eq. (1) (§2 "GNN model": "h^{l+1}[e.dst]
 * += MLP(h^l[e.src], W^l[e.type])") for the model's message function and
 * per-vertex terms (DESIGN.md §2 Q1-Q7); the gTask plan decides the operation
 * order (T2 indexing swapping) but not the result.  Backward:
 * the exact gradients of that definition (the paper is silent, Q8), the
 * transposed gather running over the transposed gTask partition.
 * Errors: WG_ERR_INVALID for null / misaligned arguments (ld * sizeof(dtype)
 * not a multiple of 16, ld < F), a missing saved / workspace / exchange
 * buffer, or a phase the plan does not accept; WG_ERR_UNSUPPORTED for
 * combinations listed at wg_plan_create; WG_ERR_CUDA for a launch failure
 * (kernel faults surface on a later call).  Asynchronous on `stream`.      */
wg_status wg_conv_forward(wg_plan p, const wg_params* params, const wg_fwd_args* a, wg_stream stream);
wg_status wg_conv_backward(wg_plan p, const wg_params* params, const wg_bwd_args* a,
                           const wg_grads* grads, wg_stream stream);

/* ------------------------------------------------------------------------ */
/* Multi-GPU layer (the paper's data-parallel scheme          */
/* P:L2199-2229, Fig 11; transform-before-communicate P:L2279-2289).         */
/* One process per GPU.  Rank p owns the T-aligned vertex block              */
/* [b_p, b_{p+1}) of every activation / gradient table, the forward gTasks   */
/* of those rows and the transposed gTasks of their out-edges.  Per layer    */
/* the table the gathers read is exchanged over NCCL (all-gather-v of the    */
/* row blocks) on the communicator's own high-priority stream; GCN / SAGE    */
/* exchange tables are column-chunked so the gather of chunk k overlaps the  */
/* exchange of chunk k+1.  Weight gradients are all-reduced (sum).           */
/* NCCL is the process's own libnccl.so.2 (loaded by torch), resolved at    */
/* run time; without it these calls return WG_ERR_UNSUPPORTED.               */
/* ------------------------------------------------------------------------ */
typedef struct wg_comm_s* wg_comm;
#define WG_COMM_ID_BYTES 128

/* 128-byte ncclUniqueId (call on one rank, broadcast it out of band, e.g.
 * through torch.distributed).                                              */
wg_status wg_comm_unique_id(void* id);
/* Collective over the `world` ranks (blocking until all have joined).      */
wg_status wg_comm_init(const void* id, int rank, int world, int device, wg_comm* out);
/* One-GPU emulation of rank `rank` of a `world`-way partition: with copy = 1
 * every exchange is a copy kernel on the communication stream that re-reads
 * and re-writes the non-owned rows (the HBM bytes an all-gather moves, with
 * WG_EMU_CTAS CTAs, default 40: ~0.7 TB/s, an NVLink 5 all-gather's rate); copy = 0
 * skips exchanges (the rank's compute alone).  No data moves between ranks
 * and gradients are not reduced.  For timing one rank on one GPU
 * (bench.py --rank-slice), not for results.                                */
wg_status wg_comm_init_emulated(int rank, int world, int device, int copy, wg_comm* out);
/* info: rank, world, device, emulated                                      */
wg_status wg_comm_info(wg_comm c, int32_t info[4]);
/* `stream` waits for the communicator's outstanding work (the gradient
 * all-reduce that wg_conv_backward_dist leaves running).                   */
wg_status wg_comm_wait(wg_comm c, wg_stream stream);
wg_status wg_comm_destroy(wg_comm c);

/* Edge-balanced 1-D partition (host computation, deterministic, so every
 * rank computes the same bounds from the same global graph): bounds[0..world]
 * with bounds[0] = 0, bounds[world] = V, interior bounds multiples of T
 * (desc->tile_rows), each rank >= 1 tile, chosen greedily so each rank's
 * in-edges + out-edges + rows are ~1/world of the total.  desc is the GLOBAL
 * graph (pointers host or device).  WG_ERR_INVALID if V has fewer tiles than
 * ranks.                                                                    */
wg_status wg_partition_1d(const wg_graph_desc* desc, int world, int64_t* bounds);
/* This rank's graph of the partition: `global` describes the whole graph (or
 * any superset of the edges touching this rank's block); bounds (nullable:
 * wg_partition_1d) fixes every rank's block.  Returns the owned range.      */
wg_status wg_graph_create_dist(wg_comm c, const wg_graph_desc* global, const int64_t* bounds, int device,
                               wg_stream stream, wg_graph* out, int64_t* v_begin, int64_t* v_end);
/* bounds[0..n_ranks] of a graph made by wg_graph_create_dist (n_ranks = 0 otherwise). */
wg_status wg_graph_bounds(wg_graph g, int64_t* bounds, int32_t* n_ranks);
/* Plan with ONE layer-level plan on every rank (the ranks exchange one
 * table): WG_PLAN_AUTO sums the ranks' a4 layer costs (an all-reduce) and
 * takes all-EDGE or all-VERTEX; WG_PLAN_RANDOM (mixed) is UNSUPPORTED.      */
wg_status wg_plan_create_dist(wg_comm c, wg_graph g, const wg_conv_desc* desc, wg_plan* out);
/* Exchange table of a plan, dir 0 = forward, 1 = backward.  info[0] rows
 * (= V, global vertex ids), info[1] row pitch of a chunk (elements),
 * info[2] chunks C, info[3] bytes (0: the layer exchanges no table).  The
 * table is C chunks, chunk k = [rows x info[1]] row-major at byte offset
 * k * rows * info[1] * sizeof(dtype); pass ld_xchg = info[1].  Caller-owned
 * device memory.                                                            */
wg_status wg_plan_xchg(wg_plan p, int dir, int64_t info[4]);
/* Forward of one layer on every rank (a->phase must be WG_PHASE_ALL; x is
 * [V x ldx] global rows).  EDGE / RGCN layers gather raw rows of x: unless
 * x_gathered, this call first all-gathers x's row blocks IN PLACE (the owned
 * rows must be current, e.g. written by the previous layer).  VERTEX layers
 * write Y = x W of the owned rows into a->xchg, exchange it chunk by chunk
 * and gather each chunk as it arrives.  y holds the owned rows.  Stream-
 * ordered on `stream`; the communicator's stream is joined before return.  */
wg_status wg_conv_forward_dist(wg_comm c, wg_plan p, const wg_params* params, const wg_fwd_args* a, int x_gathered,
                               wg_stream stream);
/* Backward of one layer on every rank (phase WG_PHASE_ALL): this rank's rows
 * of the backward table into a->xchg, chunked exchange, transposed gather
 * over the rank's out-edges; dx / dy hold owned rows.  The weight gradients
 * in `grads` are all-reduced (sum over ranks) on the communicator's stream
 * AFTER this call returns: call wg_comm_wait before reading them.          */
wg_status wg_conv_backward_dist(wg_comm c, wg_plan p, const wg_params* params, const wg_bwd_args* a,
                                const wg_grads* grads, wg_stream stream);

/* ------------------------------------------------------------------------ */
/* General restriction engine: the graph partition table  */
/* of §4.2 with arbitrary restrictions, the greedy of        */
/* P:L1431-1451, Fig 7 and Fig 9 instances.   */
/* ------------------------------------------------------------------------ */
typedef enum { WG_ATTR_DST = 0, WG_ATTR_SRC = 1, WG_ATTR_TYPE = 2, WG_ATTR_DST_DEGREE = 3,
               WG_ATTR_EDGE = 4 } wg_attr;
#define WG_UNIQ_MIN (-1)
/* uniq(attr) = k: at most k distinct values of the attribute among a
 * gTask's edges (k >= 1); k = WG_UNIQ_MIN: uniq(attr) = min, gTasks with
 * fewer distinct values preferred (orders the scan, never cuts a gTask).
 * dst-degree is the in-degree of the edge's destination.          */
typedef struct { int32_t attr, k; } wg_restriction;
typedef struct wg_gpart_s* wg_gpart;
/* Partition the edges of `desc` (a full graph; v_begin / v_end ignored):
 * sort key = the uniq = 1 attributes (restriction order), then the min
 * attributes, then the uniq = k > 1 attributes except edge-id, then dst-id if
 * absent, then edge-id (Q25); a greedy scan then cuts a gTask
 * whenever an edge would bring a k-th + 1 distinct value.  Each attribute at
 * most once; the sum of k over k > 1 attributes (edge-id excluded) <= 2048
 * (WG_ERR_UNSUPPORTED beyond).  Task records: tile = -1, type of the first
 * edge, d_lo / d_hi = smallest / largest dst-id, flags 0, n_uniq_src.
 * Synchronous on `stream`; pointers host or device.                         */
wg_status wg_gpart_create(const wg_graph_desc* desc, const wg_restriction* r, int32_t n_r, int device,
                          wg_stream stream, wg_gpart* out);
/* info: V, E, number of gTasks                                             */
wg_status wg_gpart_info(wg_gpart g, int64_t info[3]);
/* HOST copies: perm[E] (edge ids in scan order), tasks[n] (either may be NULL). */
wg_status wg_gpart_export(wg_gpart g, int64_t* perm, wg_task* tasks);
/* Bytes of the workspace wg_gpart_aggregate needs for width F.             */
size_t wg_gpart_workspace(wg_gpart g, int32_t F);
/* Agg[v] = sum_{e: dst_e = v} c_e x[src_e] (the Index / Index-add pair,
 * P:L520-536) executed over the gTasks of ANY restriction set: gTasks may
 * share destinations, so fp32 partial rows are added with vector atomics
 * (one per run of equal destinations) and a finishing pass applies the
 * destination scale and the cast (RNE for bf16).  c_e per `norm` as for GCN
 * (Q3).  Row-major x [V x ldx], out [V x ldo] in dtype; F % 4 == 0.  The
 * atomic order varies between runs (results agree to fp32 rounding).        */
wg_status wg_gpart_aggregate(wg_gpart g, wg_dtype dtype, int32_t F, wg_norm norm, const void* x, int64_t ldx,
                             void* out, int64_t ldo, void* workspace, wg_stream stream);
wg_status wg_gpart_destroy(wg_gpart g);

/* ------------------------------------------------------------------------ */
/* Training-step utility: fused softmax cross-entropy over the last layer's
 * logits [M x ld] (C classes): loss_out[0] = scale * sum_r -log softmax(x_r)[label_r],
 * dlogits = scale * (softmax(x_r) - onehot(label_r)) in the conv dtype
 * (columns [C, round_up(C, 16 B)) written 0).  Deterministic (fixed-order
 * block partials).  scratch: WG_XENT_SCRATCH_BYTES of device memory.      */
#define WG_XENT_SCRATCH_BYTES 8192
wg_status wg_softmax_xent(wg_dtype dtype, int64_t M, int32_t C, const void* logits, int64_t ld,
                          const int64_t* labels, float scale, void* dlogits, int64_t ldd, float* loss_out,
                          void* scratch, wg_stream stream);

/* Training-step utility: one Adam step (Kingma & Ba; the update torch.optim.Adam
 * computes, no weight decay) over n fp32 values in one launch:
 *   m = b1 m + (1-b1) g ; v = b2 v + (1-b2) g^2 ; t = state[0] + 1 ;
 *   param -= lr / (1 - b1^t) * m / (sqrt(v) / sqrt(1 - b2^t) + eps).
 * param / grad / exp_avg / exp_avg_sq: device, n floats each, 16-byte
 * aligned, caller-owned (every parameter of a model in one flat buffer).
 * state: device int32[2] owned by the caller, zeroed before the first step;
 * state[0] = steps taken (advanced on the device by the launch, so a
 * captured CUDA graph replays successive steps), state[1] internal.
 * Concurrent calls must not share `state`.                                  */
wg_status wg_adam_step(int64_t n, float* param, const float* grad, float* exp_avg, float* exp_avg_sq,
                       int32_t* state, float lr, float beta1, float beta2, float eps, wg_stream stream);

/* ------------------------------------------------------------------------ */
const char* wg_status_string(wg_status s);
const char* wg_last_error(void);
/* Number of kernels this library has launched on the calling thread. */
int64_t wg_launch_count(void);

/* Live per-kernel-class timing (CUDA events recorded on the launching stream
 * around every launch of the class).  cmd 0: disable; 1: enable and reset;
 * 2: synchronize the recorded events and write, for each class k in
 * [0, WG_PROF_KINDS), out[4k+0] = total ms, out[4k+1] = launches,
 * out[4k+2] = algorithmic bytes, out[4k+3] = algorithmic flops.
 * Classes: 0 gather/segment-reduce (a6/a10), 1 split combine (a8),
 * 2 tcgen05 GEMM NT (a5/a7/a9), 3 tcgen05 GEMM TN + reduce (a11),
 * 4 CUDA-core GEMM, 5 small kernels (weight prep, bias grad),
 * 6 GAT edge kernels, 7 RGCN kernels.                                      */
#define WG_PROF_KINDS 8
wg_status wg_profile(int cmd, double* out);

#ifdef __cplusplus
}
#endif
#endif /* WG_H_ */
