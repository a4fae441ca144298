/*
 * oracle/wg_oracle.c -- TEST INFRASTRUCTURE, NOT PRODUCT CODE.
 *
 * A plain, slow, obviously-correct CPU reference for the gTask-partitioned
 * graph-convolution layer of WiseGraph (Huang et al., EuroSys '24).  Only
 * tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
 * reference legs may load it.  It shares no code, header, table or helper with
 * the CUDA path (paper_conf_eurosys_huangz0wjzzzys24_b200/csrc).
 *
 * Citations: "P:L<a>-<b>" are line ranges of the paper text, with
 * the section / figure / equation they fall in.  "Q<n>" are the readings of
 * DESIGN.md §"Readings of the paper" (the paper is silent on them).
 *
 * Arithmetic: every floating-point value is a double.  Callers upcast fp32 or
 * bf16 inputs exactly to double.  There is no blocking, fusion, reordering or
 * parallelism: each conv is the per-edge message loop of Eq. (1)
 * ("h^{l+1}[e.dst] += MLP(h^l[e.src], W^l[e.type])") followed by
 * the per-vertex terms the model definition adds.
 *
 * Parity pins (tests/test_oracle_*.py): worked example of Fig 5a / Fig 7
 * (P:L1203-1217), dense-adjacency brute force, torch.autograd
 * on the dense form for every backward, integer exactness, limit cases.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------------ */
/* gTask record (SURVEY.md §8(b) wg_task; 40 bytes, natural alignment).     */
typedef struct {
    int32_t tile, type;
    int64_t e_begin, e_end;   /* positions in perm order, [e_begin, e_end) */
    int32_t d_lo, d_hi;       /* first / last key vertex in the task       */
    int32_t flags;            /* 1 = SPLIT chunk of an over-long segment   */
    int32_t n_uniq_src;       /* distinct "other endpoint" ids in the task */
} wgo_task;

#define WGO_SPLIT 1

/* ======================================================================== */
/* Graph partition (§4.2-4.3; Fig 7).            */
/*                                                                          */
/* Restriction instance (Q10/Q11/Q13):                            */
/*   uniq(key-vertex range of T rows) = 1, uniq(edge-type) = 1 (by_type),   */
/*   uniq(edge-id) <= E_max, with whole key-vertex segments packed.         */
/* "We first sort the edges of the graph according to edge attributes       */
/*  involved in the restrictions.  Then we scan these edges in order. If a  */
/*  restriction condition is satisfied after including the current edge, we */
/*  add it to the current gTask ... If any restrictions are not satisfied   */
/*  ... we stop ... and start a new gTask".                  */
/* ======================================================================== */

static const int32_t* g_kv;     /* key vertex per edge (dst fwd, src transposed) */
static const int32_t* g_ty;     /* edge type or NULL                             */
static int32_t g_T;

static int32_t edge_type(int64_t e) { return g_ty ? g_ty[e] : 0; }

/* sort key (floor(kv/T), type, kv, eid): unique, so the order is total */
static int cmp_edges(const void* pa, const void* pb) {
    int64_t a = *(const int64_t*)pa, b = *(const int64_t*)pb;
    int32_t ta = g_kv[a] / g_T, tb = g_kv[b] / g_T;
    if (ta != tb) return ta < tb ? -1 : 1;
    int32_t ya = edge_type(a), yb = edge_type(b);
    if (ya != yb) return ya < yb ? -1 : 1;
    if (g_kv[a] != g_kv[b]) return g_kv[a] < g_kv[b] ? -1 : 1;
    return a < b ? -1 : (a > b ? 1 : 0);
}

static int cmp_i32(const void* pa, const void* pb) {
    int32_t a = *(const int32_t*)pa, b = *(const int32_t*)pb;
    return a < b ? -1 : (a > b ? 1 : 0);
}

static void close_task(wgo_task* tasks, int64_t* n, int32_t tile, int32_t type,
                       int64_t b, int64_t e, int32_t flags, const int64_t* perm) {
    wgo_task* t = &tasks[(*n)++];
    t->tile = tile;
    t->type = type;
    t->e_begin = b;
    t->e_end = e;
    t->d_lo = g_kv[perm[b]];
    t->d_hi = g_kv[perm[e - 1]];
    t->flags = flags;
    t->n_uniq_src = 0;
}

/*
 * kv[e]   : vertex the partition is keyed on (dst for the forward graph,
 *           src for the transposed graph used by backward).
 * ov[e]   : the other endpoint (counted by n_uniq_src).
 * etype   : NULL, or the edge type array (used only when by_type != 0).
 * perm    : out, length E: perm[i] = edge id at sorted position i.
 * tasks   : out, capacity E (+1): the gTask table in scan order.
 * returns : number of tasks.
 */
int64_t wgo_partition(int64_t E, const int32_t* kv, const int32_t* ov, const int32_t* etype,
                      int32_t by_type, int32_t T, int64_t E_max, int64_t* perm, wgo_task* tasks) {
    g_kv = kv;
    g_ty = by_type ? etype : NULL;
    g_T = T;
    for (int64_t i = 0; i < E; ++i) perm[i] = i;
    qsort(perm, (size_t)E, sizeof(int64_t), cmp_edges);      /* step 1 */

    int64_t n = 0;
    int64_t i = 0;
    while (i < E) {                                           /* step 2: groups */
        int32_t tile = kv[perm[i]] / T, type = edge_type(perm[i]);
        int64_t gend = i;
        while (gend < E && kv[perm[gend]] / T == tile && edge_type(perm[gend]) == type) ++gend;
        int64_t open_b = -1;                                  /* no open task */
        int64_t s = i;
        while (s < gend) {                                    /* step 3: segments */
            int64_t send = s;
            while (send < gend && kv[perm[send]] == kv[perm[s]]) ++send;
            int64_t len = send - s;
            if (len > E_max) {
                if (open_b >= 0) close_task(tasks, &n, tile, type, open_b, s, 0, perm);
                open_b = -1;
                for (int64_t c = s; c < send; c += E_max) {
                    int64_t ce = c + E_max < send ? c + E_max : send;
                    close_task(tasks, &n, tile, type, c, ce, WGO_SPLIT, perm);
                }
            } else if (open_b < 0) {
                open_b = s;
            } else if ((s - open_b) + len <= E_max) {
                /* append: the open task grows to [open_b, send) */
            } else {
                close_task(tasks, &n, tile, type, open_b, s, 0, perm);
                open_b = s;
            }
            s = send;
        }
        if (open_b >= 0) close_task(tasks, &n, tile, type, open_b, gend, 0, perm);
        i = gend;
    }

    /* step 4: n_uniq_src = number of distinct other-endpoint ids per task */
    int32_t* buf = (int32_t*)malloc(sizeof(int32_t) * (size_t)(E > 0 ? E : 1));
    for (int64_t t = 0; t < n; ++t) {
        int64_t m = 0;
        for (int64_t p = tasks[t].e_begin; p < tasks[t].e_end; ++p) buf[m++] = ov[perm[p]];
        qsort(buf, (size_t)m, sizeof(int32_t), cmp_i32);
        int32_t u = 0;
        for (int64_t p = 0; p < m; ++p) if (p == 0 || buf[p] != buf[p - 1]) ++u;
        tasks[t].n_uniq_src = u;
    }
    free(buf);
    return n;
}

/* ======================================================================== */
/* General restriction engine: the graph partition table */
/* of §4.2 with a restriction per edge attribute:           */
/*   uniq(a) = k  (k >= 1): at most k distinct values of a in a gTask;     */
/*   uniq(a) = min (k = -1): gTasks with fewer distinct values preferred;  */
/*   no entry: unrestricted.                                               */
/* Attributes: 0 dst-id, 1 src-id, 2 edge type, 3 dst-degree (the         */
/* in-degree of the edge's destination, an inherent attribute P:L1361),    */
/* 4 edge-id.  Greedy of P:L1431-1451: sort by the restricted attributes,  */
/* scan in order, add the edge if every restriction still holds, else     */
/* start a new gTask.  Readings (Q25): the sort key is the      */
/* uniq = 1 attributes (spec order), then the min attributes (spec        */
/* order: sorting by them groups equal values, which minimises the        */
/* distinct count the greedy packs), then the uniq = k > 1 attributes     */
/* other than edge-id (spec order), then dst-id if absent, then edge-id   */
/* (a total order).  Task record: tile = -1, type of the first edge,      */
/* d_lo / d_hi = smallest / largest dst-id, flags 0, n_uniq_src.          */
/* ======================================================================== */
static int32_t g_nkey;
static int32_t g_key[8];
static const int32_t *g_gsrc, *g_gdst, *g_gty;
static const int64_t* g_gdeg;

static int64_t attr_value(int32_t a, int64_t e) {
    switch (a) {
        case 0: return g_gdst[e];
        case 1: return g_gsrc[e];
        case 2: return g_gty ? g_gty[e] : 0;
        case 3: return g_gdeg[g_gdst[e]];
        default: return e;
    }
}

static int cmp_general(const void* pa, const void* pb) {
    int64_t a = *(const int64_t*)pa, b = *(const int64_t*)pb;
    for (int32_t i = 0; i < g_nkey; ++i) {
        int64_t va = attr_value(g_key[i], a), vb = attr_value(g_key[i], b);
        if (va != vb) return va < vb ? -1 : 1;
    }
    return 0;
}

/* attr[i], k[i]: n restrictions (each attribute at most once).  Returns the
 * number of tasks; perm / tasks as wgo_partition; -1 on a bad spec. */
int64_t wgo_partition_general(int64_t V, int64_t E, const int32_t* src, const int32_t* dst, const int32_t* etype,
                              const int32_t* attr, const int32_t* k, int32_t n, int64_t* perm, wgo_task* tasks) {
    int64_t* deg = (int64_t*)calloc((size_t)(V > 0 ? V : 1), sizeof(int64_t));
    for (int64_t e = 0; e < E; ++e) deg[dst[e]]++;
    g_gsrc = src; g_gdst = dst; g_gty = etype; g_gdeg = deg;
    /* sort key */
    int used[5] = {0, 0, 0, 0, 0};
    g_nkey = 0;
    for (int pass = 0; pass < 3; ++pass)
        for (int32_t i = 0; i < n; ++i) {
            if (attr[i] < 0 || attr[i] > 4) { free(deg); return -1; }
            int take = pass == 0 ? k[i] == 1 : pass == 1 ? k[i] == -1 : (k[i] > 1 && attr[i] != 4);
            if (take && !used[attr[i]]) { g_key[g_nkey++] = attr[i]; used[attr[i]] = 1; }
        }
    if (!used[0]) g_key[g_nkey++] = 0;
    g_key[g_nkey++] = 4;
    for (int64_t i = 0; i < E; ++i) perm[i] = i;
    qsort(perm, (size_t)E, sizeof(int64_t), cmp_general);
    /* greedy scan: per restricted attribute, the distinct values of the open task */
    int64_t* vals[5] = {0, 0, 0, 0, 0};
    int64_t cnt[5] = {0, 0, 0, 0, 0};
    for (int32_t i = 0; i < n; ++i)
        if (k[i] >= 1) vals[attr[i]] = (int64_t*)malloc(sizeof(int64_t) * (size_t)k[i]);
    int64_t nt = 0, open_b = 0;
    for (int64_t p = 0; p < E; ++p) {
        int64_t e = perm[p];
        int fits = 1;
        for (int32_t i = 0; i < n && fits; ++i) {
            if (k[i] < 1) continue;
            int32_t a = attr[i];
            int64_t v = attr_value(a, e), j;
            for (j = 0; j < cnt[a]; ++j) if (vals[a][j] == v) break;
            if (j == cnt[a] && cnt[a] == k[i]) fits = 0;      /* a new value beyond k */
        }
        if (!fits) {                                          /* close [open_b, p) */
            wgo_task* t = &tasks[nt++];
            t->e_begin = open_b; t->e_end = p;
            open_b = p;
            for (int a = 0; a < 5; ++a) cnt[a] = 0;
        }
        for (int32_t i = 0; i < n; ++i) {                     /* record the edge's values */
            if (k[i] < 1) continue;
            int32_t a = attr[i];
            int64_t v = attr_value(a, e), j;
            for (j = 0; j < cnt[a]; ++j) if (vals[a][j] == v) break;
            if (j == cnt[a]) vals[a][cnt[a]++] = v;
        }
    }
    if (E > 0) { tasks[nt].e_begin = open_b; tasks[nt].e_end = E; ++nt; }
    for (int a = 0; a < 5; ++a) free(vals[a]);
    /* task records */
    int32_t* buf = (int32_t*)malloc(sizeof(int32_t) * (size_t)(E > 0 ? E : 1));
    for (int64_t t = 0; t < nt; ++t) {
        wgo_task* r = &tasks[t];
        r->tile = -1;
        r->type = etype ? etype[perm[r->e_begin]] : 0;
        r->flags = 0;
        r->d_lo = dst[perm[r->e_begin]]; r->d_hi = r->d_lo;
        int64_t m = 0;
        for (int64_t q = r->e_begin; q < r->e_end; ++q) {
            int32_t d = dst[perm[q]];
            if (d < r->d_lo) r->d_lo = d;
            if (d > r->d_hi) r->d_hi = d;
            buf[m++] = src[perm[q]];
        }
        qsort(buf, (size_t)m, sizeof(int32_t), cmp_i32);
        int32_t u = 0;
        for (int64_t q = 0; q < m; ++q) if (q == 0 || buf[q] != buf[q - 1]) ++u;
        r->n_uniq_src = u;
    }
    free(buf);
    free(deg);
    return nt;
}

/* ======================================================================== */
/* Helpers: degrees and the GCN / RGCN edge coefficients.                  */
/* ======================================================================== */

static void degrees(int64_t V, int64_t E, const int32_t* src, const int32_t* dst,
                    int64_t* din, int64_t* dout) {
    for (int64_t v = 0; v < V; ++v) din[v] = dout[v] = 0;
    for (int64_t e = 0; e < E; ++e) { din[dst[e]]++; dout[src[e]]++; }
}

/* GCN [24] normalisation c_e (Q3): 0 = none, 1 = right 1/deg_in(d),
 * 2 = both deg_out(s)^-1/2 deg_in(d)^-1/2, degrees clamped to >= 1 (Q16). */
static double gcn_coef(int norm, int64_t ds_out, int64_t dd_in) {
    double a = (double)(ds_out > 1 ? ds_out : 1), b = (double)(dd_in > 1 ? dd_in : 1);
    if (norm == 2) return 1.0 / sqrt(a) / sqrt(b);
    if (norm == 1) return 1.0 / b;
    return 1.0;
}

/* y[0..fo) += c * (x[0..fi) . W[fi x fo])   -- one edge message (Eq. (1) MLP) */
static void add_msg(int fi, int fo, double c, const double* x, const double* W, double* y) {
    for (int j = 0; j < fo; ++j) {
        double s = 0.0;
        for (int k = 0; k < fi; ++k) s += x[k] * W[(int64_t)k * fo + j];
        y[j] += c * s;
    }
}

/* dx[0..fi) += c * (dy[0..fo) . W^T) ; dW += c * x^T dy  (exact gradients of add_msg) */
static void add_msg_grad(int fi, int fo, double c, const double* x, const double* W,
                         const double* dy, double* dx, double* dW) {
    if (!dx && !dW) return;   /* nothing requested for this edge (sampled-row checks) */
    for (int k = 0; k < fi; ++k) {
        double s = 0.0;
        for (int j = 0; j < fo; ++j) s += dy[j] * W[(int64_t)k * fo + j];
        if (dx) dx[k] += c * s;
        if (dW) for (int j = 0; j < fo; ++j) dW[(int64_t)k * fo + j] += c * x[k] * dy[j];
    }
}

/* row_mask: NULL = all rows, else only rows v with row_mask[v] != 0 are produced
 * (used to check sampled rows of full-size graphs one by one). */
#define ROW_ON(m, v) ((m) == NULL || (m)[v])

/* ======================================================================== */
/* GCN (Kipf & Welling [24]; Q1, Q3)            */
/*   y[v] = b + sum_{e in in(v)} c_e x[s_e] W                              */
/* ======================================================================== */
void wgo_gcn_forward(int64_t V, int64_t E, const int32_t* src, const int32_t* dst, int norm,
                     int fi, int fo, const double* x, const double* W, const double* b,
                     const uint8_t* row_mask, double* y) {
    int64_t* din = malloc(sizeof(int64_t) * V);
    int64_t* dout = malloc(sizeof(int64_t) * V);
    degrees(V, E, src, dst, din, dout);
    for (int64_t v = 0; v < V; ++v)
        for (int j = 0; j < fo; ++j) y[v * fo + j] = b ? b[j] : 0.0;
    for (int64_t e = 0; e < E; ++e) {
        if (!ROW_ON(row_mask, dst[e])) continue;
        add_msg(fi, fo, gcn_coef(norm, dout[src[e]], din[dst[e]]), x + (int64_t)src[e] * fi, W,
                y + (int64_t)dst[e] * fo);
    }
    free(din); free(dout);
}

/* dx[u] = sum_{e in out(u)} c_e dy[d_e] W^T ; dW = sum_e c_e x[s_e]^T dy[d_e] ; db = sum_v dy[v] */
void wgo_gcn_backward(int64_t V, int64_t E, const int32_t* src, const int32_t* dst, int norm,
                      int fi, int fo, const double* x, const double* W, const double* dy,
                      const uint8_t* row_mask, double* dx, double* dW, double* db) {
    int64_t* din = malloc(sizeof(int64_t) * V);
    int64_t* dout = malloc(sizeof(int64_t) * V);
    degrees(V, E, src, dst, din, dout);
    if (dx) memset(dx, 0, sizeof(double) * V * fi);
    if (dW) memset(dW, 0, sizeof(double) * fi * fo);
    if (db) {
        memset(db, 0, sizeof(double) * fo);
        for (int64_t v = 0; v < V; ++v) for (int j = 0; j < fo; ++j) db[j] += dy[v * fo + j];
    }
    for (int64_t e = 0; e < E; ++e) {
        int64_t s = src[e], d = dst[e];
        double c = gcn_coef(norm, dout[s], din[d]);
        add_msg_grad(fi, fo, c, x + s * fi, W, dy + d * fo,
                     (dx && ROW_ON(row_mask, s)) ? dx + s * fi : NULL, dW);
    }
    free(din); free(dout);
}

/* ======================================================================== */
/* GraphSAGE-mean (Hamilton et al. [14]; Q4)    */
/*   y[v] = b + x[v] W_s + (1/max(1,deg_in v)) sum_{e in in(v)} x[s_e] W_n  */
/* ======================================================================== */
void wgo_sage_forward(int64_t V, int64_t E, const int32_t* src, const int32_t* dst,
                      int fi, int fo, const double* x, const double* Ws, const double* Wn,
                      const double* b, const uint8_t* row_mask, double* y) {
    int64_t* din = malloc(sizeof(int64_t) * V);
    int64_t* dout = malloc(sizeof(int64_t) * V);
    degrees(V, E, src, dst, din, dout);
    for (int64_t v = 0; v < V; ++v) {
        for (int j = 0; j < fo; ++j) y[v * fo + j] = b ? b[j] : 0.0;
        if (ROW_ON(row_mask, v)) add_msg(fi, fo, 1.0, x + v * fi, Ws, y + v * fo);
    }
    for (int64_t e = 0; e < E; ++e) {
        int64_t d = dst[e];
        if (!ROW_ON(row_mask, d)) continue;
        add_msg(fi, fo, 1.0 / (double)(din[d] > 1 ? din[d] : 1), x + (int64_t)src[e] * fi, Wn,
                y + d * fo);
    }
    free(din); free(dout);
}

void wgo_sage_backward(int64_t V, int64_t E, const int32_t* src, const int32_t* dst,
                       int fi, int fo, const double* x, const double* Ws, const double* Wn,
                       const double* dy, const uint8_t* row_mask,
                       double* dx, double* dWs, double* dWn, double* db) {
    int64_t* din = malloc(sizeof(int64_t) * V);
    int64_t* dout = malloc(sizeof(int64_t) * V);
    degrees(V, E, src, dst, din, dout);
    if (dx) memset(dx, 0, sizeof(double) * V * fi);
    if (dWs) memset(dWs, 0, sizeof(double) * fi * fo);
    if (dWn) memset(dWn, 0, sizeof(double) * fi * fo);
    if (db) memset(db, 0, sizeof(double) * fo);
    for (int64_t v = 0; v < V; ++v) {
        if (db) for (int j = 0; j < fo; ++j) db[j] += dy[v * fo + j];
        add_msg_grad(fi, fo, 1.0, x + v * fi, Ws, dy + v * fo,
                     (dx && ROW_ON(row_mask, v)) ? dx + v * fi : NULL, dWs);
    }
    for (int64_t e = 0; e < E; ++e) {
        int64_t s = src[e], d = dst[e];
        add_msg_grad(fi, fo, 1.0 / (double)(din[d] > 1 ? din[d] : 1), x + s * fi, Wn, dy + d * fo,
                     (dx && ROW_ON(row_mask, s)) ? dx + s * fi : NULL, dWn);
    }
    free(din); free(dout);
}

/* ======================================================================== */
/* GIN (Xu et al., ICLR'19 -- not in the paper; BASELINE north_star; Q5)    */
/*   z[v] = (1+eps) x[v] + sum_{e in in(v)} x[s_e]                           */
/*   a = z W1 + b1 ;  h = ReLU(a) ;  y = h W2 + b2                           */
/* The ReLU decision is the oracle's own, [a > 0] in fp64 (ReLU'(0) = 0).   */
/* ======================================================================== */
static void gin_z_row(int64_t v, int fi, double eps, const double* x, double* zv) {
    for (int k = 0; k < fi; ++k) zv[k] = (1.0 + eps) * x[v * fi + k];
}

/* z for the rows of row_mask (all rows when NULL): self term, then one pass
 * over the edges adding x[s_e] into z[d_e] (the edge loop of Eq. (1)). */
static void gin_z(int64_t V, int64_t E, const int32_t* src, const int32_t* dst, int fi,
                  double eps, const double* x, const uint8_t* row_mask, double* z) {
    for (int64_t v = 0; v < V; ++v) if (ROW_ON(row_mask, v)) gin_z_row(v, fi, eps, x, z + v * fi);
    for (int64_t e = 0; e < E; ++e) {
        if (!ROW_ON(row_mask, dst[e])) continue;
        for (int k = 0; k < fi; ++k) z[(int64_t)dst[e] * fi + k] += x[(int64_t)src[e] * fi + k];
    }
}

/* row_mask (nullable): only rows v with row_mask[v] != 0 are produced.
 * z_out ([V x fi]) and a_out ([V x fo], the pre-activation) are optional
 * outputs for the produced rows. */
void wgo_gin_forward(int64_t V, int64_t E, const int32_t* src, const int32_t* dst, int fi, int fo,
                     double eps, const double* x, const double* W1, const double* b1,
                     const double* W2, const double* b2, const uint8_t* row_mask, double* y,
                     double* z_out, double* a_out) {
    double* z = z_out ? z_out : malloc(sizeof(double) * V * fi);
    double* a = malloc(sizeof(double) * fo);
    gin_z(V, E, src, dst, fi, eps, x, row_mask, z);
    for (int64_t v = 0; v < V; ++v) {
        if (!ROW_ON(row_mask, v)) continue;
        for (int j = 0; j < fo; ++j) a[j] = b1 ? b1[j] : 0.0;
        add_msg(fi, fo, 1.0, z + v * fi, W1, a);
        if (a_out) for (int j = 0; j < fo; ++j) a_out[v * fo + j] = a[j];
        for (int j = 0; j < fo; ++j) { a[j] = a[j] > 0.0 ? a[j] : 0.0; y[v * fo + j] = b2 ? b2[j] : 0.0; }
        add_msg(fo, fo, 1.0, a, W2, y + v * fo);
    }
    if (!z_out) free(z);
    free(a);
}

/* dW2 = h^T dy ; da = (dy W2^T) * [a > 0] ; dW1 = z^T da ; dz = da W1^T ;
 * dx[u] = (1+eps) dz[u] + sum_{e in out(u)} dz[d_e] ; db1 = sum da ; db2 = sum dy
 * dy_rows (nullable): rows of dy outside this set are ZERO (they are skipped);
 * every output is then the exact gradient for that dy (dx for all V). */
void wgo_gin_backward(int64_t V, int64_t E, const int32_t* src, const int32_t* dst, int fi, int fo,
                      double eps, const double* x, const double* W1, const double* b1,
                      const double* W2, const double* dy, const uint8_t* dy_rows, double* dx, double* dW1,
                      double* db1, double* dW2, double* db2) {
    double* z = malloc(sizeof(double) * V * fi);
    double* dz = malloc(sizeof(double) * V * fi);
    double* a = malloc(sizeof(double) * fo);
    double* h = malloc(sizeof(double) * fo);
    double* dh = malloc(sizeof(double) * fo);
    double* da = malloc(sizeof(double) * fo);
    gin_z(V, E, src, dst, fi, eps, x, dy_rows, z);
    memset(dz, 0, sizeof(double) * V * fi);
    if (dW1) memset(dW1, 0, sizeof(double) * fi * fo);
    if (dW2) memset(dW2, 0, sizeof(double) * fo * fo);
    if (db1) memset(db1, 0, sizeof(double) * fo);
    if (db2) memset(db2, 0, sizeof(double) * fo);
    for (int64_t v = 0; v < V; ++v) {
        if (!ROW_ON(dy_rows, v)) continue;
        for (int j = 0; j < fo; ++j) a[j] = b1 ? b1[j] : 0.0;
        add_msg(fi, fo, 1.0, z + v * fi, W1, a);
        for (int j = 0; j < fo; ++j) {
            h[j] = a[j] > 0.0 ? a[j] : 0.0;
            dh[j] = 0.0;
        }
        if (db2) for (int j = 0; j < fo; ++j) db2[j] += dy[v * fo + j];
        add_msg_grad(fo, fo, 1.0, h, W2, dy + v * fo, dh, dW2);
        for (int j = 0; j < fo; ++j) da[j] = a[j] > 0.0 ? dh[j] : 0.0;
        if (db1) for (int j = 0; j < fo; ++j) db1[j] += da[j];
        add_msg_grad(fi, fo, 1.0, z + v * fi, W1, da, dz + v * fi, dW1);
    }
    if (dx) {
        for (int64_t u = 0; u < V; ++u) for (int k = 0; k < fi; ++k) dx[u * fi + k] = (1.0 + eps) * dz[u * fi + k];
        for (int64_t e = 0; e < E; ++e) {
            if (!ROW_ON(dy_rows, dst[e])) continue;
            for (int k = 0; k < fi; ++k) dx[(int64_t)src[e] * fi + k] += dz[(int64_t)dst[e] * fi + k];
        }
    }
    free(z); free(dz); free(a); free(h); free(dh); free(da);
}

/* ======================================================================== */
/* RGCN, Eq. (1), Schlichtkrull et al. [34] (Q2) */
/*   y[v] = sum_{e in in(v)} c_e x[s_e] W_{r_e}  (+ x[v] W_0) (+ b)          */
/*   c_e = 1 (norm 0, Eq. (1)) or 1/|{e' in in(v): r_e' = r_e}| (norm 1).   */
/* W: [R x fi x fo] row-major.                                              */
/* ======================================================================== */
static int64_t* rel_in_degree(int64_t V, int64_t E, int R, const int32_t* dst, const int32_t* et) {
    int64_t* c = calloc((size_t)V * R, sizeof(int64_t));
    for (int64_t e = 0; e < E; ++e) c[(int64_t)dst[e] * R + (et ? et[e] : 0)]++;
    return c;
}

void wgo_rgcn_forward(int64_t V, int64_t E, const int32_t* src, const int32_t* dst,
                      const int32_t* etype, int R, int norm, int fi, int fo, const double* x,
                      const double* W, const double* W0, const double* b, const uint8_t* row_mask,
                      double* y) {
    int64_t* c = rel_in_degree(V, E, R, dst, etype);
    for (int64_t v = 0; v < V; ++v) {
        for (int j = 0; j < fo; ++j) y[v * fo + j] = b ? b[j] : 0.0;
        if (W0 && ROW_ON(row_mask, v)) add_msg(fi, fo, 1.0, x + v * fi, W0, y + v * fo);
    }
    for (int64_t e = 0; e < E; ++e) {
        int64_t d = dst[e];
        if (!ROW_ON(row_mask, d)) continue;
        int r = etype ? etype[e] : 0;
        double ce = norm == 1 ? 1.0 / (double)c[d * R + r] : 1.0;
        add_msg(fi, fo, ce, x + (int64_t)src[e] * fi, W + (int64_t)r * fi * fo, y + d * fo);
    }
    free(c);
}

void wgo_rgcn_backward(int64_t V, int64_t E, const int32_t* src, const int32_t* dst,
                       const int32_t* etype, int R, int norm, int fi, int fo, const double* x,
                       const double* W, const double* W0, const double* dy,
                       const uint8_t* row_mask, double* dx, double* dW, double* dW0, double* db) {
    int64_t* c = rel_in_degree(V, E, R, dst, etype);
    if (dx) memset(dx, 0, sizeof(double) * V * fi);
    if (dW) memset(dW, 0, sizeof(double) * R * fi * fo);
    if (dW0) memset(dW0, 0, sizeof(double) * fi * fo);
    if (db) memset(db, 0, sizeof(double) * fo);
    for (int64_t v = 0; v < V; ++v) {
        if (db) for (int j = 0; j < fo; ++j) db[j] += dy[v * fo + j];
        if (W0) add_msg_grad(fi, fo, 1.0, x + v * fi, W0, dy + v * fo,
                             (dx && ROW_ON(row_mask, v)) ? dx + v * fi : NULL, dW0);
    }
    for (int64_t e = 0; e < E; ++e) {
        int64_t s = src[e], d = dst[e];
        int r = etype ? etype[e] : 0;
        double ce = norm == 1 ? 1.0 / (double)c[d * R + r] : 1.0;
        add_msg_grad(fi, fo, ce, x + s * fi, W + (int64_t)r * fi * fo, dy + d * fo,
                     (dx && ROW_ON(row_mask, s)) ? dx + s * fi : NULL,
                     dW ? dW + (int64_t)r * fi * fo : NULL);
    }
    free(c);
}

/* ======================================================================== */
/* GAT (Velickovic et al. [40]; Q6)             */
/* per head k: g_k = x W_k ; el[u] = g_k[u].a_l,k ; er[v] = g_k[v].a_r,k     */
/*   t_e = el[s_e] + er[d_e] ; l_e = t_e > 0 ? t_e : slope * t_e            */
/*   alpha_e = exp(l_e - m_v) / sum_{e' in in(v)} exp(l_e' - m_v)            */
/*   y_k[v] = sum_{e in in(v)} alpha_e g_k[s_e]                             */
/* concat != 0: y = [y_0 | ... | y_{H-1}] + b  ([V x H*fo], b [H*fo])       */
/* concat == 0: y = (1/H) sum_k y_k + b        ([V x fo],  b [fo])          */
/* W: [fi x H*fo] (head k = columns k*fo..k*fo+fo-1); a_l, a_r: [H x fo].   */
/* ======================================================================== */
static void gat_prep(int64_t V, int fi, int H, int fo, const double* x, const double* W,
                     const double* al, const double* ar, double* g, double* el, double* er) {
    int HF = H * fo;
    for (int64_t v = 0; v < V; ++v) {
        for (int j = 0; j < HF; ++j) g[v * HF + j] = 0.0;
        add_msg(fi, HF, 1.0, x + v * fi, W, g + v * HF);
        for (int k = 0; k < H; ++k) {
            double sl = 0.0, sr = 0.0;
            for (int j = 0; j < fo; ++j) {
                sl += g[v * HF + k * fo + j] * al[k * fo + j];
                sr += g[v * HF + k * fo + j] * ar[k * fo + j];
            }
            el[v * H + k] = sl;
            er[v * H + k] = sr;
        }
    }
}

/* alpha[e*H + k] for every edge (plain two passes over the edges) */
static void gat_alpha(int64_t V, int64_t E, const int32_t* src, const int32_t* dst, int H,
                      double slope, const double* el, const double* er, double* t, double* alpha) {
    double* m = malloc(sizeof(double) * V * H);
    double* den = calloc((size_t)V * H, sizeof(double));
    for (int64_t i = 0; i < V * H; ++i) m[i] = -INFINITY;
    for (int64_t e = 0; e < E; ++e)
        for (int k = 0; k < H; ++k) {
            double te = el[(int64_t)src[e] * H + k] + er[(int64_t)dst[e] * H + k];
            t[e * H + k] = te;
            double le = te > 0.0 ? te : slope * te;
            int64_t i = (int64_t)dst[e] * H + k;
            if (le > m[i]) m[i] = le;
        }
    for (int64_t e = 0; e < E; ++e)
        for (int k = 0; k < H; ++k) {
            double te = t[e * H + k], le = te > 0.0 ? te : slope * te;
            den[(int64_t)dst[e] * H + k] += exp(le - m[(int64_t)dst[e] * H + k]);
        }
    for (int64_t e = 0; e < E; ++e)
        for (int k = 0; k < H; ++k) {
            double te = t[e * H + k], le = te > 0.0 ? te : slope * te;
            int64_t i = (int64_t)dst[e] * H + k;
            alpha[e * H + k] = exp(le - m[i]) / den[i];
        }
    free(m); free(den);
}

void wgo_gat_forward(int64_t V, int64_t E, const int32_t* src, const int32_t* dst, int fi, int H,
                     int fo, int concat, double slope, const double* x, const double* W,
                     const double* al, const double* ar, const double* b, double* y,
                     double* alpha_out /* nullable, [E x H] */) {
    int HF = H * fo;
    double* g = malloc(sizeof(double) * V * HF);
    double* el = malloc(sizeof(double) * V * H);
    double* er = malloc(sizeof(double) * V * H);
    double* t = malloc(sizeof(double) * (E > 0 ? E : 1) * H);
    double* alpha = malloc(sizeof(double) * (E > 0 ? E : 1) * H);
    gat_prep(V, fi, H, fo, x, W, al, ar, g, el, er);
    gat_alpha(V, E, src, dst, H, slope, el, er, t, alpha);
    int FO = concat ? HF : fo;
    for (int64_t v = 0; v < V; ++v) for (int j = 0; j < FO; ++j) y[v * FO + j] = b ? b[j] : 0.0;
    for (int64_t e = 0; e < E; ++e)
        for (int k = 0; k < H; ++k)
            for (int j = 0; j < fo; ++j) {
                double msg = alpha[e * H + k] * g[(int64_t)src[e] * HF + k * fo + j];
                if (concat) y[(int64_t)dst[e] * FO + k * fo + j] += msg;
                else y[(int64_t)dst[e] * FO + j] += msg / (double)H;
            }
    if (alpha_out) memcpy(alpha_out, alpha, sizeof(double) * E * H);
    free(g); free(el); free(er); free(t); free(alpha);
}

/* Exact gradients of wgo_gat_forward (the paper is silent on backward, Q8):
 *   dy_k = dy[:, k] (concat) or dy / H (mean)
 *   dalpha_e = dy_k[d_e] . g_k[s_e]
 *   dl_e = alpha_e (dalpha_e - sum_{e' in in(d_e)} alpha_e' dalpha_e')
 *   dt_e = dl_e * (t_e > 0 ? 1 : slope)
 *   del[u] = sum_{out(u)} dt ; der[v] = sum_{in(v)} dt
 *   dg_k[u] = sum_{e in out(u)} alpha_e dy_k[d_e] + del[u] a_l,k + der[u] a_r,k
 *   da_l,k = sum_u del[u] g_k[u] ; da_r,k = sum_v der[v] g_k[v]
 *   dW = x^T dg ; dx = dg W^T ; db = sum_v dy[v]                             */
void wgo_gat_backward(int64_t V, int64_t E, const int32_t* src, const int32_t* dst, int fi, int H,
                      int fo, int concat, double slope, const double* x, const double* W,
                      const double* al, const double* ar, const double* dy, double* dx,
                      double* dW, double* dal, double* dar, double* db) {
    int HF = H * fo, FO = concat ? HF : fo;
    double* g = malloc(sizeof(double) * V * HF);
    double* el = malloc(sizeof(double) * V * H);
    double* er = malloc(sizeof(double) * V * H);
    double* t = malloc(sizeof(double) * (E > 0 ? E : 1) * H);
    double* alpha = malloc(sizeof(double) * (E > 0 ? E : 1) * H);
    double* dal_e = malloc(sizeof(double) * (E > 0 ? E : 1) * H);
    double* sdst = calloc((size_t)V * H, sizeof(double));
    double* del = calloc((size_t)V * H, sizeof(double));
    double* der = calloc((size_t)V * H, sizeof(double));
    double* dg = calloc((size_t)V * HF, sizeof(double));
    gat_prep(V, fi, H, fo, x, W, al, ar, g, el, er);
    gat_alpha(V, E, src, dst, H, slope, el, er, t, alpha);
#define DYK(v, k, j) (concat ? dy[(int64_t)(v) * FO + (k) * fo + (j)] : dy[(int64_t)(v) * FO + (j)] / (double)H)
    for (int64_t e = 0; e < E; ++e)
        for (int k = 0; k < H; ++k) {
            double s = 0.0;
            for (int j = 0; j < fo; ++j) s += DYK(dst[e], k, j) * g[(int64_t)src[e] * HF + k * fo + j];
            dal_e[e * H + k] = s;
            sdst[(int64_t)dst[e] * H + k] += alpha[e * H + k] * s;
        }
    for (int64_t e = 0; e < E; ++e)
        for (int k = 0; k < H; ++k) {
            double dl = alpha[e * H + k] * (dal_e[e * H + k] - sdst[(int64_t)dst[e] * H + k]);
            double dt = dl * (t[e * H + k] > 0.0 ? 1.0 : slope);
            del[(int64_t)src[e] * H + k] += dt;
            der[(int64_t)dst[e] * H + k] += dt;
            for (int j = 0; j < fo; ++j)
                dg[(int64_t)src[e] * HF + k * fo + j] += alpha[e * H + k] * DYK(dst[e], k, j);
        }
    if (dal) memset(dal, 0, sizeof(double) * HF);
    if (dar) memset(dar, 0, sizeof(double) * HF);
    for (int64_t u = 0; u < V; ++u)
        for (int k = 0; k < H; ++k)
            for (int j = 0; j < fo; ++j) {
                dg[u * HF + k * fo + j] += del[u * H + k] * al[k * fo + j] + der[u * H + k] * ar[k * fo + j];
                if (dal) dal[k * fo + j] += del[u * H + k] * g[u * HF + k * fo + j];
                if (dar) dar[k * fo + j] += der[u * H + k] * g[u * HF + k * fo + j];
            }
#undef DYK
    if (dW) memset(dW, 0, sizeof(double) * fi * HF);
    if (dx) memset(dx, 0, sizeof(double) * V * fi);
    for (int64_t u = 0; u < V; ++u)
        add_msg_grad(fi, HF, 1.0, x + u * fi, W, dg + u * HF, dx ? dx + u * fi : NULL, dW);
    if (db) {
        memset(db, 0, sizeof(double) * FO);
        for (int64_t v = 0; v < V; ++v) for (int j = 0; j < FO; ++j) db[j] += dy[v * FO + j];
    }
    free(g); free(el); free(er); free(t); free(alpha); free(dal_e); free(sdst); free(del); free(der); free(dg);
}

/* ======================================================================== */
/* Bilinear probe of a linear-conv weight gradient at any size:             */
/*   u^T dW v = sum_e c_e (x[s_e].u) (dy[d_e].v)                            */
/* (the definition of dW = sum_e c_e x[s_e]^T dy[d_e], contracted).          */
/* coef: NULL => c_e = 1, else per-edge coefficients.                       */
/* ======================================================================== */
double wgo_dw_probe(int64_t E, const int32_t* src, const int32_t* dst, const double* coef,
                    int fi, int fo, const double* x, const double* dy, const double* u,
                    const double* v) {
    double acc = 0.0;
    for (int64_t e = 0; e < E; ++e) {
        double a = 0.0, c = 0.0;
        for (int k = 0; k < fi; ++k) a += x[(int64_t)src[e] * fi + k] * u[k];
        for (int j = 0; j < fo; ++j) c += dy[(int64_t)dst[e] * fo + j] * v[j];
        acc += (coef ? coef[e] : 1.0) * a * c;
    }
    return acc;
}

/* ======================================================================== */
/* GraphSAGE with the LSTM aggregator (Hamilton et al. [14]; the paper's    */
/* fifth model, SAGE-LSTM).     */
/* Readings (Q26): the neighbour sequence of v is its in-edges in */
/* edge-id order; LSTM hidden size H = f_in; gates in PyTorch order         */
/* (i, f, g, o), z = x_t W_ih + h_{t-1} W_hh + b_l with W_ih, W_hh          */
/* [f_in x 4H] (column blocks i | f | g | o); h_0 = c_0 = 0;                 */
/*   i = s(z_i), f = s(z_f), g = tanh(z_g), o = s(z_o),                      */
/*   c_t = f c_{t-1} + i g,  h_t = o tanh(c_t);                              */
/* h_N(v) = h_deg(v) (0 for an isolated v);                                  */
/*   y[v] = b + x[v] W_s + h_N(v) W_n.                                       */
/* ======================================================================== */
static double sigm(double z) { return 1.0 / (1.0 + exp(-z)); }

/* in-edges of every vertex in edge-id order: counting sort by dst */
static void in_lists(int64_t V, int64_t E, const int32_t* dst, int64_t* ptr, int64_t* eid) {
    memset(ptr, 0, sizeof(int64_t) * (V + 1));
    for (int64_t e = 0; e < E; ++e) ptr[dst[e] + 1]++;
    for (int64_t v = 0; v < V; ++v) ptr[v + 1] += ptr[v];
    int64_t* fill = (int64_t*)malloc(sizeof(int64_t) * (V > 0 ? V : 1));
    for (int64_t v = 0; v < V; ++v) fill[v] = ptr[v];
    for (int64_t e = 0; e < E; ++e) eid[fill[dst[e]]++] = e;
    free(fill);
}

/* one LSTM step for one vertex: z (4H) <- gates; returns activated gates in
 * gt (4H: i, f, g, o), updates c (H) and h (H) */
static void lstm_step(int H, const double* xt, const double* hprev, const double* Wih, const double* Whh,
                      const double* bl, double* gt, double* c, double* h) {
    for (int j = 0; j < 4 * H; ++j) gt[j] = bl ? bl[j] : 0.0;
    add_msg(H, 4 * H, 1.0, xt, Wih, gt);
    add_msg(H, 4 * H, 1.0, hprev, Whh, gt);
    for (int j = 0; j < H; ++j) {
        gt[j] = sigm(gt[j]);
        gt[H + j] = sigm(gt[H + j]);
        gt[2 * H + j] = tanh(gt[2 * H + j]);
        gt[3 * H + j] = sigm(gt[3 * H + j]);
        c[j] = gt[H + j] * c[j] + gt[j] * gt[2 * H + j];
        h[j] = gt[3 * H + j] * tanh(c[j]);
    }
}

/* row_mask: only those rows of y (and hN) are produced.  hN (nullable): [V x fi] */
void wgo_sage_lstm_forward(int64_t V, int64_t E, const int32_t* src, const int32_t* dst, int fi, int fo,
                           const double* x, const double* Ws, const double* Wn, const double* b, const double* Wih,
                           const double* Whh, const double* bl, const uint8_t* row_mask, double* y, double* hN) {
    const int H = fi;
    int64_t* ptr = (int64_t*)malloc(sizeof(int64_t) * (V + 1));
    int64_t* eid = (int64_t*)malloc(sizeof(int64_t) * (E > 0 ? E : 1));
    in_lists(V, E, dst, ptr, eid);
    double *c = malloc(sizeof(double) * H), *h = malloc(sizeof(double) * H), *gt = malloc(sizeof(double) * 4 * H);
    for (int64_t v = 0; v < V; ++v) {
        if (!ROW_ON(row_mask, v)) continue;
        for (int j = 0; j < H; ++j) { c[j] = 0.0; h[j] = 0.0; }
        for (int64_t p = ptr[v]; p < ptr[v + 1]; ++p)
            lstm_step(H, x + (int64_t)src[eid[p]] * fi, h, Wih, Whh, bl, gt, c, h);
        if (hN) for (int j = 0; j < H; ++j) hN[v * H + j] = h[j];
        for (int j = 0; j < fo; ++j) y[v * fo + j] = b ? b[j] : 0.0;
        add_msg(fi, fo, 1.0, x + v * fi, Ws, y + v * fo);
        add_msg(H, fo, 1.0, h, Wn, y + v * fo);
    }
    free(ptr); free(eid); free(c); free(h); free(gt);
}

/* Exact gradients (backpropagation through each vertex's sequence).
 * dy_rows (nullable): rows of dy outside the set are zero (skipped); every
 * output is then the exact gradient for that dy.  Outputs nullable. */
void wgo_sage_lstm_backward(int64_t V, int64_t E, const int32_t* src, const int32_t* dst, int fi, int fo,
                            const double* x, const double* Ws, const double* Wn, const double* Wih,
                            const double* Whh, const double* bl, const double* dy, const uint8_t* dy_rows,
                            double* dx, double* dWs, double* dWn, double* db, double* dWih, double* dWhh,
                            double* dbl) {
    const int H = fi;
    int64_t* ptr = (int64_t*)malloc(sizeof(int64_t) * (V + 1));
    int64_t* eid = (int64_t*)malloc(sizeof(int64_t) * (E > 0 ? E : 1));
    in_lists(V, E, dst, ptr, eid);
    int64_t maxd = 0;
    for (int64_t v = 0; v < V; ++v) if (ptr[v + 1] - ptr[v] > maxd) maxd = ptr[v + 1] - ptr[v];
    /* per step of one sequence: activated gates, c_t, h_t (index t+1; 0 = initial) */
    double* G = malloc(sizeof(double) * 4 * H * (maxd > 0 ? maxd : 1));
    double* Cs = malloc(sizeof(double) * H * (maxd + 1));
    double* Hs = malloc(sizeof(double) * H * (maxd + 1));
    double *dh = malloc(sizeof(double) * H), *dc = malloc(sizeof(double) * H), *dz = malloc(sizeof(double) * 4 * H);
    double* dhn = malloc(sizeof(double) * H);
    if (dx) memset(dx, 0, sizeof(double) * V * fi);
    if (dWs) memset(dWs, 0, sizeof(double) * fi * fo);
    if (dWn) memset(dWn, 0, sizeof(double) * H * fo);
    if (db) memset(db, 0, sizeof(double) * fo);
    if (dWih) memset(dWih, 0, sizeof(double) * fi * 4 * H);
    if (dWhh) memset(dWhh, 0, sizeof(double) * H * 4 * H);
    if (dbl) memset(dbl, 0, sizeof(double) * 4 * H);
    for (int64_t v = 0; v < V; ++v) {
        if (!ROW_ON(dy_rows, v)) continue;
        const double* dyv = dy + v * fo;
        const int64_t T = ptr[v + 1] - ptr[v];
        /* forward of the sequence, keeping every step */
        for (int j = 0; j < H; ++j) { Cs[j] = 0.0; Hs[j] = 0.0; }
        for (int64_t t = 0; t < T; ++t) {
            for (int j = 0; j < H; ++j) Cs[(t + 1) * H + j] = Cs[t * H + j];
            lstm_step(H, x + (int64_t)src[eid[ptr[v] + t]] * fi, Hs + t * H, Wih, Whh, bl, G + t * 4 * H,
                      Cs + (t + 1) * H, Hs + (t + 1) * H);
        }
        /* y = b + x[v] W_s + h_N W_n */
        if (db) for (int j = 0; j < fo; ++j) db[j] += dyv[j];
        add_msg_grad(fi, fo, 1.0, x + v * fi, Ws, dyv, dx ? dx + v * fi : NULL, dWs);
        for (int j = 0; j < H; ++j) dhn[j] = 0.0;
        add_msg_grad(H, fo, 1.0, Hs + T * H, Wn, dyv, dhn, dWn);
        /* backpropagation through time */
        for (int j = 0; j < H; ++j) { dh[j] = dhn[j]; dc[j] = 0.0; }
        for (int64_t t = T - 1; t >= 0; --t) {
            const double* gt = G + t * 4 * H;
            for (int j = 0; j < H; ++j) {
                const double i = gt[j], f = gt[H + j], g = gt[2 * H + j], o = gt[3 * H + j];
                const double tc = tanh(Cs[(t + 1) * H + j]);
                const double dO = dh[j] * tc;
                const double dC = dc[j] + dh[j] * o * (1.0 - tc * tc);
                dz[j] = dC * g * i * (1.0 - i);
                dz[H + j] = dC * Cs[t * H + j] * f * (1.0 - f);
                dz[2 * H + j] = dC * i * (1.0 - g * g);
                dz[3 * H + j] = dO * o * (1.0 - o);
                dc[j] = dC * f;
            }
            if (dbl) for (int j = 0; j < 4 * H; ++j) dbl[j] += dz[j];
            const int64_t s = src[eid[ptr[v] + t]];
            add_msg_grad(fi, 4 * H, 1.0, x + s * fi, Wih, dz, dx ? dx + s * fi : NULL, dWih);
            for (int j = 0; j < H; ++j) dh[j] = 0.0;
            add_msg_grad(H, 4 * H, 1.0, Hs + t * H, Whh, dz, dh, dWhh);
        }
    }
    free(ptr); free(eid); free(G); free(Cs); free(Hs); free(dh); free(dc); free(dz); free(dhn);
}
