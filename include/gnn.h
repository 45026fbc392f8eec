/*
 * gnn.h — C-ABI of the B200 (sm_100a) GNN neighbor-aggregation library.
 *
 * The operations are those of Huang et al., "Understanding and Bridging the
 * Gaps in Current GNN Performance Optimizations", PPoPP'21 (cited as P:<line>
 * of /root/reference/PAPER.md).  Readings of silent or garbled passages are
 * R1..R14 in DESIGN.md §2.
 *
 * Conventions (all entry points):
 *  - Graph: CSR by destination (Fig 2): row v lists the sources u
 *    of edges u -> v.  Host arrays: rowptr int64[n+1] with
 *    rowptr[0] = 0, non-decreasing, rowptr[n] = nnz < 2^31; colidx int32[nnz]
 *    with 0 <= colidx < n_src.  Multi-edges count separately; self loops only
 *    if present (R1).
 *  - Features: row-major fp32 with row stride ld (elements), ld >= width.
 *    Pointers named *_h are HOST pointers; every other array pointer is a
 *    DEVICE pointer on the device that was current when the plan was made.
 *  - Ownership: the caller allocates and owns every feature/weight/output/
 *    workspace buffer (torch tensors in practice).  The plan owns copies of the
 *    graph and its schedule on host and device and frees them in
 *    gnn_plan_destroy (caller guarantees no call is in flight, like cudaFree).
 *  - Streams: compute calls only enqueue work on `stream` (NULL = legacy
 *    default stream); they never synchronise or allocate and can be captured
 *    into CUDA graphs.  gnn_plan_create / gnn_plan_export* are synchronous.
 *  - Errors: every entry point returns gnn_status; nothing aborts, nothing
 *    throws across the ABI.  gnn_last_error() returns a thread-local message
 *    for the last failing call.  Device faults surface at the caller's next
 *    synchronisation.
 *  - Y is fully overwritten; rows with no in-edges get 0 for every reducer (R3).
 *  - Thread-safety: a plan is immutable after creation; concurrent calls on
 *    different streams are safe if each has its own workspace.
 */
#ifndef GNN_H
#define GNN_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  GNN_OK = 0,
  GNN_ERR_INVALID_ARG = 1,   /* null pointer, bad size/stride, aliasing */
  GNN_ERR_INVALID_GRAPH = 2, /* CSR validation failed */
  GNN_ERR_WORKSPACE = 3,     /* workspace smaller than gnn_workspace_size() */
  GNN_ERR_CUDA = 4,          /* CUDA runtime error (message has cudaGetErrorString) */
  GNN_ERR_NOMEM = 5,         /* host or device allocation failed */
  GNN_ERR_UNSUPPORTED = 6,   /* valid request this build does not implement */
  GNN_ERR_INTERNAL = 7
} gnn_status;

typedef struct gnn_plan_s *gnn_plan_t;
typedef struct CUstream_st *gnn_stream_t; /* identical to cudaStream_t */

/* Reducers: Table 1 sum / mean / pooling-max. */
typedef enum { GNN_SUM = 0, GNN_MEAN = 1, GNN_MAX = 2 } gnn_reduce;
/* Edge weights: Table 2 Const, GCN 1/sqrt(d_u d_v) with
 * d_u = out-degree of u, d_v = in-degree of v (R1), or an explicit per-CSR-entry
 * array. */
typedef enum { GNN_W_ONE = 0, GNN_W_GCN = 1, GNN_W_EDGE = 2 } gnn_weight;

/*
 * Plan options.  Locality-aware task scheduling (LAS) and
 * neighbor grouping (NG).
 */
typedef struct {
  uint32_t struct_size;  /* sizeof(gnn_plan_opts), for ABI versioning */
  int32_t reorder;       /* 0 = identity task order, 1 = LAS (MinHash+LSH+merge) */
  int32_t group_size;    /* NG upper bound ng; -1 = auto (R8-ii); 0 = never split */
  int32_t tile_groups;   /* reserved (validated to [0, 256], otherwise unused): every neighbor
                            group is one work unit claimed in task order (R8) */
  int32_t cluster_cap;   /* LAS cluster size cap (32) */
  int32_t minhash_k;     /* K signature length (32) */
  int32_t lsh_rows;      /* r rows per band (2); b = K / r bands */
  int32_t pair_window;   /* W: candidate pairs (m_i, m_{i+d}), 1 <= d <= W (8) */
  int32_t min_sim;       /* re-enqueue threshold; -1 -> lsh_rows */
  int32_t deterministic; /* 1: fixed-order combine (R9); 0: float atomics */
  int32_t cluster_order; /* LAS schedule: 1 = clusters by representative signature, 0 = by smallest member */
  uint64_t seed;         /* MinHash salt stream seed */
} gnn_plan_opts;

/* Fill defaults: reorder 0, group_size -1, tile_groups 32, cluster_cap 32,
 * minhash_k 32, lsh_rows 2, pair_window 8, min_sim -1, deterministic 1,
 * cluster_order 1, seed 0. */
void gnn_plan_opts_default(gnn_plan_opts *opts);

typedef struct {
  int64_t n;            /* destination rows */
  int64_t n_src;        /* source rows (== n for gnn_plan_create) */
  int64_t nnz;
  int64_t n_groups;     /* G = sum ceil(d_v / ng) */
  int64_t n_tiles;      /* work units = neighbor groups (one unit per group, claimed in task order) */
  int64_t n_split_rows; /* rows with more than one group (combined through the workspace, a9) */
  int64_t n_empty_rows;
  int64_t n_clusters;   /* LAS clusters (n if reorder == 0) */
  int64_t n_pairs;      /* LSH candidate pairs (0 if reorder == 0) */
  int32_t group_size;   /* ng actually used */
  int32_t tile_groups;
  int32_t max_degree;
  int32_t reorder;
  double ms_validate, ms_upload, ms_degrees, ms_minhash, ms_lsh, ms_merge, ms_ng;
} gnn_plan_info;

/*
 * Build a plan (a1 CSR ingest + degrees, a2 LAS if opts->reorder, a3 NG work
 * units in task order).  Synchronous; copies the host CSR.  Validates in O(n + nnz):
 * on failure returns GNN_ERR_INVALID_GRAPH and sets *out = NULL.
 * opts may be NULL (defaults).
 */
gnn_status gnn_plan_create(int64_t n, int64_t nnz, const int64_t *rowptr_h,
                           const int32_t *colidx_h, const gnn_plan_opts *opts,
                           gnn_plan_t *out);

/*
 * Rectangular variant: n destination rows, sources indexed in [0, n_src).
 * src_degree_h (nullable, int32[n_src]) overrides the source out-degrees used
 * by GNN_W_GCN (multi-GPU local plans pass the GLOBAL out-degrees in the padded
 * all-gather layout); NULL = count colidx.
 */
gnn_status gnn_plan_create_ex(int64_t n, int64_t n_src, int64_t nnz,
                              const int64_t *rowptr_h, const int32_t *colidx_h,
                              const int32_t *src_degree_h,
                              const gnn_plan_opts *opts, gnn_plan_t *out);

/*
 * As gnn_plan_create_ex with the task order given instead of computed:
 * perm_h int32[n] must be a permutation of [0, n) (else GNN_ERR_INVALID_ARG);
 * opts->reorder is recorded but LAS does not run.  For schedules computed
 * offline and reused.
 */
gnn_status gnn_plan_create_perm(int64_t n, int64_t n_src, int64_t nnz,
                                const int64_t *rowptr_h, const int32_t *colidx_h,
                                const int32_t *src_degree_h, const int32_t *perm_h,
                                const gnn_plan_opts *opts, gnn_plan_t *out);

/*
 * Plan persistence (LAS runs once offline and is reused).
 * gnn_plan_save writes the CSR, the source out-degrees, the options and the
 * task order to `path` (with_las != 0 also writes the LAS intermediates
 * exported by gnn_plan_export_las); a checksum covers the file.
 * gnn_plan_load rebuilds the device plan on the current device from such a
 * file without rerunning LAS: the task order, the normalisers and every
 * result computed with the loaded plan are identical to the saved plan's.
 * Errors: GNN_ERR_INVALID_ARG for an unreadable, truncated, corrupt or foreign
 * file (*out = NULL); GNN_ERR_INTERNAL if writing fails.  Synchronous.
 */
gnn_status gnn_plan_save(gnn_plan_t plan, const char *path, int32_t with_las);
gnn_status gnn_plan_load(const char *path, gnn_plan_t *out);

gnn_status gnn_plan_get_info(gnn_plan_t plan, gnn_plan_info *info);

/*
 * Copy the schedule to host buffers sized from gnn_plan_info (any may be NULL):
 * perm_h int32[n] (task order), grp_row_h int32[G], grp_beg_h int64[G] (first
 * CSR entry of each group).  Bit-exact with the oracle's orc_las_merge /
 * orc_neighbor_groups.
 */
gnn_status gnn_plan_export(gnn_plan_t plan, int32_t *perm_h, int32_t *grp_row_h,
                           int64_t *grp_beg_h);

/*
 * LAS intermediates (reorder == 1 only): sig_h uint64[n * minhash_k] (GPU
 * MinHash), pairs_h int32[2 * n_pairs] (sorted (a, b), a < b),
 * cluster_of_h int32[n] (representative of each node).  Any may be NULL.
 */
gnn_status gnn_plan_export_las(gnn_plan_t plan, uint64_t *sig_h, int32_t *pairs_h,
                               int32_t *cluster_of_h);

/* Device arrays of the plan's per-node normalisers (read-only, owned by the
 * plan): nsrc = 1/sqrtf(d_out) [n_src], ndst = 1/sqrtf(d_in) [n] (0 if degree 0). */
gnn_status gnn_plan_normalizers(gnn_plan_t plan, const float **nsrc, const float **ndst);

gnn_status gnn_plan_destroy(gnn_plan_t plan);

/* Workspace operations */
typedef enum {
  GNN_OP_AGGREGATE = 0,     /* f_out = F */
  GNN_OP_GAT_AGGREGATE = 1, /* f_out = H * Fh, heads = H */
  GNN_OP_EDGECONV = 2,      /* f_in, f_out */
  GNN_OP_GCN_LAYER = 3,     /* f_in, f_out */
  GNN_OP_GAT_LAYER = 4,     /* f_in, f_out = H * Fh, heads = H */
  GNN_OP_SAGE_LSTM_LAYER = 5, /* f_in, f_out = F_out, heads = T (hidden F = 32) */
  GNN_OP_ATTN_AGGREGATE = 6,  /* f_out = H * Fh, heads = H */
  GNN_OP_ATTN_AGGREGATE_MEAN = 7 /* as 6, with head_mean (adds an n x H*Fh buffer) */
} gnn_op;

/* Bytes of device workspace a call needs (may be 0; pass NULL then).  The
 * workspace must be 256-byte aligned.  Unused size arguments are ignored. */
size_t gnn_workspace_size(gnn_plan_t plan, int op, int32_t f_in, int32_t f_out, int32_t heads);

/*
 * a6 + a9: graph operation y_v = REDUCE_{u->v} e_uv * x_u (Table 1 x Table 2,
 * Eq 1 inner part P:217), evaluated over the plan's neighbor groups in task
 * order: persistent workers claim work units (one neighbor group each) in task
 * order; a single-group row is finished by its worker; the group partials of a
 * longer row are combined in fixed group order (R9) in the workspace by the
 * last group to finish, or with atomics (deterministic == 0, sum/mean only).
 * Epilogue (linear property):
 * GCN x ndst[v], mean / D_v, then + add_row[v] (nullable, EdgeConv's Q), then
 * ReLU if relu != 0.
 *   edge_w: [nnz] in CSR order, required iff weight == GNN_W_EDGE.
 *   X: [n_src, ldx] with F <= ldx; Y: [n, ldy]; X and Y must not overlap.
 *   add_row: [n, ld_add] or NULL.
 * F == 0 is a no-op.
 * Kernels (results bit-identical across them): rows of >= 64
 * features stream through a per-warp shared-memory ring (cp.async), narrower
 * rows use the register kernel.  When the source rows exceed L2 (n_src * row
 * bytes > 128 MB), the plan's highest out-degree sources (up to 32 MB of rows,
 * the list built on the first such call) are marked evict_last in L2 for the
 * duration of the call and returned to evict_normal after it (cache hints
 * only; env GNN_L2_PIN=0 disables).  Every aggregation entry point below
 * (gnn_gat_aggregate, gnn_attn_aggregate, gnn_gcn_aggregate_prescaled,
 * gnn_aggregate_accumulate, gnn_edgeconv_aggregate) behaves the same way.
 */
gnn_status gnn_aggregate(gnn_plan_t plan, int reduce, int weight, const float *edge_w,
                         const float *X, int64_t ldx, int32_t F, float *Y, int64_t ldy,
                         int32_t relu, const float *add_row, int64_t ld_add,
                         void *ws, size_t ws_bytes, gnn_stream_t stream);

/*
 * Source-block accumulation (NEXT-2 groundwork, SURVEY §8(e) lever ii): with a
 * plan over the same destination rows but only the entries whose sources lie
 * in one block (e.g. one rank's slot of the all-gather), y_v = (accumulate ?
 * y_v : 0) + SUM_{u->v in the plan} e_uv * x_u -- raw sums, no epilogue;
 * rows the plan leaves empty keep y_v (accumulate) or get 0.  weight: ONE or
 * EDGE (pre-scale the sources for GCN and finish with gnn_scale_rows).
 * Deterministic: each call is the fixed chain of R9 over the block's groups,
 * and blocks are added in the caller's order.
 * gnn_scale_rows: y_v = ReLU?(y_v * scale[v]) on n rows x F (device scale[n]).
 */
gnn_status gnn_aggregate_accumulate(gnn_plan_t plan, int weight, const float *edge_w, const float *X,
                                    int64_t ldx, int32_t F, float *Y, int64_t ldy, int32_t accumulate,
                                    void *ws, size_t ws_bytes, gnn_stream_t stream);
gnn_status gnn_scale_rows(float *Y, int64_t ldy, int64_t n, int32_t F, const float *scale, int32_t relu,
                          gnn_stream_t stream);

/*
 * a7: fused GAT graph operation (Eq 2; Listing 1 P:622-646 fused, DVRA
 * P:943-968, division postponed by the linear property).  Per head h:
 * e_uv = LeakyReLU(s_u[h] + t_v[h], neg_slope), alpha = softmax_v(e),
 * y_v[h] = SUM_u alpha_uv z_u[h].  Edge scores never reach HBM.
 *   Zs: [n_src, ldz] rows = [z_u (H*Fh floats) | s_u (H floats)], ldz >= H*Fh+H.
 *   t:  [n, ldt] (t_v per head).  Y: [n, ldy], ldy >= H*Fh.  1 <= H <= 256.
 * The softmax is shifted by the per-row bound LeakyReLU(max_u s_u[h] + t_v[h])
 * (one extra pass over the n_src x H score columns; R9).  Inputs
 * must be finite; rows of Zs that no CSR entry references still enter that
 * maximum, so padding rows should hold finite values (zeros).
 */
gnn_status gnn_gat_aggregate(gnn_plan_t plan, const float *Zs, int64_t ldz,
                             const float *t, int64_t ldt, int32_t H, int32_t Fh,
                             float neg_slope, float *Y, int64_t ldy,
                             void *ws, size_t ws_bytes, gnn_stream_t stream);

/*
 * GAT transform (a5 for Table 2's GAT; reading R5): Zst rows =
 * [z_v | s_v | t_v] with z = X W (W: [f_in, ldw >= H*Fh] row-major), s_v[h] =
 * <z_v[h], a_src_h>, t_v[h] = <z_v[h], a_dst_h>.  Heads of a multiple of 32
 * features: one tcgen05 3xTF32 GEMM of H*Fh columns whose epilogue
 * accumulates s and t from the stored z (fp32, head order); other head sizes
 * fold the scores into extra GEMM columns X (W_h a_h) (needs ldw == H*Fh and
 * ldz >= round_up(H*Fh + 2H, 8)).  X: [m, ldx]; Zst: [m, ldz], ldz >= H*Fh + 2H.
 * Workspace: gnn_gat_transform_workspace_size(m, f_in, H, Fh) bytes, 256-byte
 * aligned.
 */
gnn_status gnn_gat_transform(const float *X, int64_t ldx, int64_t m, int32_t f_in, const float *W,
                             int64_t ldw, const float *a_src, const float *a_dst, int32_t H,
                             int32_t Fh, float *Zst, int64_t ldz, void *ws, size_t ws_bytes,
                             gnn_stream_t stream);
size_t gnn_gat_transform_workspace_size(int64_t m, int32_t f_in, int32_t H, int32_t Fh);

/* gnn_gat_transform whose epilogue also writes [z | s | t] to n_mirrors peer
 * replicas (NEXT-2; mirror contract as gnn_gemm_mirrored, laid out like Zst). */
gnn_status gnn_gat_transform_mirrored(const float *X, int64_t ldx, int64_t m, int32_t f_in,
                                      const float *W, int64_t ldw, const float *a_src,
                                      const float *a_dst, int32_t H, int32_t Fh, float *Zst,
                                      int64_t ldz, float *const *mirrors, int32_t n_mirrors,
                                      void *ws, size_t ws_bytes, gnn_stream_t stream);

/*
 * Full GAT layer: [Z | s | t] by gnn_gat_transform, then gnn_gat_aggregate.
 * W: [f_in, H*Fh] row-major.  Requires n_src == n.  Workspace from
 * gnn_workspace_size(plan, GNN_OP_GAT_LAYER, f_in, H * Fh, H).
 */
gnn_status gnn_gat_layer(gnn_plan_t plan, const float *X, int64_t ldx, int32_t f_in,
                         const float *W, const float *a_src, const float *a_dst,
                         int32_t H, int32_t Fh, float neg_slope, float *Y, int64_t ldy,
                         void *ws, size_t ws_bytes, gnn_stream_t stream);

/*
 * a8: EdgeConv max aggregation given the pre-transformed [P | Q] rows
 * (redundancy bypass P:1014-1021, reading R6): y_v = ReLU(Q_v + MAX_u P_u),
 * empty row -> 0.  PQ: [n, ldpq], P = columns [0, f_out), Q = [f_out, 2 f_out).
 */
gnn_status gnn_edgeconv_aggregate(gnn_plan_t plan, const float *PQ, int64_t ldpq,
                                  int32_t f_out, float *Y, int64_t ldy,
                                  void *ws, size_t ws_bytes, gnn_stream_t stream);

/*
 * Full EdgeConv layer y_v = MAX_u ReLU(Theta(x_u - x_v) + Phi x_v + b):
 * [P | Q] = X [Theta^T | (Phi - Theta)^T] (+ b on Q) by gnn_gemm, then
 * gnn_edgeconv_aggregate.  theta, phi: [f_out, f_in] row-major; bias nullable.
 */
gnn_status gnn_edgeconv(gnn_plan_t plan, const float *X, int64_t ldx, int32_t f_in,
                        const float *theta, const float *phi, const float *bias,
                        int32_t f_out, float *Y, int64_t ldy, void *ws, size_t ws_bytes,
                        gnn_stream_t stream);

/*
 * a5: dense transform H = X W (Eq 1 "(x) W") in fp32 accuracy,
 * X: [m, ldx] (k used), W: [k, ldw] (n used), H: [m, ldh].
 * Epilogue: row_scale (nullable, [m]) multiplies row i; col_bias (nullable, [n])
 * is added after the scale; relu != 0 clamps.  H must not overlap X or W.
 * With ws != NULL the tcgen05 3xTF32 tensor-core kernel runs for every shape
 * (the workspace holds the split, pre-swizzled W image; outputs wider than one
 * launch takes -- n > 320 with k > 256, or n > 512 -- run as ceil(n/256)
 * launches over equal column slices); ws must be 16-byte aligned and hold
 * gnn_gemm_workspace_size(m, k, n) bytes, else GNN_ERR_INVALID_ARG /
 * GNN_ERR_WORKSPACE (never a silent fallback).  With ws == NULL the SIMT fp32
 * FFMA kernel runs.
 */
gnn_status gnn_gemm(const float *X, int64_t ldx, const float *W, int64_t ldw, float *H,
                    int64_t ldh, int64_t m, int32_t k, int32_t n, const float *row_scale,
                    const float *col_bias, int32_t relu, void *ws, size_t ws_bytes,
                    gnn_stream_t stream);
size_t gnn_gemm_workspace_size(int64_t m, int32_t k, int32_t n);

/*
 * NEXT-2 (SURVEY §8(e) lever iii, §8(f)): the all-gather of a row-partitioned
 * layer fused into the producer.  gnn_gemm whose epilogue also writes every
 * output tile to n_mirrors (<= 7) extra destinations -- the same rows of the
 * peer GPUs' replica buffers, opened with gnn_ipc_open -- with the same TMA
 * bulk-tensor stores that write H, so the rows leave over NVLink as soon as
 * each tile is done instead of in a separate collective.  mirrors[q]: device
 * pointer (local or peer), 16-byte aligned, laid out like H (ldh, m rows, n
 * columns), not overlapping X or H.  Needs the tcgen05 path (ws from
 * gnn_gemm_workspace_size) with 16-byte aligned X/H rows, else
 * GNN_ERR_UNSUPPORTED (never a silent non-mirrored run).  The kernel's stores
 * are complete (and fenced at system scope) when it ends; consumers on other
 * GPUs must order after it (e.g. a stream-ordered NCCL all_reduce of a flag).
 */
gnn_status gnn_gemm_mirrored(const float *X, int64_t ldx, const float *W, int64_t ldw, float *H,
                             int64_t ldh, int64_t m, int32_t k, int32_t n, const float *row_scale,
                             const float *col_bias, int32_t relu, float *const *mirrors,
                             int32_t n_mirrors, void *ws, size_t ws_bytes, gnn_stream_t stream);

/*
 * Device memory shareable across processes (CUDA IPC) for the mirrors:
 * gnn_ipc_alloc returns a fresh cudaMalloc allocation and its 64-byte IPC
 * handle (written to `handle`); another process on this or a peer GPU maps
 * it with gnn_ipc_open (peer access enabled lazily) and unmaps it with
 * gnn_ipc_close; the owner releases it with gnn_ipc_free.
 */
gnn_status gnn_ipc_alloc(size_t bytes, void **ptr, void *handle);
gnn_status gnn_ipc_free(void *ptr);
gnn_status gnn_ipc_open(const void *handle, void **ptr);
gnn_status gnn_ipc_close(void *ptr);

/* GEMM implementation selector (process-wide): 0 = auto, 1 = SIMT FFMA,
 * 2 = tcgen05 3xTF32, 3 = tcgen05 3xTF32 with register-fed X tiles instead
 * of TMA (same results bit for bit; kept for A/B measurement).  Under 0 and
 * 2 the X tiles arrive by TMA (cp.async.bulk.tensor, SWIZZLE_128B) whenever
 * X and ldx are 16-byte aligned.  Returns the previous value. */
int gnn_set_gemm_impl(int impl);


/*
 * a4 mapping override (process-wide; the hook of the paper's mapping tuner,
 * P:1128-1168): every later graph op whose F, strides and pointers
 * admit it uses vec floats per lane-vector (1, 2, 4 or 8), `lanes` lanes per
 * worker (4, 8, 16 or 32) and nv vectors per lane (1, 2 or 4; nv > 1 needs
 * lanes == 32 (vec 8: nv <= 2), or lanes*nv == 32 with lanes 16 (vec >= 2) or
 * lanes 8 (vec >= 4)).  The feature chunk lanes*vec*nv bounds
 * the width of H one sweep over the schedule gathers (wider rows take several
 * sweeps).  An op whose shapes do not admit the override uses the automatic
 * rule.  vec = lanes = nv = 0 restores the automatic rule.
 * Returns GNN_ERR_INVALID_ARG for an unsupported combination.  Results are
 * unchanged bit for bit in the deterministic variant (the chain of R9 is per
 * feature and does not depend on the mapping).
 */
gnn_status gnn_set_agg_mapping(int32_t vec, int32_t lanes, int32_t nv);

/*
 * Load-balance trace of the aggregation kernels (the "Balanced vs Actual"
 * measurement of Fig 8; process-wide, NULL = off).  When set,
 * every later graph-op launch resets trace_dev (device, 8 x uint64) and its
 * persistent workers record: [0] the sum over workers of the time spent in
 * their work units (ns, %globaltimer), [1] the number of workers, [2] the
 * earliest worker start, [3] the latest worker end, [4] work units, [5] the
 * longest single-worker busy time.  Balanced time = [0] / [1] (all workers
 * are resident at once: perfect balance); actual = [3] - [2].  Costs two
 * timer reads per unit; for measurement only.  The caller keeps the buffer
 * alive while set.
 */
void gnn_set_agg_trace(void *trace_dev);

/*
 * NG bound of an existing plan (reading R8): rebuilds the work
 * units and the task-ordered index stream for group_size (> 0: groups of at
 * most group_size entries; 0: never split rows; -1: the default rule); the
 * LAS schedule is kept.  Synchronous (host rebuild + upload); the caller
 * guarantees that no call using the plan is in flight.  Deterministic results
 * depend on (CSR, group size, F) only (R9), so they change with the bound.
 * Workspace sizes change too: query gnn_workspace_size again.
 */
gnn_status gnn_plan_set_group_size(gnn_plan_t plan, int32_t group_size);

/* Result of gnn_tune_aggregate. */
typedef struct {
  int32_t group_size;     /* chosen NG bound (left in the plan) */
  int32_t vec, lanes, nv; /* chosen a4 mapping (0,0,0 = the automatic rule) */
  float ms;               /* median time of one gnn_aggregate call with both */
  float ms_default;       /* the same at entry (automatic mapping, entry bound) */
  int32_t rounds;         /* NG rounds run (one bound per round) */
  int32_t mappings_tried; /* mapping templates timed */
} gnn_tune_result;

/*
 * NEXT-1 online tuner: phase 1 times the a4 mapping templates
 * (vector width x lanes per worker x vectors per lane, at most two feature
 * chunks) at the plan's current bound ("first exhaust GPU resources by
 * scheduling more warps"); phase 2 tries NG bounds, one per
 * round, multiples of 16 up to ten times the average degree (and the max
 * degree), a doubling ladder then bisection around the best, at most
 * max_rounds rounds (<= 0: 20).  Each candidate = 1 warm-up +
 * median of 3 gnn_aggregate calls timed with CUDA events on `stream`.  The
 * plan keeps the best bound and uses the chosen mapping for later calls of
 * width F (a process-wide gnn_set_agg_mapping override takes precedence;
 * tuning with one active returns GNN_ERR_INVALID_ARG).  Arguments as
 * gnn_aggregate (relu off; Y is overwritten).  Synchronous; allocates its own
 * workspace; not graph-capturable.
 */
gnn_status gnn_tune_aggregate(gnn_plan_t plan, int reduce, int weight, const float *edge_w,
                              const float *X, int64_t ldx, int32_t F, float *Y, int64_t ldy,
                              int32_t max_rounds, gnn_tune_result *out, gnn_stream_t stream);

/*
 * GCN layer (Eq 1): Y = ACT((A_gcn X) W).  order: 0 = auto (aggregate at
 * min(f_in, f_out)), 1 = transform first (H = X W scaled by nsrc, aggregate,
 * x ndst), 2 = aggregate first.  Workspace: gnn_workspace_size(plan,
 * GNN_OP_GCN_LAYER, f_in, f_out, 0).  X has n_src rows; Y has n rows.
 */
gnn_status gnn_gcn_layer(gnn_plan_t plan, const float *X, int64_t ldx, int32_t f_in,
                         const float *W, int64_t ldw, int32_t f_out, int32_t relu,
                         int32_t order, float *Y, int64_t ldy, void *ws, size_t ws_bytes,
                         gnn_stream_t stream);

/*
 * Second half of a transform-first GCN layer (Eq 1 reassociated, R4-i; linear
 * property): y_v = ACT(ndst[v] * SUM_{u->v} Hs[u]) where the caller's
 * Hs rows are already scaled by nsrc[u] (gnn_gemm row_scale = the plan's nsrc
 * from gnn_plan_normalizers).  Hs: [n_src, ldh]; Y: [n, ldy].
 */
gnn_status gnn_gcn_aggregate_prescaled(gnn_plan_t plan, const float *Hs, int64_t ldh, int32_t F,
                                       float *Y, int64_t ldy, int32_t relu, void *ws,
                                       size_t ws_bytes, gnn_stream_t stream);

/*
 * GAT parameter fold (device, O(f_in * H * Fh)): Wext[:, 0:H*Fh] = W,
 * Wext[:, H*Fh + h] = W_h . a_src_h, Wext[:, H*Fh + H + h] = W_h . a_dst_h, so
 * X Wext = [Z | s | t] (Table 2 GAT scores as extra GEMM columns).
 * W: [f_in, H*Fh] row-major; Wext: [f_in, ldwe], ldwe >= H*Fh + 2H.
 */
gnn_status gnn_gat_fold_weights(const float *W, const float *a_src, const float *a_dst,
                                int32_t f_in, int32_t H, int32_t Fh, float *Wext, int64_t ldwe,
                                gnn_stream_t stream);

/*
 * a10: multi-GPU destination-row partition (host only, reading R10):
 * bounds[p] = smallest i with rowptr[i] >= ceil(p * nnz / P), bounds[0] = 0,
 * bounds[P] = n.  bounds_h: int64[nparts + 1].
 */
gnn_status gnn_partition_rows(int64_t n, const int64_t *rowptr_h, int32_t nparts,
                              int64_t *bounds_h);

/*
 * Local CSR of rank `rank` (host only): rows [bounds[rank], bounds[rank+1]),
 * every source u translated to the padded all-gather layout
 * owner(u) * r_max + (u - bounds[owner(u)]), r_max = max part size.
 * Outputs (caller-allocated, sizes from a NULL-output query):
 *   *r_max, *local_nnz; local_rowptr_h int64[rows+1]; local_colidx_h
 *   int32[local_nnz]; src_degree_h int32[nparts * r_max] = global out-degree of
 *   each padded source slot (0 for pad slots).
 */
gnn_status gnn_local_csr(int64_t n, const int64_t *rowptr_h, const int32_t *colidx_h,
                         const int64_t *bounds_h, int32_t nparts, int32_t rank,
                         int64_t *r_max, int64_t *local_nnz, int64_t *local_rowptr_h,
                         int32_t *local_colidx_h, int32_t *src_degree_h);

/*
 * Source block q of rank `rank`'s rows (host only; NEXT-2 source-block
 * pipelining): the CSR of rows [bounds[rank], bounds[rank+1]) restricted to
 * the entries whose source u lies in [bounds[q], bounds[q+1]), with u stored
 * relative to the block (u - bounds[q]); entry order within a row is kept.
 * Size query with NULL outputs: *block_nnz.  block_rowptr_h int64[rows+1],
 * block_colidx_h int32[block_nnz].
 */
gnn_status gnn_local_csr_block(int64_t n, const int64_t *rowptr_h, const int32_t *colidx_h,
                               const int64_t *bounds_h, int32_t nparts, int32_t rank, int32_t q,
                               int64_t *block_nnz, int64_t *block_rowptr_h, int32_t *block_colidx_h);

/*
 * Host-only planner steps (no GPU needed).  gnn_plan_create runs exactly these
 * after the GPU MinHash; they are exported so the host logic can be checked
 * against the oracle without a device.
 *
 * gnn_las_host: a2 steps 2-5 (LSH banding P:819-825, pair merging P:827-844,
 *   task scheduling P:846-853; reading R7) from MinHash signatures sig_h
 *   uint64[n * K].  Outputs perm_h int32[n], cluster_of_h int32[n] (nullable),
 *   *n_pairs, *n_clusters.
 * gnn_groups_host: a3 neighbor groups in task order (reading R8).
 *   ng <= 0 = one group per row.  Call with NULL arrays first to get
 *   *n_groups; then grp_row_h int32[G], grp_beg_h int64[G].
 */
gnn_status gnn_las_host(int64_t n, const int64_t *rowptr_h, const uint64_t *sig_h, int32_t K,
                        int32_t r, int32_t W, int32_t cap, int32_t min_sim, int32_t cluster_order,
                        int32_t *perm_h,
                        int32_t *cluster_of_h, int64_t *n_pairs, int64_t *n_clusters);
gnn_status gnn_groups_host(int64_t n, const int64_t *rowptr_h, const int32_t *perm_h, int32_t ng,
                           int64_t *n_groups, int32_t *grp_row_h, int64_t *grp_beg_h);

/*
 * NEXT-3 GraphSAGE-LSTM (Fig 6; setting P:1366-1367: 32 in /
 * 32 out, 16 sampled neighbours; reading R13).
 *
 * gnn_sample_neighbors: table[v*T + t] (device, [n, T] int32) = the t-th
 * neighbour of row v drawn uniformly with replacement by the counter-based
 * rule colidx[rowptr[v] + fmix64(seed + (v*T + t + 1) * 0x9E3779B97F4A7C15)
 * mod d_v]; -1 for every sample of an empty row.  1 <= T <= 32.
 */
gnn_status gnn_sample_neighbors(gnn_plan_t plan, int32_t T, uint64_t seed, int32_t *table,
                                gnn_stream_t stream);

/*
 * Fused LSTM aggregation with sparse fetching + SAGE combine:
 * h_T(v) = LSTM over the rows GS[u_1..u_T] of v's sampled neighbours (h_0 =
 * c_0 = 0; cell of Fig 6: i, f, o sigmoid, z tanh, c = f c + i z,
 * h = o tanh(c)); y_v = GS[v][4F : 4F+F_out] + W_neigh h_T(v).
 * GS: [n_src, ldg] device rows = the pre-transformed features (redundancy
 * bypass): GS[u][4j+g] = gate g (i, f, z, o) of hidden unit j of
 * x_u W_ih^T + b_ih + b_hh, and GS[u][4F+o] = (x_u W_self^T + b)[o].
 * R = W_hh [4F, F] (gate blocks i, f, z, o, PyTorch layout), W_neigh
 * [F_out, F].  F (hidden) must be 32 (else GNN_ERR_UNSUPPORTED), 1 <= F_out
 * <= 32, 1 <= T <= 32; GS 16-byte aligned, ldg a multiple of 4.
 * Empty rows: h_T = 0.  Y: [n, ldy].
 */
gnn_status gnn_sage_lstm_aggregate(gnn_plan_t plan, const int32_t *table, int32_t T,
                                   const float *GS, int64_t ldg, int32_t F, const float *R,
                                   const float *W_neigh, int32_t F_out, float *Y, int64_t ldy,
                                   gnn_stream_t stream);

/*
 * One GraphSAGE-LSTM layer: y_v = W_self x_v + W_neigh LSTM(x_{u_1..u_T}) + b,
 * computed as [W_ih | W_self] folded into one tensor-core GEMM (3xTF32) over
 * the nodes (GS, above), gnn_sample_neighbors(seed), then the fused cell
 * kernel.  W_ih [4F, f_in], W_hh [4F, F], b_ih/b_hh [4F], W_self [F_out,
 * f_in], W_neigh [F_out, F], bias [F_out] (nullable).  Workspace:
 * gnn_workspace_size(plan, GNN_OP_SAGE_LSTM_LAYER, f_in, F_out, T).
 */
gnn_status gnn_sage_lstm_layer(gnn_plan_t plan, const float *X, int64_t ldx, int32_t f_in,
                               const float *W_ih, const float *W_hh, const float *b_ih,
                               const float *b_hh, const float *W_self, const float *W_neigh,
                               const float *bias, int32_t F, int32_t F_out, int32_t T, uint64_t seed,
                               float *Y, int64_t ldy, void *ws, size_t ws_bytes, gnn_stream_t stream);

/*
 * NEXT-4: the edge functions of Table 2 feeding Table 1's
 * Softmax_aggr, fused like GAT (scores never reach HBM; reading
 * R14).  Per edge u->v and head h (Fh features per head, F = H*Fh):
 *   GNN_SCORE_GAT      e = LeakyReLU(s_u + t_v)            Zs = [z | s], Tv = t [n, H]
 *   GNN_SCORE_SYM_GAT  e = LeakyReLU(s_u + t_v) + LeakyReLU(s_v + t_u)   Zs = [z | s | t]
 *   GNN_SCORE_LINEAR   e = tanh(s_u)                       Zs = [z | s]
 *   GNN_SCORE_GAAN     e = <q_u, k_v>                      Zs = [z | q], Tv = k [n, F]
 *   GNN_SCORE_GENE     e = <W_a, tanh(a_u + b_v)>          Zs = [z | a], Tv = b [n, F], Wa [H, Fh]
 * y_v[h] = SUM_u softmax_u(e_uv[h]) z_u[h]; head_mean = 1 averages the heads
 * (Y [n, Fh]) instead of concatenating them (Y [n, F]).  Empty rows give 0.
 * s, t, q, k, a, b are the W_l h / W_r h projections (caller's GEMM).  Zs:
 * [n_src, ldz] device, Tv: [n, ldt].  Sym-GAT needs n == n_src.  GaAN and
 * Gene-linear need Fh / vec to be a power of two <= 32 for some vector width
 * vec in {8, 4, 2, 1} dividing Fh (else GNN_ERR_UNSUPPORTED).  Workspace:
 * gnn_workspace_size(plan, head_mean ? GNN_OP_ATTN_AGGREGATE_MEAN :
 * GNN_OP_ATTN_AGGREGATE, 0, F, H).
 */
typedef enum {
  GNN_SCORE_GAT = 0,
  GNN_SCORE_SYM_GAT = 1,
  GNN_SCORE_LINEAR = 2,
  GNN_SCORE_GAAN = 3,
  GNN_SCORE_GENE = 4
} gnn_score;
gnn_status gnn_attn_aggregate(gnn_plan_t plan, int score, const float *Zs, int64_t ldz,
                              const float *Tv, int64_t ldt, const float *Wa, int32_t H, int32_t Fh,
                              float neg_slope, int32_t head_mean, float *Y, int64_t ldy, void *ws,
                              size_t ws_bytes, gnn_stream_t stream);

/* Number of kernels this library launched since load (for bench accounting). */
uint64_t gnn_launch_count(void);

const char *gnn_last_error(void);
const char *gnn_version(void);

#ifdef __cplusplus
}
#endif
#endif /* GNN_H */
