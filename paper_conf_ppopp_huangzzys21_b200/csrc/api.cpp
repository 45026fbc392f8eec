// api.cpp — the C-ABI of libgnn.so (include/gnn.h): validation, plan
// lifetime, dispatch to the sm_100a kernels.  No exception crosses the ABI.
#include <algorithm>
#include <atomic>
#include <chrono>
#include <climits>
#include <cstring>
#include <exception>
#include <new>
#include <string>

#include "gnn_internal.h"

namespace gnn {
static gnn_status pack_mirrors(float *const *mirrors, int32_t n_mirrors, GemmMirrors &m);
}

namespace gnn {

static thread_local std::string t_last_error;
static std::atomic<uint64_t> g_launches{0};

void set_error(const std::string &msg) { t_last_error = msg; }
void count_launch(uint64_t k) { g_launches.fetch_add(k, std::memory_order_relaxed); }

gnn_status cuda_status(cudaError_t e, const char *what) {
  if (e == cudaSuccess) return GNN_OK;
  set_error(std::string(what) + ": " + cudaGetErrorString(e));
  return e == cudaErrorMemoryAllocation ? GNN_ERR_NOMEM : GNN_ERR_CUDA;
}

static double ms_since(std::chrono::steady_clock::time_point t0) {
  return std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
}

static size_t align256(size_t b) { return (b + 255) & ~(size_t)255; }

static void free_plan(gnn_plan_s *p) {
  if (!p) return;
  int cur = 0;
  cudaGetDevice(&cur);
  cudaSetDevice(p->device);
  for (void *d : p->dev_allocs) cudaFree(d);
  for (void *d : p->sched_allocs) cudaFree(d);
  if (p->d_hot) cudaFree(p->d_hot);
  cudaSetDevice(cur);
  delete p;
}

#define GNN_TRY(...)                                       \
  try {                                                     \
    __VA_ARGS__                                             \
  } catch (const std::bad_alloc &) {                        \
    gnn::set_error("host allocation failed");               \
    return GNN_ERR_NOMEM;                                   \
  } catch (const std::exception &ex) {                      \
    gnn::set_error(std::string("internal: ") + ex.what()); \
    return GNN_ERR_INTERNAL;                                \
  } catch (...) {                                           \
    gnn::set_error("internal: unknown exception");          \
    return GNN_ERR_INTERNAL;                                \
  }

static gnn_status check(bool ok, const char *msg) {
  if (ok) return GNN_OK;
  set_error(msg);
  return GNN_ERR_INVALID_ARG;
}

// overlap of [a, a + na) and [b, b + nb) in bytes
static bool overlaps(const void *a, size_t na, const void *b, size_t nb) {
  if (!a || !b || na == 0 || nb == 0) return false;
  const char *x = (const char *)a, *y = (const char *)b;
  return x < y + nb && y < x + na;
}
static size_t span_bytes(int64_t rows, int64_t ld, int64_t width) {
  return rows <= 0 ? 0 : sizeof(float) * (size_t)((rows - 1) * ld + width);
}

}  // namespace gnn

using namespace gnn;

extern "C" {

const char *gnn_last_error(void) { return t_last_error.c_str(); }
const char *gnn_version(void) { return "gnn-b200 0.1 (sm_100a)"; }
uint64_t gnn_launch_count(void) { return g_launches.load(); }

void gnn_plan_opts_default(gnn_plan_opts *o) {
  if (!o) return;
  std::memset(o, 0, sizeof(*o));
  o->struct_size = sizeof(gnn_plan_opts);
  o->reorder = 0;
  o->group_size = -1;
  o->tile_groups = 32;
  o->cluster_cap = 32;
  o->minhash_k = 32;
  o->lsh_rows = 2;
  o->pair_window = 8;
  o->min_sim = -1;
  o->deterministic = 1;
  o->cluster_order = 1;
  o->seed = 0;
}

}  // extern "C"

namespace gnn {
// Plan construction shared by gnn_plan_create_ex (perm_h == NULL: LAS or the
// identity order per opts) and gnn_plan_create_perm / gnn_plan_load (the task
// order given, e.g. a LAS schedule computed offline).
gnn_status create_plan(int64_t n, int64_t n_src, int64_t nnz, const int64_t *rowptr_h, const int32_t *colidx_h,
                       const int32_t *src_degree_h, const int32_t *perm_h, const gnn_plan_opts *opts_in,
                       gnn_plan_t *out) {
  {
    if (!out) return check(false, "out is NULL");
    *out = nullptr;
    auto t0 = std::chrono::steady_clock::now();
    gnn_plan_opts opts;
    gnn_plan_opts_default(&opts);
    if (opts_in) {
      if (opts_in->struct_size != sizeof(gnn_plan_opts)) return check(false, "opts.struct_size mismatch");
      opts = *opts_in;
    }
    if (n < 0 || n_src < 0 || nnz < 0 || n >= INT32_MAX || n_src >= INT32_MAX) {
      set_error("negative or too large sizes");
      return GNN_ERR_INVALID_GRAPH;
    }
    if (nnz >= INT32_MAX) {
      set_error("nnz >= 2^31 is not supported (int32 device indices)");
      return GNN_ERR_INVALID_GRAPH;
    }
    if (!rowptr_h || (nnz > 0 && !colidx_h)) return check(false, "rowptr/colidx is NULL");
    if (opts.tile_groups == 0) opts.tile_groups = 32;
    if (opts.tile_groups < 1 || opts.tile_groups > 256) return check(false, "tile_groups out of [1, 256]");
    if (opts.reorder) {
      if (opts.minhash_k < 1 || opts.minhash_k > 64) return check(false, "minhash_k out of [1, 64]");
      if (opts.lsh_rows < 1 || opts.minhash_k % opts.lsh_rows) return check(false, "lsh_rows must divide minhash_k");
      if (opts.pair_window < 1) return check(false, "pair_window < 1");
      if (opts.cluster_cap < 1) return check(false, "cluster_cap < 1");
    }
    // a1: CSR validation, O(n + nnz)
    if (rowptr_h[0] != 0 || rowptr_h[n] != nnz) {
      set_error("rowptr[0] != 0 or rowptr[n] != nnz");
      return GNN_ERR_INVALID_GRAPH;
    }
    int32_t maxd = 0;
    for (int64_t v = 0; v < n; ++v) {
      const int64_t d = rowptr_h[v + 1] - rowptr_h[v];
      if (d < 0) {
        set_error("rowptr is decreasing at row " + std::to_string(v));
        return GNN_ERR_INVALID_GRAPH;
      }
      if (d > maxd) maxd = (int32_t)d;
    }
    for (int64_t k = 0; k < nnz; ++k)
      if (colidx_h[k] < 0 || colidx_h[k] >= n_src) {
        set_error("colidx out of range at entry " + std::to_string(k));
        return GNN_ERR_INVALID_GRAPH;
      }
    gnn_plan_s *p = new gnn_plan_s();
    p->n = n;
    p->n_src = n_src;
    p->nnz = nnz;
    p->opts = opts;
    p->max_degree = maxd;
    p->T = opts.tile_groups;
    // NG bound (R8-ii): largest multiple of 16 <= 10 * average degree
    // (P:1163-1165), clamped to [16, 4096]
    int64_t ng = opts.group_size;
    if (ng < 0) ng = default_group_size(n, nnz);
    p->info.group_size = (int32_t)ng;
    if (ng == 0) ng = 1 << 30;  // never split
    p->ng = (int32_t)ng;
    p->rowptr.assign(rowptr_h, rowptr_h + n + 1);
    cudaGetDevice(&p->device);
    p->info.ms_validate = ms_since(t0);

    auto fail = [&](gnn_status st) {
      free_plan(p);
      return st;
    };
    // upload CSR (int32 on device)
    t0 = std::chrono::steady_clock::now();
    std::vector<int32_t> rp32((size_t)n + 1);
    for (int64_t v = 0; v <= n; ++v) rp32[v] = (int32_t)rowptr_h[v];
    void *d_rowptr = nullptr, *d_colidx = nullptr, *d_nsrc = nullptr, *d_ndst = nullptr, *d_dout = nullptr;
    cudaError_t e = cudaMalloc(&d_rowptr, sizeof(int32_t) * (n + 1));
    if (e == cudaSuccess) p->dev_allocs.push_back(d_rowptr);
    if (e == cudaSuccess) e = cudaMalloc(&d_colidx, sizeof(int32_t) * (nnz > 0 ? nnz : 1));
    if (e == cudaSuccess) p->dev_allocs.push_back(d_colidx);
    if (e == cudaSuccess) e = cudaMalloc(&d_nsrc, sizeof(float) * (n_src > 0 ? n_src : 1));
    if (e == cudaSuccess) p->dev_allocs.push_back(d_nsrc);
    if (e == cudaSuccess) e = cudaMalloc(&d_ndst, sizeof(float) * (size_t)(n + 4));  // + 4: 16-byte bulk reads
    if (e == cudaSuccess) p->dev_allocs.push_back(d_ndst);
    if (e == cudaSuccess) e = cudaMalloc(&d_dout, sizeof(int32_t) * (n_src > 0 ? n_src : 1));
    if (e == cudaSuccess) p->dev_allocs.push_back(d_dout);
    if (e == cudaSuccess) e = cudaMemcpy(d_rowptr, rp32.data(), sizeof(int32_t) * (n + 1), cudaMemcpyHostToDevice);
    if (e == cudaSuccess && nnz > 0)
      e = cudaMemcpy(d_colidx, colidx_h, sizeof(int32_t) * nnz, cudaMemcpyHostToDevice);
    if (e == cudaSuccess && src_degree_h && n_src > 0)
      e = cudaMemcpy(d_dout, src_degree_h, sizeof(int32_t) * n_src, cudaMemcpyHostToDevice);
    if (e != cudaSuccess) return fail(cuda_status(e, "plan allocation/upload"));
    p->dg.rowptr = (const int32_t *)d_rowptr;
    p->dg.colidx = (const int32_t *)d_colidx;
    p->dg.nsrc = (const float *)d_nsrc;
    p->dg.ndst = (const float *)d_ndst;
    p->d_dout = (const int32_t *)d_dout;
    p->info.ms_upload = ms_since(t0);
    // a1: degrees + normalisers on the GPU
    t0 = std::chrono::steady_clock::now();
    e = launch_degrees(p->dg.rowptr, p->dg.colidx, n, n_src, nnz,
                       src_degree_h ? (const int32_t *)d_dout : nullptr, (int32_t *)d_dout,
                       (float *)d_nsrc, (float *)d_ndst, nullptr);
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    if (e != cudaSuccess) return fail(cuda_status(e, "degrees"));
    p->info.ms_degrees = ms_since(t0);
    // a2: locality-aware task scheduling
    if (perm_h) {
      // given task order: must be a permutation of [0, n)
      std::vector<uint8_t> seen((size_t)n, 0);
      for (int64_t i = 0; i < n; ++i) {
        const int32_t v = perm_h[i];
        if (v < 0 || v >= n || seen[(size_t)v]) {
          set_error("perm is not a permutation of [0, n) (entry " + std::to_string(i) + ")");
          return fail(GNN_ERR_INVALID_ARG);
        }
        seen[(size_t)v] = 1;
      }
      p->perm.assign(perm_h, perm_h + n);
      p->n_clusters = 0;
    } else if (opts.reorder && n > 0) {
      t0 = std::chrono::steady_clock::now();
      const int32_t K = opts.minhash_k;
      uint64_t *d_sig = nullptr;
      e = cudaMalloc(&d_sig, sizeof(uint64_t) * (size_t)n * K);
      if (e != cudaSuccess) return fail(cuda_status(e, "minhash alloc"));
      e = launch_minhash(p->dg.rowptr, p->dg.colidx, n, K, opts.seed, d_sig, nullptr);
      p->sig.resize((size_t)n * K);
      if (e == cudaSuccess)
        e = cudaMemcpy(p->sig.data(), d_sig, sizeof(uint64_t) * (size_t)n * K, cudaMemcpyDeviceToHost);
      cudaFree(d_sig);
      if (e != cudaSuccess) return fail(cuda_status(e, "minhash"));
      p->info.ms_minhash = ms_since(t0);
      t0 = std::chrono::steady_clock::now();
      const int64_t np = las_lsh_pairs(n, rowptr_h, p->sig.data(), K, opts.lsh_rows, opts.pair_window, p->pairs);
      p->info.n_pairs = np;
      p->info.ms_lsh = ms_since(t0);
      t0 = std::chrono::steady_clock::now();
      const int32_t min_sim = opts.min_sim < 0 ? opts.lsh_rows : opts.min_sim;
      p->n_clusters = las_merge(n, p->sig.data(), K, p->pairs, opts.cluster_cap, min_sim, opts.cluster_order, p->perm,
                                p->cluster_of);
      p->info.ms_merge = ms_since(t0);
    } else {
      p->perm.resize((size_t)n);
      for (int64_t v = 0; v < n; ++v) p->perm[v] = (int32_t)v;
      p->n_clusters = n;
    }
    // a3: neighbor grouping + tiles
    t0 = std::chrono::steady_clock::now();
    p->colidx_h = colidx_h;
    gnn_status st = build_schedule(p);
    p->colidx_h = nullptr;
    if (st != GNN_OK) return fail(st);
    p->info.ms_ng = ms_since(t0);
    p->info.n = n;
    p->info.n_src = n_src;
    p->info.nnz = nnz;
    p->info.n_clusters = p->n_clusters;
    p->info.tile_groups = p->T;
    p->info.max_degree = maxd;
    p->info.reorder = opts.reorder;
    *out = p;
    return GNN_OK;
  }
}
}  // namespace gnn

extern "C" {

gnn_status gnn_plan_create_ex(int64_t n, int64_t n_src, int64_t nnz, const int64_t *rowptr_h,
                              const int32_t *colidx_h, const int32_t *src_degree_h,
                              const gnn_plan_opts *opts_in, gnn_plan_t *out) {
  GNN_TRY({ return create_plan(n, n_src, nnz, rowptr_h, colidx_h, src_degree_h, nullptr, opts_in, out); })
}

gnn_status gnn_plan_create_perm(int64_t n, int64_t n_src, int64_t nnz, const int64_t *rowptr_h,
                                const int32_t *colidx_h, const int32_t *src_degree_h, const int32_t *perm_h,
                                const gnn_plan_opts *opts_in, gnn_plan_t *out) {
  GNN_TRY({
    if (!perm_h && n > 0) return check(false, "perm_h is NULL");
    return create_plan(n, n_src, nnz, rowptr_h, colidx_h, src_degree_h, perm_h, opts_in, out);
  })
}

gnn_status gnn_plan_create(int64_t n, int64_t nnz, const int64_t *rowptr_h, const int32_t *colidx_h,
                           const gnn_plan_opts *opts, gnn_plan_t *out) {
  return gnn_plan_create_ex(n, n, nnz, rowptr_h, colidx_h, nullptr, opts, out);
}

gnn_status gnn_plan_get_info(gnn_plan_t p, gnn_plan_info *info) {
  if (!p || !info) return check(false, "plan/info is NULL");
  *info = p->info;
  return GNN_OK;
}

gnn_status gnn_plan_export(gnn_plan_t p, int32_t *perm_h, int32_t *grp_row_h, int64_t *grp_beg_h) {
  if (!p) return check(false, "plan is NULL");
  if (perm_h) std::memcpy(perm_h, p->perm.data(), sizeof(int32_t) * p->perm.size());
  if (grp_row_h) std::memcpy(grp_row_h, p->grp_row.data(), sizeof(int32_t) * p->grp_row.size());
  if (grp_beg_h) std::memcpy(grp_beg_h, p->grp_beg.data(), sizeof(int64_t) * p->grp_beg.size());
  return GNN_OK;
}

gnn_status gnn_plan_export_las(gnn_plan_t p, uint64_t *sig_h, int32_t *pairs_h, int32_t *cluster_of_h) {
  if (!p) return check(false, "plan is NULL");
  if (!p->opts.reorder || p->sig.empty()) {
    set_error(p->opts.reorder ? "plan has no LAS intermediates (given order, or loaded without them)"
                              : "plan was built without reorder");
    return GNN_ERR_INVALID_ARG;
  }
  if (sig_h) std::memcpy(sig_h, p->sig.data(), sizeof(uint64_t) * p->sig.size());
  if (pairs_h) std::memcpy(pairs_h, p->pairs.data(), sizeof(int32_t) * p->pairs.size());
  if (cluster_of_h) std::memcpy(cluster_of_h, p->cluster_of.data(), sizeof(int32_t) * p->cluster_of.size());
  return GNN_OK;
}

gnn_status gnn_plan_normalizers(gnn_plan_t p, const float **nsrc, const float **ndst) {
  if (!p) return check(false, "plan is NULL");
  if (nsrc) *nsrc = p->dg.nsrc;
  if (ndst) *ndst = p->dg.ndst;
  return GNN_OK;
}

gnn_status gnn_plan_destroy(gnn_plan_t p) {
  GNN_TRY({
    free_plan(p);
    return GNN_OK;
  })
}

// GAT transform workspace: the tensor-core W image of the H*Fh-column GEMM
// with the score epilogue, or (heads not a multiple of 32 wide) the folded
// weights [W | W a_src | W a_dst] and the W image of that wider GEMM
static size_t ws_gat_transform(int64_t m, int32_t f_in, int32_t H, int32_t Fh) {
  const int32_t ld = ((H * Fh + 2 * H) + 7) / 8 * 8;
  const size_t fold = align256(gemm_tc_workspace(m, f_in, ld)) + align256(sizeof(float) * (size_t)f_in * ld);
  return std::max(align256(gemm_tc_workspace(m, f_in, H * Fh)), fold);
}
// layer workspaces: [transform workspace][layer buffers][aggregation workspace]
static size_t ws_gat_layer_head(int64_t n, int32_t f_in, int32_t HF, int32_t H, int32_t *ldwe) {
  const int32_t ld = ((HF + 2 * H) + 7) / 8 * 8;
  if (ldwe) *ldwe = ld;
  return ws_gat_transform(n, f_in, H, HF / H) + align256(sizeof(float) * (size_t)n * ld);
}
static size_t ws_edgeconv_head(int64_t n, int32_t f_in, int32_t f_out) {
  const size_t ld = 2 * (size_t)f_out;
  return align256(gemm_tc_workspace(n, f_in, (int32_t)ld)) + align256(sizeof(float) * (size_t)f_in * ld) +
         align256(sizeof(float) * ld) + align256(sizeof(float) * (size_t)n * ld);
}
static int32_t ld8(int32_t f) { return (f + 7) / 8 * 8; }

// GraphSAGE-LSTM layer workspace: [gemm ws][Wcat f_in x ld][bcat ld][table n x T][GS n_src x ld]
static constexpr int32_t kSageF = 32;
static size_t ws_sage_lstm(const gnn_plan_s *p, int32_t f_in, int32_t f_out, int32_t T) {
  const int32_t ld = 4 * kSageF + f_out;
  const int32_t ldp = (ld + 7) / 8 * 8;  // GS row stride: 16-byte aligned rows for the cell kernel
  return align256(gemm_tc_workspace(p->n_src, f_in, ld)) + align256(sizeof(float) * (size_t)f_in * ld) +
         align256(sizeof(float) * (size_t)ld) + align256(sizeof(int32_t) * (size_t)p->n * (size_t)(T > 0 ? T : 0)) +
         align256(sizeof(float) * (size_t)p->n_src * ldp);
}

size_t gnn_workspace_size(gnn_plan_t p, int op, int32_t f_in, int32_t f_out, int32_t heads) {
  if (!p) return 0;
  switch (op) {
    case GNN_OP_AGGREGATE: return agg_workspace_bytes(p, 0, f_out, 0);
    case GNN_OP_GAT_AGGREGATE: return agg_workspace_bytes(p, 3, f_out, heads);
    case GNN_OP_EDGECONV: return ws_edgeconv_head(p->n, f_in, f_out) + agg_workspace_bytes(p, 2, f_out, 0);
    case GNN_OP_GAT_LAYER:
      return ws_gat_layer_head(p->n, f_in, f_out, heads, nullptr) + agg_workspace_bytes(p, 3, f_out, heads);
    case GNN_OP_GCN_LAYER: {
      const bool tf = f_out <= f_in;  // auto order; both orders fit in max()
      (void)tf;
      const size_t a = align256(gemm_tc_workspace(p->n_src, f_in, f_out)) +
                       align256(sizeof(float) * (size_t)p->n_src * ld8(f_out)) + agg_workspace_bytes(p, 0, f_out, 0);
      const size_t b = align256(gemm_tc_workspace(p->n, f_in, f_out)) +
                       align256(sizeof(float) * (size_t)p->n * ld8(f_in)) + agg_workspace_bytes(p, 0, f_in, 0);
      return a > b ? a : b;
    }
    case GNN_OP_SAGE_LSTM_LAYER: return ws_sage_lstm(p, f_in, f_out, heads);
    case GNN_OP_ATTN_AGGREGATE: return agg_workspace_bytes(p, 4, f_out, heads);
    case GNN_OP_ATTN_AGGREGATE_MEAN:
      return align256(sizeof(float) * (size_t)p->n * (size_t)(f_out > 0 ? f_out : 0)) + agg_workspace_bytes(p, 4, f_out, heads);
    default: return 0;
  }
}

static gnn_status agg_common(gnn_plan_t p, AggArgs &a, void *ws, size_t ws_bytes, gnn_stream_t stream) {
  a.deterministic = p->opts.deterministic;
  return launch_aggregate(p, a, ws, ws_bytes, (cudaStream_t)stream);
}

gnn_status gnn_aggregate(gnn_plan_t p, int reduce, int weight, const float *edge_w, const float *X,
                         int64_t ldx, int32_t F, float *Y, int64_t ldy, int32_t relu, const float *add_row,
                         int64_t ld_add, void *ws, size_t ws_bytes, gnn_stream_t stream) {
  GNN_TRY({
    if (!p) return check(false, "plan is NULL");
    if (reduce < 0 || reduce > 2) return check(false, "reduce out of range");
    if (weight < 0 || weight > 2) return check(false, "weight out of range");
    if (F < 0) return check(false, "F < 0");
    if (F == 0) return GNN_OK;
    if (!Y || (p->nnz > 0 && !X)) return check(false, "X/Y is NULL");
    if (ldx < F || ldy < F) return check(false, "ld < F");
    if (weight == GNN_W_EDGE && !edge_w && p->nnz > 0) return check(false, "edge_w required for GNN_W_EDGE");
    if (add_row && ld_add < F) return check(false, "ld_add < F");
    if (overlaps(X, span_bytes(p->n_src, ldx, F), Y, span_bytes(p->n, ldy, F)))
      return check(false, "X and Y overlap");
    AggArgs a{};
    a.mode = reduce;
    a.weight = weight;
    a.edge_w = edge_w;
    a.X = X;
    a.ldx = ldx;
    a.F = F;
    a.Y = Y;
    a.ldy = ldy;
    a.add_row = add_row;
    a.ld_add = ld_add;
    a.relu = relu;
    return agg_common(p, a, ws, ws_bytes, stream);
  })
}

gnn_status gnn_aggregate_accumulate(gnn_plan_t p, int weight, const float *edge_w, const float *X, int64_t ldx,
                                    int32_t F, float *Y, int64_t ldy, int32_t accumulate, void *ws, size_t ws_bytes,
                                    gnn_stream_t stream) {
  GNN_TRY({
    if (!p) return check(false, "plan is NULL");
    if (weight != GNN_W_ONE && weight != GNN_W_EDGE) return check(false, "accumulate: weight must be ONE or EDGE");
    if (F < 0) return check(false, "F < 0");
    if (F == 0) return GNN_OK;
    if (!Y || (p->nnz > 0 && !X)) return check(false, "X/Y is NULL");
    if (ldx < F || ldy < F) return check(false, "ld < F");
    if (weight == GNN_W_EDGE && !edge_w && p->nnz > 0) return check(false, "edge_w required for GNN_W_EDGE");
    if (overlaps(X, span_bytes(p->n_src, ldx, F), Y, span_bytes(p->n, ldy, F)))
      return check(false, "X and Y overlap");
    AggArgs a{};
    a.mode = 0;
    a.weight = weight;
    a.edge_w = edge_w;
    a.X = X;
    a.ldx = ldx;
    a.F = F;
    a.Y = Y;
    a.ldy = ldy;
    a.accum = accumulate ? 1 : 0;
    return agg_common(p, a, ws, ws_bytes, stream);
  })
}

gnn_status gnn_scale_rows(float *Y, int64_t ldy, int64_t n, int32_t F, const float *scale, int32_t relu,
                          gnn_stream_t stream) {
  GNN_TRY({
    if (n < 0 || F < 0 || ldy < F) return check(false, "bad scale_rows sizes");
    if (n > 0 && F > 0 && (!Y || !scale)) return check(false, "Y/scale is NULL");
    return cuda_status(launch_scale_rows(Y, ldy, n, F, scale, relu, (cudaStream_t)stream), "scale rows");
  })
}

gnn_status gnn_gat_aggregate(gnn_plan_t p, const float *Zs, int64_t ldz, const float *t, int64_t ldt,
                             int32_t H, int32_t Fh, float neg_slope, float *Y, int64_t ldy, void *ws,
                             size_t ws_bytes, gnn_stream_t stream) {
  GNN_TRY({
    if (!p) return check(false, "plan is NULL");
    if (H < 1 || Fh < 1 || H > 256) return check(false, "H in [1, 256] and Fh >= 1 required");
    const int32_t F = H * Fh;
    if (!Y || !t || (p->nnz > 0 && !Zs)) return check(false, "Zs/t/Y is NULL");
    if (ldz < F + H || ldt < H || ldy < F) return check(false, "ldz < H*Fh+H or ldt < H or ldy < H*Fh");
    if (overlaps(Zs, span_bytes(p->n_src, ldz, F + H), Y, span_bytes(p->n, ldy, F)))
      return check(false, "Zs and Y overlap");
    AggArgs a{};
    a.mode = 3;
    a.X = Zs;
    a.ldx = ldz;
    a.F = F;
    a.Y = Y;
    a.ldy = ldy;
    a.t = t;
    a.ldt = ldt;
    a.H = H;
    a.Fh = Fh;
    a.slope = neg_slope;
    return agg_common(p, a, ws, ws_bytes, stream);
  })
}

size_t gnn_gemm_workspace_size(int64_t m, int32_t k, int32_t n) { return gemm_tc_workspace(m, k, n); }

gnn_status gnn_gemm(const float *X, int64_t ldx, const float *W, int64_t ldw, float *H, int64_t ldh,
                    int64_t m, int32_t k, int32_t n, const float *row_scale, const float *col_bias,
                    int32_t relu, void *ws, size_t ws_bytes, gnn_stream_t stream) {
  GNN_TRY({
    if (m < 0 || k < 0 || n < 0) return check(false, "negative GEMM size");
    if (m == 0 || n == 0) return GNN_OK;
    if (!H || (k > 0 && (!X || !W))) return check(false, "X/W/H is NULL");
    if (ldx < k || ldw < n || ldh < n) return check(false, "GEMM leading dimension too small");
    if (overlaps(H, span_bytes(m, ldh, n), X, span_bytes(m, ldx, k)) ||
        overlaps(H, span_bytes(m, ldh, n), W, span_bytes(k, ldw, n)))
      return check(false, "H overlaps X or W");
    return launch_gemm(X, ldx, W, ldw, H, ldh, m, k, n, row_scale, col_bias, relu, ws, ws_bytes,
                       (cudaStream_t)stream);
  })
}

gnn_status gnn_gemm_mirrored(const float *X, int64_t ldx, const float *W, int64_t ldw, float *H, int64_t ldh,
                             int64_t m, int32_t k, int32_t n, const float *row_scale, const float *col_bias,
                             int32_t relu, float *const *mirrors, int32_t n_mirrors, void *ws, size_t ws_bytes,
                             gnn_stream_t stream) {
  GNN_TRY({
    if (m < 0 || k < 1 || n < 0) return check(false, "GEMM sizes: m, n >= 0, k >= 1");
    if (m == 0 || n == 0) return GNN_OK;
    if (!H || !X || !W) return check(false, "X/W/H is NULL");
    if (ldx < k || ldw < n || ldh < n) return check(false, "GEMM leading dimension too small");
    if (overlaps(H, span_bytes(m, ldh, n), X, span_bytes(m, ldx, k)) ||
        overlaps(H, span_bytes(m, ldh, n), W, span_bytes(k, ldw, n)))
      return check(false, "H overlaps X or W");
    GemmMirrors mir;
    gnn_status st = pack_mirrors(mirrors, n_mirrors, mir);
    if (st != GNN_OK) return st;
    for (int32_t q = 0; q < n_mirrors; ++q)
      if (overlaps(mirrors[q], span_bytes(m, ldh, n), X, span_bytes(m, ldx, k)) ||
          overlaps(mirrors[q], span_bytes(m, ldh, n), H, span_bytes(m, ldh, n)))
        return check(false, "a mirror overlaps X or H");
    if (!ws) return check(false, "the mirrored GEMM needs the tcgen05 workspace");
    return launch_gemm(X, ldx, W, ldw, H, ldh, m, k, n, row_scale, col_bias, relu, ws, ws_bytes,
                       (cudaStream_t)stream, &mir);
  })
}

int gnn_set_gemm_impl(int impl) { return set_gemm_impl(impl); }

// CUDA IPC for the mirrors of a multi-process exchange (NEXT-2)
gnn_status gnn_ipc_alloc(size_t bytes, void **ptr, void *handle) {
  GNN_TRY({
    if (!ptr || !handle || bytes == 0) return check(false, "gnn_ipc_alloc: NULL argument or zero size");
    *ptr = nullptr;
    cudaError_t e = cudaMalloc(ptr, bytes);
    if (e != cudaSuccess) return cuda_status(e, "gnn_ipc_alloc cudaMalloc");
    cudaIpcMemHandle_t h;
    e = cudaIpcGetMemHandle(&h, *ptr);
    if (e != cudaSuccess) {
      cudaFree(*ptr);
      *ptr = nullptr;
      return cuda_status(e, "gnn_ipc_alloc cudaIpcGetMemHandle");
    }
    memcpy(handle, &h, sizeof(h));
    return GNN_OK;
  })
}

gnn_status gnn_ipc_free(void *ptr) {
  GNN_TRY({ return ptr ? cuda_status(cudaFree(ptr), "gnn_ipc_free") : GNN_OK; })
}

gnn_status gnn_ipc_open(const void *handle, void **ptr) {
  GNN_TRY({
    if (!ptr || !handle) return check(false, "gnn_ipc_open: NULL argument");
    cudaIpcMemHandle_t h;
    memcpy(&h, handle, sizeof(h));
    return cuda_status(cudaIpcOpenMemHandle(ptr, h, cudaIpcMemLazyEnablePeerAccess), "gnn_ipc_open");
  })
}

gnn_status gnn_ipc_close(void *ptr) {
  GNN_TRY({ return ptr ? cuda_status(cudaIpcCloseMemHandle(ptr), "gnn_ipc_close") : GNN_OK; })
}

void gnn_set_agg_trace(void *trace_dev) { set_agg_trace(trace_dev); }

gnn_status gnn_set_agg_mapping(int32_t vec, int32_t lanes, int32_t nv) {
  GNN_TRY({
    if (!set_agg_mapping(vec, lanes, nv)) {
      set_error("gnn_set_agg_mapping: unsupported (vec, lanes, nv)");
      return GNN_ERR_INVALID_ARG;
    }
    return GNN_OK;
  })
}

}  // extern "C"

namespace gnn {
// [Z | s | t] = X W with s[h] = Z_h . a_src_h, t[h] = Z_h . a_dst_h (Table 2
// GAT, reading R5).  Heads of a multiple of 32 features: one
// tensor-core GEMM of H*Fh columns whose epilogue accumulates the scores from
// the Z values it stores.  Otherwise the scores are extra GEMM columns of the
// folded weights [W | W_h a_src_h | W_h a_dst_h] (a reassociation of Z a).
static gnn_status gat_transform(const float *X, int64_t ldx, int64_t m, int32_t f_in, const float *W, int64_t ldw,
                                const float *a_src, const float *a_dst, int32_t H, int32_t Fh, float *Zst,
                                int64_t ldz, void *ws, size_t ws_bytes, cudaStream_t s,
                                const GemmMirrors *mir = nullptr) {
  if (m == 0) return GNN_OK;
  if (ws_bytes < ws_gat_transform(m, f_in, H, Fh)) {
    set_error("gat transform workspace too small: need " + std::to_string(ws_gat_transform(m, f_in, H, Fh)));
    return GNN_ERR_WORKSPACE;
  }
  const int32_t HF = H * Fh;
  cudaError_t e = launch_gemm_att(X, ldx, W, ldw, Zst, ldz, m, f_in, H, Fh, a_src, a_dst, ws, ws_bytes, s, mir);
  if (e == cudaSuccess) return GNN_OK;
  if (e != cudaErrorNotSupported) return cuda_status(e, "gat transform");
  (void)cudaGetLastError();
  const int32_t ld = ((HF + 2 * H) + 7) / 8 * 8;
  if (ldw != HF) {
    set_error("gat transform: the folded path needs ldw == H * Fh");
    return GNN_ERR_UNSUPPORTED;
  }
  const size_t gws = align256(gemm_tc_workspace(m, f_in, ld));
  float *Wext = (float *)((char *)ws + gws);
  e = launch_gat_weights(W, a_src, a_dst, f_in, H, Fh, Wext, ld, s);
  if (e != cudaSuccess) return cuda_status(e, "gat weights");
  // the folded GEMM writes ld >= HF + 2H columns: stage through Zst only if it is wide enough
  if (ldz < ld) {
    set_error("gat transform: ldz must be >= round_up(H*Fh + 2H, 8) for this head size");
    return GNN_ERR_INVALID_ARG;
  }
  return launch_gemm(X, ldx, Wext, ld, Zst, ldz, m, f_in, ld, nullptr, nullptr, 0, ws, gws, s, mir);
}

// validate and pack the mirror pointers of the *_mirrored entry points
static gnn_status pack_mirrors(float *const *mirrors, int32_t n_mirrors, GemmMirrors &m) {
  memset(&m, 0, sizeof(m));
  if (n_mirrors < 0 || n_mirrors > kMaxMirrors || (n_mirrors > 0 && !mirrors)) {
    set_error("n_mirrors must be in [0, 7] with a mirror pointer array");
    return GNN_ERR_INVALID_ARG;
  }
  for (int32_t q = 0; q < n_mirrors; ++q) {
    if (!mirrors[q] || ((uintptr_t)mirrors[q] & 15)) {
      set_error("mirror pointers must be non-NULL and 16-byte aligned");
      return GNN_ERR_INVALID_ARG;
    }
    m.dst[q] = mirrors[q];
  }
  m.count = n_mirrors;
  return GNN_OK;
}
}  // namespace gnn

extern "C" {

size_t gnn_gat_transform_workspace_size(int64_t m, int32_t f_in, int32_t H, int32_t Fh) {
  if (m < 0 || f_in < 1 || H < 1 || Fh < 1) return 0;
  return ws_gat_transform(m, f_in, H, Fh);
}

gnn_status gnn_gat_transform(const float *X, int64_t ldx, int64_t m, int32_t f_in, const float *W, int64_t ldw,
                             const float *a_src, const float *a_dst, int32_t H, int32_t Fh, float *Zst, int64_t ldz,
                             void *ws, size_t ws_bytes, gnn_stream_t stream) {
  GNN_TRY({
    if (m < 0 || f_in < 1 || H < 1 || H > 256 || Fh < 1) return check(false, "bad GAT transform sizes");
    if (m > 0 && (!X || !W || !a_src || !a_dst || !Zst || !ws)) return check(false, "NULL argument");
    if (ldx < f_in || ldw < (int64_t)H * Fh || ldz < (int64_t)H * Fh + 2 * H)
      return check(false, "leading dimension too small (ldz >= H*Fh + 2H)");
    if (overlaps(Zst, span_bytes(m, ldz, (int64_t)H * Fh + 2 * H), X, span_bytes(m, ldx, f_in)))
      return check(false, "Zst overlaps X");
    return gat_transform(X, ldx, m, f_in, W, ldw, a_src, a_dst, H, Fh, Zst, ldz, ws, ws_bytes,
                         (cudaStream_t)stream);
  })
}

gnn_status gnn_gat_transform_mirrored(const float *X, int64_t ldx, int64_t m, int32_t f_in, const float *W,
                                      int64_t ldw, const float *a_src, const float *a_dst, int32_t H, int32_t Fh,
                                      float *Zst, int64_t ldz, float *const *mirrors, int32_t n_mirrors, void *ws,
                                      size_t ws_bytes, gnn_stream_t stream) {
  GNN_TRY({
    if (m < 0 || f_in < 1 || H < 1 || H > 256 || Fh < 1) return check(false, "bad GAT transform sizes");
    if (m > 0 && (!X || !W || !a_src || !a_dst || !Zst || !ws)) return check(false, "NULL argument");
    if (ldx < f_in || ldw < (int64_t)H * Fh || ldz < (int64_t)H * Fh + 2 * H)
      return check(false, "leading dimension too small (ldz >= H*Fh + 2H)");
    if (overlaps(Zst, span_bytes(m, ldz, (int64_t)H * Fh + 2 * H), X, span_bytes(m, ldx, f_in)))
      return check(false, "Zst overlaps X");
    GemmMirrors mir;
    gnn_status st = pack_mirrors(mirrors, n_mirrors, mir);
    if (st != GNN_OK) return st;
    return gat_transform(X, ldx, m, f_in, W, ldw, a_src, a_dst, H, Fh, Zst, ldz, ws, ws_bytes,
                         (cudaStream_t)stream, &mir);
  })
}

gnn_status gnn_gat_layer(gnn_plan_t p, const float *X, int64_t ldx, int32_t f_in, const float *W,
                         const float *a_src, const float *a_dst, int32_t H, int32_t Fh, float neg_slope,
                         float *Y, int64_t ldy, void *ws, size_t ws_bytes, gnn_stream_t stream) {
  GNN_TRY({
    if (!p) return check(false, "plan is NULL");
    if (p->n != p->n_src) return check(false, "gnn_gat_layer needs a square plan (n_src == n)");
    if (H < 1 || H > 256 || Fh < 1 || f_in < 1) return check(false, "H in [1, 256], Fh, f_in >= 1 required");
    if (!X || !W || !a_src || !a_dst || !Y) return check(false, "NULL argument");
    if (ldx < f_in || ldy < (int64_t)H * Fh) return check(false, "leading dimension too small");
    const int32_t HF = H * Fh;
    int32_t ldwe = 0;
    const size_t head = ws_gat_layer_head(p->n, f_in, HF, H, &ldwe);
    const size_t need = head + agg_workspace_bytes(p, 3, HF, H);
    if (!ws || ws_bytes < need) {
      set_error("workspace too small: need " + std::to_string(need));
      return GNN_ERR_WORKSPACE;
    }
    char *base = (char *)ws;
    const size_t tws = ws_gat_transform(p->n, f_in, H, Fh);
    float *Zst = (float *)(base + tws);
    cudaStream_t s = (cudaStream_t)stream;
    // [Z | s | t] (R5)
    gnn_status st = gat_transform(X, ldx, p->n, f_in, W, HF, a_src, a_dst, H, Fh, Zst, ldwe, base, tws, s);
    if (st != GNN_OK) return st;
    AggArgs a{};
    a.mode = 3;
    a.X = Zst;
    a.ldx = ldwe;
    a.F = HF;
    a.Y = Y;
    a.ldy = ldy;
    a.t = Zst + HF + H;
    a.ldt = ldwe;
    a.H = H;
    a.Fh = Fh;
    a.slope = neg_slope;
    return agg_common(p, a, base + head, ws_bytes - head, stream);
  })
}

gnn_status gnn_edgeconv_aggregate(gnn_plan_t p, const float *PQ, int64_t ldpq, int32_t f_out, float *Y,
                                  int64_t ldy, void *ws, size_t ws_bytes, gnn_stream_t stream) {
  GNN_TRY({
    if (!p) return check(false, "plan is NULL");
    if (p->n != p->n_src) return check(false, "EdgeConv needs a square plan");
    if (f_out < 1) return check(false, "f_out < 1");
    if (!PQ || !Y) return check(false, "PQ/Y is NULL");
    if (ldpq < 2 * (int64_t)f_out || ldy < f_out) return check(false, "leading dimension too small");
    if (overlaps(PQ, span_bytes(p->n, ldpq, 2 * f_out), Y, span_bytes(p->n, ldy, f_out)))
      return check(false, "PQ and Y overlap");
    AggArgs a{};
    a.mode = 2;
    a.weight = GNN_W_ONE;
    a.X = PQ;
    a.ldx = ldpq;
    a.F = f_out;
    a.Y = Y;
    a.ldy = ldy;
    a.add_row = PQ + f_out;
    a.ld_add = ldpq;
    a.relu = 1;
    return agg_common(p, a, ws, ws_bytes, stream);
  })
}

gnn_status gnn_edgeconv(gnn_plan_t p, const float *X, int64_t ldx, int32_t f_in, const float *theta,
                        const float *phi, const float *bias, int32_t f_out, float *Y, int64_t ldy, void *ws,
                        size_t ws_bytes, gnn_stream_t stream) {
  GNN_TRY({
    if (!p) return check(false, "plan is NULL");
    if (p->n != p->n_src) return check(false, "EdgeConv needs a square plan");
    if (f_in < 1 || f_out < 1) return check(false, "f_in/f_out < 1");
    if (!X || !theta || !phi || !Y) return check(false, "NULL argument");
    if (ldx < f_in || ldy < f_out) return check(false, "leading dimension too small");
    const size_t head = ws_edgeconv_head(p->n, f_in, f_out);
    const size_t need = head + agg_workspace_bytes(p, 2, f_out, 0);
    if (!ws || ws_bytes < need) {
      set_error("workspace too small: need " + std::to_string(need));
      return GNN_ERR_WORKSPACE;
    }
    const int64_t ld = 2 * (int64_t)f_out;
    char *base = (char *)ws;
    const size_t gws = align256(gemm_tc_workspace(p->n, f_in, (int32_t)ld));
    float *Wpq = (float *)(base + gws);
    float *bpq = (float *)(base + gws + align256(sizeof(float) * (size_t)f_in * ld));
    float *PQ = (float *)((char *)bpq + align256(sizeof(float) * ld));
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e = launch_edgeconv_weights(theta, phi, bias, f_in, f_out, Wpq, bpq, s);
    if (e != cudaSuccess) return cuda_status(e, "edgeconv weights");
    gnn_status st = launch_gemm(X, ldx, Wpq, ld, PQ, ld, p->n, f_in, (int32_t)ld, nullptr, bpq, 0, base, gws, s);
    if (st != GNN_OK) return st;
    return gnn_edgeconv_aggregate(p, PQ, ld, f_out, Y, ldy, base + head, ws_bytes - head, stream);
  })
}

gnn_status gnn_gcn_layer(gnn_plan_t p, const float *X, int64_t ldx, int32_t f_in, const float *W, int64_t ldw,
                         int32_t f_out, int32_t relu, int32_t order, float *Y, int64_t ldy, void *ws,
                         size_t ws_bytes, gnn_stream_t stream) {
  GNN_TRY({
    if (!p) return check(false, "plan is NULL");
    if (f_in < 1 || f_out < 1) return check(false, "f_in/f_out < 1");
    if (!X || !W || !Y) return check(false, "NULL argument");
    if (ldx < f_in || ldw < f_out || ldy < f_out) return check(false, "leading dimension too small");
    if (order < 0 || order > 2) return check(false, "order out of range");
    if (order == 0) order = f_out <= f_in ? 1 : 2;
    cudaStream_t s = (cudaStream_t)stream;
    if (order == 1) {
      // transform first: Hs = (X W) * nsrc[u]; y = ndst[v] * sum_u Hs[u]  (Eq 1 reassociated, R4-i)
      const int32_t ldh = ld8(f_out);
      const size_t gws = align256(gemm_tc_workspace(p->n_src, f_in, f_out));
      const size_t head = gws + align256(sizeof(float) * (size_t)p->n_src * ldh);
      const size_t need = head + agg_workspace_bytes(p, 0, f_out, 0);
      if (!ws || ws_bytes < need) {
        set_error("workspace too small: need " + std::to_string(need));
        return GNN_ERR_WORKSPACE;
      }
      float *Hs = (float *)((char *)ws + gws);
      gnn_status st = launch_gemm(X, ldx, W, ldw, Hs, ldh, p->n_src, f_in, f_out, p->dg.nsrc, nullptr, 0, ws, gws, s);
      if (st != GNN_OK) return st;
      AggArgs a{};
      a.mode = 0;
      a.weight = 3;  // W_DST_ONLY
      a.X = Hs;
      a.ldx = ldh;
      a.F = f_out;
      a.Y = Y;
      a.ldy = ldy;
      a.relu = relu;
      return agg_common(p, a, (char *)ws + head, ws_bytes - head, stream);
    }
    // aggregate first: A = A_gcn X; Y = ACT(A W)
    const int32_t lda = ld8(f_in);
    const size_t gws = align256(gemm_tc_workspace(p->n, f_in, f_out));
    const size_t head = gws + align256(sizeof(float) * (size_t)p->n * lda);
    const size_t need = head + agg_workspace_bytes(p, 0, f_in, 0);
    if (!ws || ws_bytes < need) {
      set_error("workspace too small: need " + std::to_string(need));
      return GNN_ERR_WORKSPACE;
    }
    float *A = (float *)((char *)ws + gws);
    AggArgs a{};
    a.mode = 0;
    a.weight = GNN_W_GCN;
    a.X = X;
    a.ldx = ldx;
    a.F = f_in;
    a.Y = A;
    a.ldy = lda;
    gnn_status st = agg_common(p, a, (char *)ws + head, ws_bytes - head, stream);
    if (st != GNN_OK) return st;
    return launch_gemm(A, lda, W, ldw, Y, ldy, p->n, f_in, f_out, nullptr, nullptr, relu, ws, gws, s);
  })
}

gnn_status gnn_gcn_aggregate_prescaled(gnn_plan_t p, const float *Hs, int64_t ldh, int32_t F, float *Y,
                                       int64_t ldy, int32_t relu, void *ws, size_t ws_bytes, gnn_stream_t stream) {
  GNN_TRY({
    if (!p) return check(false, "plan is NULL");
    if (F < 0) return check(false, "F < 0");
    if (F == 0) return GNN_OK;
    if (!Y || (p->nnz > 0 && !Hs)) return check(false, "Hs/Y is NULL");
    if (ldh < F || ldy < F) return check(false, "ld < F");
    if (overlaps(Hs, span_bytes(p->n_src, ldh, F), Y, span_bytes(p->n, ldy, F)))
      return check(false, "Hs and Y overlap");
    AggArgs a{};
    a.mode = 0;
    a.weight = 3;  // W_DST_ONLY: weight 1 in the loop, x ndst[v] in the epilogue
    a.X = Hs;
    a.ldx = ldh;
    a.F = F;
    a.Y = Y;
    a.ldy = ldy;
    a.relu = relu;
    return agg_common(p, a, ws, ws_bytes, stream);
  })
}

gnn_status gnn_gat_fold_weights(const float *W, const float *a_src, const float *a_dst, int32_t f_in, int32_t H,
                                int32_t Fh, float *Wext, int64_t ldwe, gnn_stream_t stream) {
  GNN_TRY({
    if (!W || !a_src || !a_dst || !Wext) return check(false, "NULL argument");
    if (f_in < 1 || H < 1 || Fh < 1) return check(false, "f_in, H, Fh must be >= 1");
    if (ldwe < (int64_t)H * Fh + 2 * H) return check(false, "ldwe < H*Fh + 2H");
    return cuda_status(launch_gat_weights(W, a_src, a_dst, f_in, H, Fh, Wext, (int32_t)ldwe, (cudaStream_t)stream),
                       "gat fold");
  })
}

gnn_status gnn_partition_rows(int64_t n, const int64_t *rowptr_h, int32_t nparts, int64_t *bounds_h) {
  GNN_TRY({
    if (n < 0 || nparts < 1 || !rowptr_h || !bounds_h) return check(false, "bad partition arguments");
    const int64_t E = rowptr_h[n];
    bounds_h[0] = 0;
    for (int32_t q = 1; q < nparts; ++q) {
      const int64_t target = (q * E + nparts - 1) / nparts;
      // smallest i in [bounds[q-1], n] with rowptr[i] >= target (binary search)
      int64_t lo = bounds_h[q - 1], hi = n;
      while (lo < hi) {
        const int64_t mid = lo + (hi - lo) / 2;
        if (rowptr_h[mid] >= target) hi = mid;
        else lo = mid + 1;
      }
      bounds_h[q] = lo;
    }
    bounds_h[nparts] = n;
    return GNN_OK;
  })
}

gnn_status gnn_local_csr(int64_t n, const int64_t *rowptr_h, const int32_t *colidx_h, const int64_t *bounds_h,
                         int32_t nparts, int32_t rank, int64_t *r_max, int64_t *local_nnz,
                         int64_t *local_rowptr_h, int32_t *local_colidx_h, int32_t *src_degree_h) {
  GNN_TRY({
    if (n < 0 || !rowptr_h || !bounds_h || nparts < 1 || rank < 0 || rank >= nparts || !r_max || !local_nnz)
      return check(false, "bad local_csr arguments");
    int64_t rm = 0;
    for (int32_t q = 0; q < nparts; ++q) rm = std::max<int64_t>(rm, bounds_h[q + 1] - bounds_h[q]);
    const int64_t lo = bounds_h[rank], hi = bounds_h[rank + 1];
    *r_max = rm;
    *local_nnz = rowptr_h[hi] - rowptr_h[lo];
    if (!local_rowptr_h && !local_colidx_h && !src_degree_h) return GNN_OK;  // size query
    // owner lookup: owner of u = the q with bounds[q] <= u < bounds[q+1]
    auto owner = [&](int64_t u) {
      int64_t a = 0, b = nparts - 1;
      while (a < b) {
        const int64_t mid = (a + b + 1) / 2;
        if (bounds_h[mid] <= u) a = mid;
        else b = mid - 1;
      }
      // skip empty parts that share the same bound
      while (a + 1 < nparts && bounds_h[a + 1] <= u) ++a;
      return a;
    };
    if (local_rowptr_h)
      for (int64_t v = lo; v <= hi; ++v) local_rowptr_h[v - lo] = rowptr_h[v] - rowptr_h[lo];
    if (local_colidx_h)
      for (int64_t k = rowptr_h[lo]; k < rowptr_h[hi]; ++k) {
        const int64_t u = colidx_h[k];
        const int64_t q = owner(u);
        local_colidx_h[k - rowptr_h[lo]] = (int32_t)(q * rm + (u - bounds_h[q]));
      }
    if (src_degree_h) {
      std::memset(src_degree_h, 0, sizeof(int32_t) * (size_t)(nparts * rm));
      for (int64_t k = 0; k < rowptr_h[n]; ++k) {
        const int64_t u = colidx_h[k];
        const int64_t q = owner(u);
        src_degree_h[q * rm + (u - bounds_h[q])] += 1;
      }
    }
    return GNN_OK;
  })
}

gnn_status gnn_local_csr_block(int64_t n, const int64_t *rowptr_h, const int32_t *colidx_h, const int64_t *bounds_h,
                               int32_t nparts, int32_t rank, int32_t q, int64_t *block_nnz, int64_t *block_rowptr_h,
                               int32_t *block_colidx_h) {
  GNN_TRY({
    if (n < 0 || !rowptr_h || !colidx_h || !bounds_h || nparts < 1 || rank < 0 || rank >= nparts || q < 0 ||
        q >= nparts || !block_nnz)
      return check(false, "bad local_csr_block arguments");
    const int64_t lo = bounds_h[rank], hi = bounds_h[rank + 1], qlo = bounds_h[q], qhi = bounds_h[q + 1];
    int64_t cnt = 0;
    if (block_rowptr_h) block_rowptr_h[0] = 0;
    for (int64_t v = lo; v < hi; ++v) {
      for (int64_t k = rowptr_h[v]; k < rowptr_h[v + 1]; ++k) {
        const int64_t u = colidx_h[k];
        if (u < qlo || u >= qhi) continue;
        if (block_colidx_h) block_colidx_h[cnt] = (int32_t)(u - qlo);
        ++cnt;
      }
      if (block_rowptr_h) block_rowptr_h[v - lo + 1] = cnt;
    }
    *block_nnz = cnt;
    return GNN_OK;
  })
}

gnn_status gnn_las_host(int64_t n, const int64_t *rowptr_h, const uint64_t *sig_h, int32_t K, int32_t r,
                        int32_t W, int32_t cap, int32_t min_sim, int32_t cluster_order, int32_t *perm_h,
                        int32_t *cluster_of_h,
                        int64_t *n_pairs, int64_t *n_clusters) {
  GNN_TRY({
    if (n < 0 || !rowptr_h || (n > 0 && !sig_h) || !perm_h) return check(false, "bad las_host arguments");
    if (K < 1 || r < 1 || K % r || W < 1 || cap < 1) return check(false, "bad LAS parameters");
    std::vector<int32_t> pairs, perm, cl;
    const int64_t np = las_lsh_pairs(n, rowptr_h, sig_h, K, r, W, pairs);
    const int64_t nc = las_merge(n, sig_h, K, pairs, cap, min_sim < 0 ? r : min_sim, cluster_order, perm, cl);
    std::memcpy(perm_h, perm.data(), sizeof(int32_t) * (size_t)n);
    if (cluster_of_h) std::memcpy(cluster_of_h, cl.data(), sizeof(int32_t) * (size_t)n);
    if (n_pairs) *n_pairs = np;
    if (n_clusters) *n_clusters = nc;
    return GNN_OK;
  })
}

gnn_status gnn_groups_host(int64_t n, const int64_t *rowptr_h, const int32_t *perm_h, int32_t ng,
                           int64_t *n_groups, int32_t *grp_row_h, int64_t *grp_beg_h) {
  GNN_TRY({
    if (n < 0 || !rowptr_h || !n_groups) return check(false, "bad groups_host arguments");
    std::vector<int32_t> gr;
    std::vector<int64_t> gb;
    schedule_host(n, rowptr_h, perm_h, ng > 0 ? ng : (1 << 30), gr, gb);
    *n_groups = (int64_t)gr.size();
    if (grp_row_h) std::memcpy(grp_row_h, gr.data(), sizeof(int32_t) * gr.size());
    if (grp_beg_h) std::memcpy(grp_beg_h, gb.data(), sizeof(int64_t) * gb.size());
    return GNN_OK;
  })
}



// ---------------------------------------------------------------------------
// NEXT-3 GraphSAGE-LSTM (Fig 6, reading R13)
// ---------------------------------------------------------------------------
gnn_status gnn_sample_neighbors(gnn_plan_t p, int32_t T, uint64_t seed, int32_t *table, gnn_stream_t stream) {
  GNN_TRY({
    if (!p || (!table && p->n > 0)) return check(false, "plan/table is NULL");
    if (T < 1 || T > 32) return check(false, "T must be in [1, 32]");
    return cuda_status(launch_sample_neighbors(p, T, seed, table, (cudaStream_t)stream), "sample neighbors");
  })
}

gnn_status gnn_sage_lstm_aggregate(gnn_plan_t p, const int32_t *table, int32_t T, const float *GS, int64_t ldg,
                                   int32_t F, const float *R, const float *W_neigh, int32_t F_out, float *Y,
                                   int64_t ldy, gnn_stream_t stream) {
  GNN_TRY({
    if (!p) return check(false, "plan is NULL");
    if (F != kSageF) {
      set_error("gnn_sage_lstm_aggregate: hidden size F must be 32");
      return GNN_ERR_UNSUPPORTED;
    }
    if (T < 1 || T > 32) return check(false, "T must be in [1, 32]");
    if (F_out < 1 || F_out > 32) {
      set_error("gnn_sage_lstm_aggregate: F_out must be in [1, 32]");
      return GNN_ERR_UNSUPPORTED;
    }
    if (p->n > 0 && (!table || !GS || !R || !W_neigh || !Y)) return check(false, "NULL argument");
    if (ldg < 4 * F + F_out || ldg % 4 != 0 || ldy < F_out) return check(false, "ldg < 4F+F_out (or not a multiple of 4) or ldy < F_out");
    if (reinterpret_cast<uintptr_t>(GS) % 16 != 0) return check(false, "GS must be 16-byte aligned");
    if (overlaps(GS, span_bytes(p->n_src, ldg, 4 * F + F_out), Y, span_bytes(p->n, ldy, F_out)))
      return check(false, "GS and Y overlap");
    return cuda_status(launch_sage_lstm(p, table, T, GS, ldg, R, W_neigh, F_out, Y, ldy, (cudaStream_t)stream),
                       "sage lstm");
  })
}

gnn_status gnn_sage_lstm_layer(gnn_plan_t p, const float *X, int64_t ldx, int32_t f_in, const float *W_ih,
                               const float *W_hh, const float *b_ih, const float *b_hh, const float *W_self,
                               const float *W_neigh, const float *bias, int32_t F, int32_t F_out, int32_t T,
                               uint64_t seed, float *Y, int64_t ldy, void *ws, size_t ws_bytes,
                               gnn_stream_t stream) {
  GNN_TRY({
    if (!p) return check(false, "plan is NULL");
    if (F != kSageF) {
      set_error("gnn_sage_lstm_layer: hidden size F must be 32");
      return GNN_ERR_UNSUPPORTED;
    }
    if (f_in < 1 || T < 1 || T > 32 || F_out < 1 || F_out > 32) return check(false, "f_in < 1, T or F_out out of [1, 32]");
    if (!X || !W_ih || !W_hh || !b_ih || !b_hh || !W_self || !W_neigh || !Y) return check(false, "NULL argument");
    if (ldx < f_in || ldy < F_out) return check(false, "leading dimension too small");
    const size_t need = ws_sage_lstm(p, f_in, F_out, T);
    if (!ws || ws_bytes < need) {
      set_error("workspace too small: need " + std::to_string(need));
      return GNN_ERR_WORKSPACE;
    }
    const int32_t ld = 4 * F + F_out;
    char *base = (char *)ws;
    const size_t gws = align256(gemm_tc_workspace(p->n_src, f_in, ld));
    float *Wcat = (float *)(base + gws);
    float *bcat = (float *)((char *)Wcat + align256(sizeof(float) * (size_t)f_in * ld));
    int32_t *table = (int32_t *)((char *)bcat + align256(sizeof(float) * (size_t)ld));
    float *GS = (float *)((char *)table + align256(sizeof(int32_t) * (size_t)p->n * T));
    cudaStream_t s = (cudaStream_t)stream;
    cudaError_t e = launch_lstm_weights(W_ih, b_ih, b_hh, W_self, bias, f_in, F, F_out, Wcat, bcat, s);
    if (e != cudaSuccess) return cuda_status(e, "lstm weights");
    // redundancy bypass: G = X W_ih^T + b_ih + b_hh and S = X W_self^T + b, once per node
    const int32_t ldp = (ld + 7) / 8 * 8;
    gnn_status st = launch_gemm(X, ldx, Wcat, ld, GS, ldp, p->n_src, f_in, ld, nullptr, bcat, 0, base, gws, s);
    if (st != GNN_OK) return st;
    e = launch_sample_neighbors(p, T, seed, table, s);
    if (e != cudaSuccess) return cuda_status(e, "sample neighbors");
    return cuda_status(launch_sage_lstm(p, table, T, GS, ldp, W_hh, W_neigh, F_out, Y, ldy, s), "sage lstm");
  })
}

// ---------------------------------------------------------------------------
// NEXT-4: Table 2 edge functions + softmax aggregation (reading R14)
// ---------------------------------------------------------------------------
gnn_status gnn_attn_aggregate(gnn_plan_t p, int score, const float *Zs, int64_t ldz, const float *Tv, int64_t ldt,
                              const float *Wa, int32_t H, int32_t Fh, float neg_slope, int32_t head_mean, float *Y,
                              int64_t ldy, void *ws, size_t ws_bytes, gnn_stream_t stream) {
  GNN_TRY({
    if (!p) return check(false, "plan is NULL");
    if (score < GNN_SCORE_GAT || score > GNN_SCORE_GENE) return check(false, "score out of range");
    if (H < 1 || Fh < 1 || H > 256) return check(false, "H in [1, 256] and Fh >= 1 required");
    const int32_t F = H * Fh;
    const int32_t extra = (score == GNN_SCORE_GAT || score == GNN_SCORE_LINEAR) ? H
                          : score == GNN_SCORE_SYM_GAT ? 2 * H : F;
    const bool needs_tv = score == GNN_SCORE_GAT || score == GNN_SCORE_GAAN || score == GNN_SCORE_GENE;
    const int32_t tv_w = score == GNN_SCORE_GAT ? H : F;
    if (!Y || (p->nnz > 0 && !Zs)) return check(false, "Zs/Y is NULL");
    if (needs_tv && !Tv) return check(false, "Tv (t, k or b) is required for this score");
    if (score == GNN_SCORE_GENE && !Wa) return check(false, "Wa is required for Gene-linear");
    if (ldz < F + extra) return check(false, "ldz too small for [z | score columns]");
    if (needs_tv && ldt < tv_w) return check(false, "ldt too small");
    if (score == GNN_SCORE_SYM_GAT && p->n != p->n_src) return check(false, "Sym-GAT needs a square plan");
    const int32_t width = head_mean ? Fh : F;
    if (ldy < width) return check(false, "ldy too small");
    if (overlaps(Zs, span_bytes(p->n_src, ldz, F + extra), Y, span_bytes(p->n, ldy, width)))
      return check(false, "Zs and Y overlap");
    size_t head = 0;
    float *Yf = Y;
    int64_t ldf = ldy;
    if (head_mean) {
      head = align256(sizeof(float) * (size_t)p->n * (size_t)F);
      Yf = (float *)ws;
      ldf = F;
    }
    const size_t need = head + agg_workspace_bytes(p, 4, F, H);  // Sym-GAT (2H keys) bounds every score
    if (!ws || ws_bytes < need) {
      set_error("workspace too small: need " + std::to_string(need));
      return GNN_ERR_WORKSPACE;
    }
    static const int kMode[5] = {3, 4, 5, 6, 7};
    AggArgs a{};
    a.mode = kMode[score];
    a.X = Zs;
    a.ldx = ldz;
    a.F = F;
    a.Y = Yf;
    a.ldy = ldf;
    a.t = score == GNN_SCORE_GAT ? Tv : nullptr;
    a.ldt = ldt;
    a.kb = (score == GNN_SCORE_GAAN || score == GNN_SCORE_GENE) ? Tv : nullptr;
    a.ldk = ldt;
    a.Wa = Wa;
    a.H = H;
    a.Fh = Fh;
    a.slope = neg_slope;
    gnn_status st = agg_common(p, a, (char *)ws + head, ws_bytes - head, stream);
    if (st != GNN_OK || !head_mean) return st;
    return cuda_status(launch_head_mean(Yf, ldf, p->n, H, Fh, Y, ldy, (cudaStream_t)stream), "head mean");
  })
}


}  // extern "C"
