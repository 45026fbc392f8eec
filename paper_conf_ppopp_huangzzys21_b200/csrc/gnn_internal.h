// gnn_internal.h — private declarations of libgnn.so (never installed).
// The public boundary is include/gnn.h.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#include <mutex>
#include <string>
#include <vector>

#include "../../include/gnn.h"

#ifdef __CUDACC__
namespace gnn {
// Blackwell packed fp32 FMA (FFMA2): (a0, a1) = (x0, x1) * s + (a0, a1), each
// lane rounded once exactly like fmaf, so chains stay bit-identical; one
// instruction for two FMAs (ptxas folds the broadcast of s into the operand)
__device__ __forceinline__ void fma2_bcast(float &a0, float &a1, float x0, float x1, float s) {
  unsigned long long acc, xx, ss;
  asm("mov.b64 %0, {%1, %2};" : "=l"(acc) : "f"(a0), "f"(a1));
  asm("mov.b64 %0, {%1, %2};" : "=l"(xx) : "f"(x0), "f"(x1));
  asm("mov.b64 %0, {%1, %1};" : "=l"(ss) : "f"(s));
  asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(acc) : "l"(xx), "l"(ss));
  asm("mov.b64 {%0, %1}, %2;" : "=f"(a0), "=f"(a1) : "l"(acc));
}
}  // namespace gnn
#endif

namespace gnn {

// Device-side view of a plan handed to the graph kernels (all int32: the
// plan rejects nnz >= 2^31).
struct DevGraph {
  const int32_t *rowptr;        // [n+1]
  const int32_t *colidx;        // [nnz] CSR order
  const float *nsrc;            // [n_src] 1/sqrtf(d_out)
  const float *ndst;            // [n]     1/sqrtf(d_in)
  const int4 *unit_desc;        // [n_units+1] work units in task order: {tpos, beg, row, m}
                                //   tpos = offset in colidx_t, beg = CSR offset of the unit's first entry,
                                //   m = long-row index (-1: the unit is the whole row); [n_units] = {nnz,0,0,-1}
  const int32_t *colidx_t;      // [nnz + 16] source indices in task order
  const int32_t *multi_slot;    // [n_multi] workspace slot of a long row's first group
  const int32_t *multi_units;   // [n_multi] number of units of a long row
  const int32_t *multi_row;     // [n_multi] row id of each split row
  const int32_t *empty_rows;    // [n_empty]
  const int32_t *perm;          // [n] task (LAS) order of the rows
  int32_t n_units, n_multi, n_empty, ng;
};

}  // namespace gnn

struct gnn_plan_s {
  int device = 0;
  int64_t n = 0, n_src = 0, nnz = 0;
  gnn_plan_opts opts{};
  int32_t ng = 0;      // effective group bound (INT32_MAX-ish when "never split")
  int32_t T = 32;
  int32_t max_degree = 0;
  // host copies
  const int32_t *colidx_h = nullptr;  // caller's array, valid only during gnn_plan_create
  std::vector<int64_t> rowptr;
  std::vector<int32_t> perm, grp_row;
  std::vector<int64_t> grp_beg;
  std::vector<uint64_t> sig;
  std::vector<int32_t> pairs, cluster_of;
  int64_t n_clusters = 0, n_multi = 0, n_empty = 0, multi_slots = 0, max_tile_edges = 0;
  gnn_plan_info info{};
  // device allocations (owned); sched_allocs = the NG schedule (rebuilt by
  // gnn_plan_set_group_size)
  std::vector<void *> dev_allocs;
  std::vector<void *> sched_allocs;
  // per-plan a4 mapping chosen by gnn_tune_aggregate for width tuned_F
  // (tuned_vec == 0: none)
  int32_t tuned_F = 0, tuned_vec = 0, tuned_lanes = 0, tuned_nv = 0;
  gnn::DevGraph dg{};
  const int32_t *d_dout = nullptr;  // device source out-degrees (counted or the override)
  // hot source rows (the highest out-degrees, in degree order) whose L2 lines
  // an aggregation marks evict_last for its duration (k_graph.cu); built on
  // first use from d_dout, freed with the plan
  mutable std::once_flag hot_once;
  mutable int32_t *d_hot = nullptr;
  mutable int32_t n_hot = 0;
};

namespace gnn {

// error plumbing (api.cpp)
void set_error(const std::string &msg);
gnn_status cuda_status(cudaError_t e, const char *what);
void count_launch(uint64_t k = 1);

gnn_status create_plan(int64_t n, int64_t n_src, int64_t nnz, const int64_t *rowptr_h, const int32_t *colidx_h,
                       const int32_t *src_degree_h, const int32_t *perm_h, const gnn_plan_opts *opts_in,
                       gnn_plan_t *out);

// planner (plan.cpp) — host side
gnn_status build_schedule(gnn_plan_s *p);
void schedule_host(int64_t n, const int64_t *rowptr, const int32_t *perm, int64_t ng,
                   std::vector<int32_t> &grp_row, std::vector<int64_t> &grp_beg);
int64_t las_lsh_pairs(int64_t n, const int64_t *rowptr, const uint64_t *sig, int32_t K, int32_t r,
                      int32_t W, std::vector<int32_t> &pairs);
int64_t las_merge(int64_t n, const uint64_t *sig, int32_t K, const std::vector<int32_t> &pairs,
                  int32_t cap, int32_t min_sim, int32_t cluster_order, std::vector<int32_t> &perm,
                  std::vector<int32_t> &cluster_of);

// kernels (k_graph.cu)
cudaError_t launch_degrees(const int32_t *rowptr, const int32_t *colidx, int64_t n, int64_t n_src,
                           int64_t nnz, const int32_t *src_degree_override, int32_t *d_out_tmp,
                           float *nsrc, float *ndst, cudaStream_t s);
cudaError_t launch_minhash(const int32_t *rowptr, const int32_t *colidx, int64_t n, int32_t K,
                           uint64_t seed, uint64_t *sig, cudaStream_t s);

struct AggArgs {
  int mode;            // 0 sum, 1 mean, 2 max, 3 gat, 4 sym-gat, 5 linear, 6 gaan, 7 gene-linear
  int weight;          // gnn_weight (sum/mean/max)
  const float *edge_w;
  const float *X;
  int64_t ldx;
  int32_t F;
  float *Y;
  int64_t ldy;
  const float *add_row;
  int64_t ld_add;
  int32_t relu;
  // GAT
  const float *t;
  int64_t ldt;
  int32_t H, Fh;
  float slope;
  // GaAN k / Gene b per destination row, Gene W_a
  const float *kb;
  int64_t ldk;
  const float *Wa;
  // split-row workspace
  float *ws_part;
  int32_t *ws_cnt;
  int32_t deterministic;
  int32_t accum;  // Y += sums (gnn_aggregate_accumulate)
};
// NEXT-3 GraphSAGE-LSTM (k_lstm.cu)
cudaError_t launch_sample_neighbors(const gnn_plan_s *p, int32_t T, uint64_t seed, int32_t *table, cudaStream_t s);
cudaError_t launch_lstm_weights(const float *W_ih, const float *b_ih, const float *b_hh, const float *W_self,
                                const float *bias, int32_t f_in, int32_t F, int32_t F_out, float *Wcat,
                                float *bcat, cudaStream_t s);
cudaError_t launch_sage_lstm(const gnn_plan_s *p, const int32_t *table, int32_t T, const float *GS, int64_t ldg,
                             const float *R, const float *Wn, int32_t F_out, float *Y, int64_t ldy, cudaStream_t s);
bool set_agg_mapping(int32_t vec, int32_t lanes, int32_t nv);
bool mapping_supported(int32_t vec, int32_t lanes, int32_t nv);
bool agg_override_active();
void set_agg_trace(void *dev_buf);
bool agg_mapping_ok(const AggArgs &a, int32_t fh_or_0, int32_t vec, int32_t lanes, int32_t nv);
gnn_status rebuild_schedule(gnn_plan_s *p, int64_t group_size);
int64_t default_group_size(int64_t n, int64_t nnz);
size_t agg_workspace_bytes(const gnn_plan_s *p, int mode, int32_t F, int32_t H);
cudaError_t launch_scale_rows(float *Y, int64_t ldy, int64_t n, int32_t F, const float *scale, int32_t relu,
                              cudaStream_t s);
cudaError_t launch_head_mean(const float *Yf, int64_t ldf, int64_t n, int32_t H, int32_t Fh, float *Y, int64_t ldy,
                             cudaStream_t s);
gnn_status launch_aggregate(const gnn_plan_s *p, const AggArgs &a, void *ws, size_t ws_bytes,
                            cudaStream_t s);

// GEMM (k_gemm.cu)
// Mirrors (NEXT-2): extra destinations with the output's layout (ldh, rows,
// columns) -- the same rows of peer GPUs' replica buffers -- that the tcgen05
// epilogue writes with the same TMA stores as H (all-gather fused into the
// producer).  Only the TMA-store epilogue takes them.
constexpr int kMaxMirrors = 7;
struct GemmMirrors {
  float *dst[kMaxMirrors];
  int32_t count;
};
gnn_status launch_gemm(const float *X, int64_t ldx, const float *W, int64_t ldw, float *H,
                       int64_t ldh, int64_t m, int32_t k, int32_t n, const float *row_scale,
                       const float *col_bias, int32_t relu, void *ws, size_t ws_bytes, cudaStream_t s,
                       const GemmMirrors *mir = nullptr);
size_t gemm_tc_workspace(int64_t m, int32_t k, int32_t n);
cudaError_t launch_gemm_att(const float *X, int64_t ldx, const float *W, int64_t ldw, float *Z, int64_t ldz, int64_t m,
                            int32_t k, int32_t H, int32_t Fh, const float *a_src, const float *a_dst, void *ws,
                            size_t ws_bytes, cudaStream_t s, const GemmMirrors *mir = nullptr);
int set_gemm_impl(int impl);

// small helper kernels (k_graph.cu)
cudaError_t launch_gat_weights(const float *W, const float *a_src, const float *a_dst, int32_t f_in,
                               int32_t H, int32_t Fh, float *Wext, int32_t ldwe, cudaStream_t s);
cudaError_t launch_edgeconv_weights(const float *theta, const float *phi, const float *bias,
                                    int32_t f_in, int32_t f_out, float *Wpq, float *bpq,
                                    cudaStream_t s);

}  // namespace gnn
