// k_agg.cuh — the aggregation kernel family (a6/a7/a8/a9) of libgnn.so:
// device templates and launch templates, instantiated per reducer in
// k_agg_sum.cu / k_agg_max.cu / k_agg_gat.cu (parallel compilation).
//
// Paper: Huang et al., PPoPP'21 (PAPER.md P:<line>).  Design: DESIGN.md §5.
#pragma once
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>
#include <stdlib.h>

#include <algorithm>
#include <type_traits>

#include "gnn_internal.h"

namespace gnn {

// ---------------------------------------------------------------------------
// a6/a7/a8/a9: the aggregation kernel family.
//
// Mapping (a4, feature-length-adaptive): a "worker"
// is LANES consecutive lanes (LANES in {4, 8, 16, 32}); each lane owns NV
// vectors of VEC consecutive features (VEC in {1,2,4,8}; VEC = 8 is one
// 256-bit LDG per lane).  Chunk width CW = LANES*VEC*NV features; wider rows
// loop over chunks.  A persistent grid of workers claims work units (one
// neighbour group each) in task (LAS) order from one atomic
// counter per feature chunk.
//
// Per group: indices are loaded LANES at a time (one coalesced load), then
// broadcast with sub-warp shuffles; U source rows are in flight per worker
// (register kernel) or S rows in a per-warp shared-memory ring (cp.async
// chain).  Group partial = sequential fp32 chain in CSR order (reading R9).
// Single-group rows finish in the worker (epilogue + store).  The groups of
// a longer row write their partials to the workspace; the last to arrive
// (per-row arrival counter) merges them in group order (P:885-894 with a
// fixed order) and applies the postponed epilogue (linear property,
// P:970-986).  The atomic variant adds the partials into one accumulator row.
// ---------------------------------------------------------------------------
enum { M_SUM = 0, M_MEAN = 1, M_MAX = 2, M_GAT = 3, M_SYM = 4, M_LIN = 5, M_GAAN = 6, M_GENE = 7 };
// attention modes (softmax aggregation of Table 1 with a Table 2 score, R9/R14)
__host__ __device__ constexpr bool is_att(int mode) { return mode >= M_GAT; }
// scores that are an Fh-vector product per head (GaAN, Gene-linear)
__host__ __device__ constexpr bool vec_score(int mode) { return mode == M_GAAN || mode == M_GENE; }
// internal weight code: weight 1 inside the loop, x ndst[v] in the epilogue
// (transform-first GCN whose GEMM epilogue already applied nsrc[u])
constexpr int W_DST_ONLY = 3;
__device__ __forceinline__ bool scales_dst(int w) { return w == GNN_W_GCN || w == W_DST_ONLY; }

struct KParams {
  DevGraph g;
  int mode, weight;
  const float *edge_w;
  const float *X;
  int64_t ldx;
  int32_t F;
  float *Y;
  int64_t ldy;
  const float *add_row;
  int64_t ld_add;
  int32_t relu;
  const float *t;
  int64_t ldt;
  int32_t H, Fh;
  float slope;
  const uint32_t *smax;  // attention: order-encoded source maxima (k_score_max): [H] s (GAT, Linear),
                         // [2H] s then t (Sym-GAT), [H] |q_u[h]| (GaAN)
  const float *kb;       // GaAN k / Gene b: [n, ldk] per destination row
  int64_t ldk;
  const float *Wa;       // Gene: [H, Fh]
  int32_t *ws_unit;  // work-unit counters (one per feature chunk), zeroed per call
  int32_t n_unit_ctr; // number of unit counters (>= feature chunks of any mapping)
  float *ws_acc;   // [n_multi][FW] atomic accumulators (deterministic == 0): sum / max keys / GAT a | l
  float *ws_rowmax;  // [n_multi][H] GAT, deterministic == 0: exact row maxima of the scores (pre-pass)
  float *ws_part;  // [multi slots][FW] per-group partials (deterministic)
  int32_t *ws_cnt; // [n_multi][nch] arrival counters
  int32_t FW;      // partial slot width: F (+ 2 nmeta for attention), rounded to 8
  int32_t nmeta;   // attention: (m, l) entries per slot = H + max chunks; entry of (chunk ci, head h) = h + ci
  int32_t deterministic;
  int32_t accum;      // 1: Y += this call's sums (source-block accumulation, NEXT-2); rows without
                      // entries keep their value
  int32_t nch;        // feature chunks per row (arrival counters per multi-unit row)
  int32_t n_persist;  // persistent CTAs
  // load-balance trace (Fig 8 analogue), nullable: [0] sum of
  // worker busy ns, [1] workers, [2] earliest worker start, [3] latest worker
  // end (%globaltimer ns), [4] units, [5] longest worker busy ns
  unsigned long long *trace;
};

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

// Cache policy of the three streams (A/B switches, compile time):
//   GNN_LD_NA  gathered source rows bypass L1 allocation (L1 keeps the
//              kernel's local memory; the rows are reused through L2)
//   GNN_EF     the task-ordered index stream is loaded and the output rows are
//              stored evict-first (.cs), so they do not push the reused
//              source rows out of L2
#ifndef GNN_LD_NA
#define GNN_LD_NA 1
#endif
#ifndef GNN_EF
#define GNN_EF 1
#endif
#if GNN_LD_NA
#define GNN_LDNC "ld.global.nc.L1::no_allocate"
#else
#define GNN_LDNC "ld.global.nc"
#endif
template <int VEC>
__device__ __forceinline__ void ldv(const float *p, float (&v)[VEC]) {
  if constexpr (VEC == 8) {
    asm volatile(GNN_LDNC ".v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]), "=f"(v[6]),
                   "=f"(v[7])
                 : "l"(p));
  } else if constexpr (VEC == 4) {
    asm volatile(GNN_LDNC ".v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]) : "l"(p));
  } else if constexpr (VEC == 2) {
    asm volatile(GNN_LDNC ".v2.f32 {%0,%1}, [%2];" : "=f"(v[0]), "=f"(v[1]) : "l"(p));
  } else {
    asm volatile(GNN_LDNC ".f32 %0, [%1];" : "=f"(v[0]) : "l"(p));
  }
}

template <int VEC>
__device__ __forceinline__ void stv(float *p, const float (&v)[VEC]) {
  if constexpr (VEC == 8) {
    asm volatile("st.global.v8.f32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "f"(v[0]), "f"(v[1]),
                 "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]), "f"(v[7])
                 : "memory");
  } else if constexpr (VEC == 4) {
    *reinterpret_cast<float4 *>(p) = make_float4(v[0], v[1], v[2], v[3]);
  } else if constexpr (VEC == 2) {
    *reinterpret_cast<float2 *>(p) = make_float2(v[0], v[1]);
  } else {
    p[0] = v[0];
  }
}

// output rows: written once, read by the next kernel (evict-first in L2, GNN_EF)
template <int VEC>
__device__ __forceinline__ void stv_out(float *p, const float (&v)[VEC]) {
#if GNN_EF
  if constexpr (VEC == 8) {
    asm volatile("st.global.cs.v8.f32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "f"(v[0]), "f"(v[1]),
                 "f"(v[2]), "f"(v[3]), "f"(v[4]), "f"(v[5]), "f"(v[6]), "f"(v[7])
                 : "memory");
  } else if constexpr (VEC == 4) {
    asm volatile("st.global.cs.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p), "f"(v[0]), "f"(v[1]), "f"(v[2]), "f"(v[3])
                 : "memory");
  } else if constexpr (VEC == 2) {
    asm volatile("st.global.cs.v2.f32 [%0], {%1,%2};" ::"l"(p), "f"(v[0]), "f"(v[1]) : "memory");
  } else {
    asm volatile("st.global.cs.f32 [%0], %1;" ::"l"(p), "f"(v[0]) : "memory");
  }
#else
  stv<VEC>(p, v);
#endif
}

// streaming index load: read once, do not keep in L1
__device__ __forceinline__ int32_t ld_stream_i32(const int32_t *p) {
  int32_t r;
#if GNN_EF
  asm volatile("ld.global.cs.nc.s32 %0, [%1];" : "=r"(r) : "l"(p));  // evict-first in L2
#else
  asm volatile("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(r) : "l"(p));
#endif
  return r;
}
__device__ __forceinline__ float ld_stream_f32(const float *p) {
  float r;
  asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(r) : "l"(p));
  return r;
}

// a[i] = fmaf(s, x[i], a[i]) for i < VEC, as packed FFMA2 pairs (bit-identical)
template <int VEC>
__device__ __forceinline__ void fma_vec(float (&a)[VEC], const float (&x)[VEC], float s) {
  if constexpr (VEC % 2 == 0) {
#pragma unroll
    for (int i = 0; i < VEC; i += 2) fma2_bcast(a[i], a[i + 1], x[i], x[i + 1], s);
  } else {
#pragma unroll
    for (int i = 0; i < VEC; ++i) a[i] = fmaf(s, x[i], a[i]);
  }
}

// fixed ReLU: y > 0 ? y : +0 (matches the oracle replica, R9)
__device__ __forceinline__ float relu_f(float y) { return y > 0.0f ? y : 0.0f; }

// LeakyReLU (Table 2 GAT) as one min/max: for slope <= 1,
// max(x, slope*x) is x for x >= 0 and slope*x below 0 (min for slope > 1)
__device__ __forceinline__ float leaky_f(float x, float slope) {
  return slope <= 1.0f ? fmaxf(x, slope * x) : fminf(x, slope * x);
}
__device__ __forceinline__ float ex2_f(float x) {
  float r;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
// order-preserving float <-> uint32 key (atomicMax on floats, exact)
__device__ __forceinline__ uint32_t fkey(float f) {
  const uint32_t b = __float_as_uint(f);
  return (b & 0x80000000u) ? ~b : (b | 0x80000000u);
}
__device__ __forceinline__ float fkey_decode(uint32_t k) {
  return __uint_as_float((k & 0x80000000u) ? (k & 0x7fffffffu) : ~k);
}
constexpr float kLog2e = 1.4426950408889634f;
// GAT softmax shift (reading R9 GAT): a group is accumulated against the
// reference m = LeakyReLU(max_u s_u[h] + t_v[h]), an upper bound of every
// score of the row (LeakyReLU and rounding are monotone), so each term is
// exp(e - m) <= 1 and there is no per-edge rescaling.  If the bound is
// looser than kGatSlack for some head (exp(-kGatSlack) keeps all terms
// normal) the group is recomputed against its own exact max.
constexpr float kGatSlack = 32.0f;

template <int MODE, int VEC, int NV>
struct Part {
  float a[NV][VEC];
  float m[NV];  // GAT running max
  float l[NV];  // GAT running sum
};

template <int MODE, int VEC, int NV>
__device__ __forceinline__ void part_init(Part<MODE, VEC, NV> &P) {
#pragma unroll
  for (int n = 0; n < NV; ++n) {
#pragma unroll
    for (int i = 0; i < VEC; ++i) P.a[n][i] = (MODE == M_MAX) ? -INFINITY : 0.0f;
    P.m[n] = -INFINITY;
    P.l[n] = 0.0f;
  }
}

// (m1,l1,a1) <- (m1,l1,a1) (+) (m2,l2,a2): online-softmax merge, fixed form.
__device__ __forceinline__ void gat_merge(float &m1, float &l1, float *a1, float m2, float l2,
                                          const float *a2, int cnt) {
  const float m = fmaxf(m1, m2);
  const float c1 = __expf(m1 - m), c2 = __expf(m2 - m);
  l1 = fmaf(l2, c2, l1 * c1);
  for (int i = 0; i < cnt; ++i) a1[i] = fmaf(a2[i], c2, a1[i] * c1);
  m1 = m;
}

// combine partial B into A (A = A (+) B) in fixed form
template <int MODE, int VEC, int NV>
__device__ __forceinline__ void part_combine(Part<MODE, VEC, NV> &A, const Part<MODE, VEC, NV> &B) {
#pragma unroll
  for (int n = 0; n < NV; ++n) {
    if constexpr (is_att(MODE)) {
      gat_merge(A.m[n], A.l[n], A.a[n], B.m[n], B.l[n], B.a[n], VEC);
    } else {
#pragma unroll
      for (int i = 0; i < VEC; ++i)
        A.a[n][i] = (MODE == M_MAX) ? fmaxf(A.a[n][i], B.a[n][i]) : A.a[n][i] + B.a[n][i];
    }
  }
}

// epilogue on one value (linear property: normalisation postponed)
__device__ __forceinline__ float epi(const KParams &p, int mode, float a, float l, float ndst,
                                     float deg_f, const float *addp) {
  float y;
  if (is_att(mode)) {
    y = a / l;
  } else {
    y = a;
    if (scales_dst(p.weight)) y = y * ndst;
    if (mode == M_MEAN) y = y / deg_f;
    if (addp) y = y + *addp;
  }
  if (p.relu) y = relu_f(y);
  return y;
}

// load VEC floats from L2 (bypassing L1: data written by other SMs in this launch)
template <int VEC>
__device__ __forceinline__ void ldv_cg(const float *p, float (&v)[VEC]) {
  if constexpr (VEC == 8) {
    const float4 a = __ldcg(reinterpret_cast<const float4 *>(p));
    const float4 b = __ldcg(reinterpret_cast<const float4 *>(p) + 1);
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w; v[4] = b.x; v[5] = b.y; v[6] = b.z; v[7] = b.w;
  } else if constexpr (VEC == 4) {
    const float4 a = __ldcg(reinterpret_cast<const float4 *>(p));
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
  } else if constexpr (VEC == 2) {
    const float2 a = __ldcg(reinterpret_cast<const float2 *>(p));
    v[0] = a.x; v[1] = a.y;
  } else {
    v[0] = __ldcg(p);
  }
}

template <int MODE, int VEC, int NV, int LANES>
__device__ __forceinline__ void store_row(const KParams &p, int32_t row, int32_t deg, int32_t c0,
                                          int lane, const Part<MODE, VEC, NV> &P, const float *ndst_pre = nullptr) {
  const float ndst =
      (!is_att(MODE) && scales_dst(p.weight)) ? (ndst_pre ? *ndst_pre : __ldg(p.g.ndst + row)) : 1.0f;
  const float deg_f = (float)deg;
#pragma unroll
  for (int n = 0; n < NV; ++n) {
    const int32_t f = c0 + (n * LANES + lane) * VEC;
    if (f >= p.F) continue;
    float y[VEC];
    float addv[VEC];
    if (p.add_row) ldv<VEC>(p.add_row + (int64_t)row * p.ld_add + f, addv);
#pragma unroll
    for (int i = 0; i < VEC; ++i) y[i] = epi(p, p.mode, P.a[n][i], P.l[n], ndst, deg_f, p.add_row ? &addv[i] : nullptr);
    if (p.accum) {  // raw sums only (validated by gnn_aggregate_accumulate): y = y_old + this block's sum
      float old[VEC];
      ldv_cg<VEC>(p.Y + (int64_t)row * p.ldy + f, old);
#pragma unroll
      for (int i = 0; i < VEC; ++i) y[i] = old[i] + y[i];
    }
    stv_out<VEC>(p.Y + (int64_t)row * p.ldy + f, y);
  }
}


// ---------------------------------------------------------------------------
// v8 work distribution (measured: scripts/stream_bench_k.cu): persistent
// workers grab work units in task (LAS) order through one atomic counter, so
// the units in flight across the GPU are consecutive in the schedule and share
// their source rows in L2; load balance is dynamic (NG's goal,
// P:855-884) with no CTA barrier.  A unit is a whole row (<= R groups) or an
// R-group slice of a longer row; its source indices are read from the
// task-ordered colidx_t (one contiguous stream per unit).
// ---------------------------------------------------------------------------

// fast tanh for the Linear / Gene-linear scores: 1 - 2 / (e^{2x} + 1), in [-1, 1]
__device__ __forceinline__ float tanh_fast(float x) { return 1.0f - __fdividef(2.0f, __expf(2.0f * x) + 1.0f); }

// sum over the LPH lanes of one head (LPH a power of two, aligned segments);
// the butterfly leaves the same value in every lane of the segment
template <int LANES>
__device__ __forceinline__ float head_sum(float x, int lph, unsigned mask) {
  for (int off = 1; off < lph; off <<= 1) x += __shfl_xor_sync(mask, x, off, LANES);
  return x;
}

// one neighbour group: fresh fp32 chain in CSR order (R9); indices from the
// task-ordered stream, LANES at a time, U source rows in flight per worker
// (sum / mean / max and GAT)
#ifndef GNN_GAT_U
#define GNN_GAT_U 0  // 0: the GAT chain keeps the generic rows-in-flight rule
#endif
template <int MODE, int VEC, int NV, int LANES>
__device__ __forceinline__ void group_chain(const KParams &p, const int32_t *idx, int32_t len, int32_t beg,
                                            int32_t row, int32_t c0, int lane, unsigned mask,
                                            Part<MODE, VEC, NV> &G, int32_t m = -1) {
  constexpr int FPL = VEC * NV;
  constexpr int U0 = FPL >= 32 ? 1 : (32 / FPL > 8 ? 8 : 32 / FPL);
  // rows in flight per worker; GAT may take fewer (GNN_GAT_U) to stay in registers
  constexpr int U = (MODE == M_GAT && GNN_GAT_U > 0 && GNN_GAT_U < U0) ? GNN_GAT_U : U0;
  part_init(G);
  const int weight = p.weight;
  const float *xl = p.X + c0 + lane * VEC;
  bool valid[NV];
  int32_t head[NV];
  float tv[NV];
  float nmb[NV];   // GAT: -m * log2(e) for the current reference m
  float seen[NV];  // GAT: exact max score of the group
  // GAT, atomic variant (deterministic == 0) on a split row: every group of the
  // row uses the row's exact score maximum from the pre-pass, so their (a, l)
  // partials can be added with atomics; never loose
  const bool rowmax = MODE == M_GAT && !p.deterministic && m >= 0;
  // GAT: a one-edge group takes its own score as reference (term = 1 exactly)
  const bool one = MODE == M_GAT && len == 1 && !rowmax;
#pragma unroll
  for (int n = 0; n < NV; ++n) {
    const int32_t f = c0 + (n * LANES + lane) * VEC;
    valid[n] = f < p.F;
    head[n] = 0;
    tv[n] = 0.0f;
    nmb[n] = 0.0f;
    seen[n] = -INFINITY;
    if constexpr (MODE == M_GAT) {
      head[n] = valid[n] ? f / p.Fh : 0;
      tv[n] = valid[n] ? __ldg(p.t + (int64_t)row * p.ldt + head[n]) : 0.0f;
      const float mb = !valid[n] ? 0.0f
                       : rowmax  ? __ldcg(p.ws_rowmax + (size_t)m * p.H + head[n])
                                 : leaky_f(fkey_decode(__ldg(p.smax + head[n])) + tv[n], p.slope);
      G.m[n] = mb;
      nmb[n] = -mb * kLog2e;
    }
  }
  // index batches: the next batch (and its weights) is requested before the
  // current one is consumed
  auto load_batch = [&](int32_t k, int32_t &u, float &w) {
    const int32_t c = min(LANES, len - k);
    u = 0;
    w = 1.0f;
    if (lane < c) {
      u = ld_stream_i32(idx + k + lane);
      if constexpr (MODE != M_GAT) {
        if (weight == GNN_W_GCN) w = __ldg(p.g.nsrc + u);
        else if (weight == GNN_W_EDGE) w = ld_stream_f32(p.edge_w + beg + k + lane);
      }
    }
  };
#pragma unroll 1
  for (int pass = 0;; ++pass) {
    int32_t nx_u = 0;
    float nx_w = 1.0f;
    if (len > 0) load_batch(0, nx_u, nx_w);
    for (int32_t k = 0; k < len; k += LANES) {
      const int32_t cnt = min(LANES, len - k);
      const int32_t my_u = nx_u;
      const float my_w = nx_w;
      if (k + LANES < len) load_batch(k + LANES, nx_u, nx_w);
      float v[U][NV][VEC];
      float sc[U][NV];
#pragma unroll
      for (int q = 0; q < U; ++q) {
        if (q < cnt) {
          const int32_t u = __shfl_sync(mask, my_u, q, LANES);
#pragma unroll
          for (int n = 0; n < NV; ++n) {
            if (valid[n]) ldv<VEC>(xl + (int64_t)u * p.ldx + n * LANES * VEC, v[q][n]);
            if constexpr (MODE == M_GAT) sc[q][n] = valid[n] ? __ldg(p.X + (int64_t)u * p.ldx + p.F + head[n]) : 0.0f;
          }
        }
      }
      for (int32_t j = 0; j < cnt; j += U) {
#pragma unroll
        for (int q = 0; q < U; ++q) {
          const int32_t e = j + q;
          if (e < cnt) {
            if constexpr (MODE == M_GAT) {
              // e_uv = LeakyReLU(s_u + t_v); term exp(e_uv - m) (one ex2 per edge and head)
#pragma unroll
              for (int n = 0; n < NV; ++n) {
                if (!valid[n]) continue;
                const float sco = leaky_f(sc[q][n] + tv[n], p.slope);
                seen[n] = fmaxf(seen[n], sco);
                const float ex = one ? 1.0f : ex2_f(fmaf(sco, kLog2e, nmb[n]));
                G.l[n] += ex;
                fma_vec<VEC>(G.a[n], v[q][n], ex);
              }
            } else {
              const float w = __shfl_sync(mask, my_w, e, LANES);
#pragma unroll
              for (int n = 0; n < NV; ++n) {
                if (!valid[n]) continue;
                if constexpr (MODE == M_MAX) {
#pragma unroll
                  for (int i = 0; i < VEC; ++i) G.a[n][i] = fmaxf(G.a[n][i], w * v[q][n][i]);
                } else {
                  fma_vec<VEC>(G.a[n], v[q][n], w);
                }
              }
            }
            if (e + U < cnt) {
              const int32_t u = __shfl_sync(mask, my_u, e + U, LANES);
#pragma unroll
              for (int n = 0; n < NV; ++n) {
                if (valid[n]) ldv<VEC>(xl + (int64_t)u * p.ldx + n * LANES * VEC, v[q][n]);
                if constexpr (MODE == M_GAT)
                  sc[q][n] = valid[n] ? __ldg(p.X + (int64_t)u * p.ldx + p.F + head[n]) : 0.0f;
              }
            }
          }
        }
      }
    }
    if constexpr (MODE != M_GAT) {
      break;
    } else {
      if (one) {
#pragma unroll
        for (int n = 0; n < NV; ++n) G.m[n] = seen[n];
        break;
      }
      // bound too loose for some head of this worker: redo against the exact max
      bool loose = false;
#pragma unroll
      for (int n = 0; n < NV; ++n) loose |= valid[n] && !(G.m[n] - seen[n] <= kGatSlack);
      if (pass == 1 || rowmax || !__any_sync(mask, loose)) break;
#pragma unroll
      for (int n = 0; n < NV; ++n) {
        G.m[n] = seen[n];
        nmb[n] = -seen[n] * kLog2e;
        G.l[n] = 0.0f;
#pragma unroll
        for (int i = 0; i < VEC; ++i) G.a[n][i] = 0.0f;
      }
    }
  }
}

// group chain of the Table 2 scores other than GAT (R14; GAT keeps its own
// specialised chain above, which measured 10% faster than this generalised
// one at 8x32).  Attention modes: softmax terms
// exp(e - m) against a per-row upper bound m of the scores (R9 GAT), with an
// exact-max recompute when the bound is loose.
template <int MODE, int VEC, int NV, int LANES>
__device__ __forceinline__ void group_chain_att(const KParams &p, const int32_t *idx, int32_t len, int32_t beg,
                                            int32_t row, int32_t c0, int lane, unsigned mask,
                                            Part<MODE, VEC, NV> &G) {
  constexpr bool ATT = is_att(MODE);
  constexpr bool VS = vec_score(MODE);
  constexpr int FPL = VEC * NV;
  constexpr int U0 = FPL >= 32 ? 1 : (32 / FPL > 8 ? 8 : 32 / FPL);
  constexpr int U = (VS && U0 > 2) ? 2 : U0;
  constexpr int VQ = VS ? VEC : 1;  // per-slot score vector (GaAN q_u / Gene a_u slice)
  part_init(G);
  const int weight = p.weight;
  const float *xl = p.X + c0 + lane * VEC;
  const int lph = VS ? p.Fh / VEC : 1;  // lanes per head
  bool valid[NV];
  int32_t head[NV];
  float tv[NV];     // GAT/Sym: t_v[h]
  float sv[NV];     // Sym: s_v[h]
  float kv[NV][VQ];  // GaAN k_v / Gene b_v slice
  float wa[NV][VQ];  // Gene W_a slice
  float nmb[NV];    // -m * log2(e) for the current reference m
  float seen[NV];   // exact max score of the group
  // a one-edge group takes its own score as reference (term = 1 exactly)
  const bool one = ATT && len == 1;
#pragma unroll
  for (int n = 0; n < NV; ++n) {
    const int32_t f = c0 + (n * LANES + lane) * VEC;
    valid[n] = f < p.F;
    head[n] = 0;
    tv[n] = 0.0f;
    sv[n] = 0.0f;
    nmb[n] = 0.0f;
    seen[n] = -INFINITY;
#pragma unroll
    for (int i = 0; i < VQ; ++i) kv[n][i] = wa[n][i] = 0.0f;
    if constexpr (ATT) {
      head[n] = valid[n] ? f / p.Fh : 0;
      const int h = head[n];
      float mb = 0.0f;
      if constexpr (MODE == M_GAT) {
        tv[n] = valid[n] ? __ldg(p.t + (int64_t)row * p.ldt + h) : 0.0f;
        mb = leaky_f(fkey_decode(__ldg(p.smax + h)) + tv[n], p.slope);
      } else if constexpr (MODE == M_SYM) {
        const float *zv = p.X + (int64_t)row * p.ldx + p.F;
        tv[n] = valid[n] ? __ldg(zv + p.H + h) : 0.0f;
        sv[n] = valid[n] ? __ldg(zv + h) : 0.0f;
        mb = leaky_f(fkey_decode(__ldg(p.smax + h)) + tv[n], p.slope) +
             leaky_f(sv[n] + fkey_decode(__ldg(p.smax + p.H + h)), p.slope);
      } else if constexpr (MODE == M_LIN) {
        mb = 1.0f;  // tanh <= 1
      } else {
        if (valid[n]) {
          ldv<VEC>(p.kb + (int64_t)row * p.ldk + f, kv[n]);
          if constexpr (MODE == M_GENE) ldv<VEC>(p.Wa + f, wa[n]);
        }
        float part = 0.0f;
#pragma unroll
        for (int i = 0; i < VEC; ++i) part = MODE == M_GAAN ? fmaf(kv[n][i], kv[n][i], part) : part + fabsf(wa[n][i]);
        part = head_sum<LANES>(part, lph, mask);
        // GaAN: <q_u, k_v> <= max_u |q_u| |k_v| (Cauchy-Schwarz); Gene: |<W_a, tanh(.)>| <= |W_a|_1
        mb = MODE == M_GAAN ? fkey_decode(__ldg(p.smax + h)) * sqrtf(part) : part;
      }
      if (!valid[n]) mb = 0.0f;
      G.m[n] = mb;
      nmb[n] = -mb * kLog2e;
    }
  }
  // index batches: the next batch (and its weights) is requested before the
  // current one is consumed
  auto load_batch = [&](int32_t k, int32_t &u, float &w) {
    const int32_t c = min(LANES, len - k);
    u = 0;
    w = 1.0f;
    if (lane < c) {
      u = ld_stream_i32(idx + k + lane);
      if constexpr (!ATT) {
        if (weight == GNN_W_GCN) w = __ldg(p.g.nsrc + u);
        else if (weight == GNN_W_EDGE) w = ld_stream_f32(p.edge_w + beg + k + lane);
      }
    }
  };
  // per-slot score inputs of source row u
  auto load_score = [&](int32_t u, int n, float &a, float &b, float (&vq)[VQ]) {
    if constexpr (MODE == M_GAT || MODE == M_LIN) {
      a = valid[n] ? __ldg(p.X + (int64_t)u * p.ldx + p.F + head[n]) : 0.0f;
    } else if constexpr (MODE == M_SYM) {
      a = valid[n] ? __ldg(p.X + (int64_t)u * p.ldx + p.F + head[n]) : 0.0f;
      b = valid[n] ? __ldg(p.X + (int64_t)u * p.ldx + p.F + p.H + head[n]) : 0.0f;
    } else if constexpr (VS) {
      if (valid[n]) ldv<VEC>(xl + (int64_t)u * p.ldx + p.F + n * LANES * VEC, vq);
      else
#pragma unroll
        for (int i = 0; i < VQ; ++i) vq[i] = 0.0f;
    }
  };
#pragma unroll 1
  for (int pass = 0;; ++pass) {
    int32_t nx_u = 0;
    float nx_w = 1.0f;
    if (len > 0) load_batch(0, nx_u, nx_w);
    for (int32_t k = 0; k < len; k += LANES) {
      const int32_t cnt = min(LANES, len - k);
      const int32_t my_u = nx_u;
      const float my_w = nx_w;
      if (k + LANES < len) load_batch(k + LANES, nx_u, nx_w);
      float v[U][NV][VEC];
      float sc[U][NV], sc2[U][NV];
      float vq[U][NV][VQ];
#pragma unroll
      for (int q = 0; q < U; ++q) {
        if (q < cnt) {
          const int32_t u = __shfl_sync(mask, my_u, q, LANES);
#pragma unroll
          for (int n = 0; n < NV; ++n) {
            if (valid[n]) ldv<VEC>(xl + (int64_t)u * p.ldx + n * LANES * VEC, v[q][n]);
            if constexpr (ATT) load_score(u, n, sc[q][n], sc2[q][n], vq[q][n]);
          }
        }
      }
      for (int32_t j = 0; j < cnt; j += U) {
#pragma unroll
        for (int q = 0; q < U; ++q) {
          const int32_t e = j + q;
          if (e < cnt) {
            if constexpr (ATT) {
              // the score e_uv (Table 2), then the term exp(e_uv - m): one ex2 per edge and head
              float sco[NV];
#pragma unroll
              for (int n = 0; n < NV; ++n) {
                if constexpr (MODE == M_GAT) {
                  sco[n] = leaky_f(sc[q][n] + tv[n], p.slope);
                } else if constexpr (MODE == M_SYM) {
                  sco[n] = leaky_f(sc[q][n] + tv[n], p.slope) + leaky_f(sv[n] + sc2[q][n], p.slope);
                } else if constexpr (MODE == M_LIN) {
                  sco[n] = tanh_fast(sc[q][n]);
                } else {
                  float part = 0.0f;
#pragma unroll
                  for (int i = 0; i < VEC; ++i)
                    part = MODE == M_GAAN ? fmaf(vq[q][n][i], kv[n][i], part)
                                          : fmaf(wa[n][i], tanh_fast(vq[q][n][i] + kv[n][i]), part);
                  sco[n] = head_sum<LANES>(part, lph, mask);
                }
              }
#pragma unroll
              for (int n = 0; n < NV; ++n) {
                if (!valid[n]) continue;
                seen[n] = fmaxf(seen[n], sco[n]);
                const float ex = one ? 1.0f : ex2_f(fmaf(sco[n], kLog2e, nmb[n]));
                G.l[n] += ex;
                fma_vec<VEC>(G.a[n], v[q][n], ex);
              }
            } else {
              const float w = __shfl_sync(mask, my_w, e, LANES);
#pragma unroll
              for (int n = 0; n < NV; ++n) {
                if (!valid[n]) continue;
                if constexpr (MODE == M_MAX) {
#pragma unroll
                  for (int i = 0; i < VEC; ++i) G.a[n][i] = fmaxf(G.a[n][i], w * v[q][n][i]);
                } else {
                  fma_vec<VEC>(G.a[n], v[q][n], w);
                }
              }
            }
            if (e + U < cnt) {
              const int32_t u = __shfl_sync(mask, my_u, e + U, LANES);
#pragma unroll
              for (int n = 0; n < NV; ++n) {
                if (valid[n]) ldv<VEC>(xl + (int64_t)u * p.ldx + n * LANES * VEC, v[q][n]);
                if constexpr (ATT) load_score(u, n, sc[q][n], sc2[q][n], vq[q][n]);
              }
            }
          }
        }
      }
    }
    if constexpr (!ATT) {
      break;
    } else {
      if (one) {
#pragma unroll
        for (int n = 0; n < NV; ++n) G.m[n] = seen[n];
        break;
      }
      // bound too loose for some head of this worker: redo against the exact max
      bool loose = false;
#pragma unroll
      for (int n = 0; n < NV; ++n) loose |= valid[n] && !(G.m[n] - seen[n] <= kGatSlack);
      if (pass == 1 || !__any_sync(mask, loose)) break;
#pragma unroll
      for (int n = 0; n < NV; ++n) {
        G.m[n] = seen[n];
        nmb[n] = -seen[n] * kLog2e;
        G.l[n] = 0.0f;
#pragma unroll
        for (int i = 0; i < VEC; ++i) G.a[n][i] = 0.0f;
      }
    }
  }
}

// ---------------------------------------------------------------------------
// cp.async-staged group chain (sum / mean / max with any weight, GAT): the
// source rows of a group stream through a per-warp ring of S shared-memory
// slots with cp.async (LDGSTS, L2 -> shared, bypassing L1 and registers), so
// the bytes in flight are bounded by shared memory rather than registers
// (scripts/gather_roofline.cu on this B200: random 1 KB rows from a 100 MB
// working set 18.6 TB/s vs 10.9 TB/s for register loads; HBM-bound 7.3 TB/s
// either way).  Worker = one warp; lane owns features c0 + n*128 + 4*lane
// (n < NV): the (4, 32, NV) lane mapping, so partials, merge and epilogue
// are shared with the register kernel and results are bit-identical (the
// chain of R9 is per feature, in CSR order).  Every lane copies exactly the
// 16-byte vectors it later reads; per-edge extras (GCN nsrc[u], explicit
// edge weight, GAT scores s_u[h]) are 4-byte copies by lanes 0..H-1 into the
// slot tail and read by all lanes after a __syncwarp.
// ---------------------------------------------------------------------------
__device__ __forceinline__ void cp_async16(uint32_t dst, const void *src) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async4(uint32_t dst, const void *src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(dst), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}
// branch-free forms for the lean chain: a 16-byte copy that zero-fills (reads
// nothing) when src_bytes == 0, and a predicated 4-byte copy
__device__ __forceinline__ void cp_async16_zfill(uint32_t dst, const void *src, uint32_t src_bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(src_bytes) : "memory");
}
__device__ __forceinline__ void cp_async16_if(uint32_t dst, const void *src, uint32_t pred) {
  asm volatile(
      "{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %2, 0;\n\t@q cp.async.cg.shared.global [%0], [%1], 16;\n\t}" ::"r"(dst),
      "l"(src), "r"(pred)
      : "memory");
}
__device__ __forceinline__ void cp_async4_if(uint32_t dst, const void *src, uint32_t pred) {
  asm volatile(
      "{\n\t.reg .pred q;\n\tsetp.ne.b32 q, %2, 0;\n\t@q cp.async.ca.shared.global [%0], [%1], 4;\n\t}" ::"r"(dst),
      "l"(src), "r"(pred)
      : "memory");
}
// slot size in floats: NV*128 features + the extras (H <= 32 GAT scores, or one weight), 16-byte multiple
template <int MODE, int NV>
__host__ __device__ constexpr int cp_slot_floats() {
  return NV * 128 + (MODE == M_GAT ? 32 : 4);
}
// lean chain (sum / mean / max): a slot holds only the row's features of one
// chunk, min(F, NV*128) rounded to 16 bytes (C5 agg1: 400 B instead of 528 B,
// so the ring holds more rows in the same shared memory); lanes past F issue
// no copy and their reads of the next slot's bytes are never stored.  The
// per-CTA allocation is padded by one full-width slot for the last lane's reads.
template <int MODE, int NV>
__host__ __device__ inline int cp_ring_slot(int32_t F) {
  if (MODE == M_GAT) return cp_slot_floats<MODE, NV>();
  const int w = F < NV * 128 ? F : NV * 128;
  return (w + 3) & ~3;
}

// Lean chain for sum / mean / max (no GAT): the per-edge issue is branch-free
// (row copies zero-fill on the lanes past F), the per-edge weights ride in
// registers (one load per lane per 32 edges, one shuffle per edge, instead of
// a 4-byte copy and a shared read per edge) and the ring slots are running
// counters, which cuts the instructions per edge of the F <= 128 gather (C5
// agg1 is issue-bound, not byte-bound).  Same rows, same arithmetic order as
// group_chain_cp.
#ifndef GNN_CP_U
#define GNN_CP_U 4  // edges per cp.async commit group (C5 agg1, same box: U = 1 / 2 / 4 -> 10.1 / 9.5 / 8.5 ms)
#endif
template <int MODE, int NV, int S>
__device__ __forceinline__ void group_chain_cp_lean(const KParams &p, const int32_t *idx, int32_t len, int32_t beg,
                                                    int32_t c0, int lane, float *ring, Part<MODE, 4, NV> &G) {
  constexpr int VEC = 4;
  const int SLOT = cp_ring_slot<MODE, NV>(p.F);
  // U consecutive edges share one commit group, one wait and one pair of
  // warp barriers; the R9 chain still adds them one by one in CSR order
  constexpr int U = (S % GNN_CP_U == 0) ? GNN_CP_U : (S % 2 == 0 ? 2 : 1);
  constexpr int NG = S / U;  // commit groups in flight
  static_assert(MODE != M_GAT, "lean chain: sum / mean / max only");
  static_assert(32 % U == 0 && S <= 32, "U divides the 32-entry index window, S fits it");
  part_init(G);
  const int weight = p.weight;
  const bool has_w = weight == GNN_W_GCN || weight == GNN_W_EDGE;
  const uint32_t ring_s = (uint32_t)__cvta_generic_to_shared(ring);
  uint32_t lv[NV];  // this lane copies vector n (inside F)
#pragma unroll
  for (int n = 0; n < NV; ++n) lv[n] = (c0 + (n * 32 + lane) * VEC < p.F) ? 1u : 0u;
  // row addresses: one IMAD.WIDE.U32 per edge (u unsigned x the row pitch in
  // bytes, cp_admissible: ldx * 4 < 2^32)
  const char *xl = reinterpret_cast<const char *>(p.X + c0 + lane * VEC);
  const uint32_t ldxb = (uint32_t)p.ldx * 4u;
  const uint32_t my_off = (uint32_t)(lane * VEC * 4);
  uint32_t slot_w = ring_s;  // next issue slot (address)
  int slot_i = 0;
  // per-edge weights travel in registers, one 32-edge window per lane set:
  // lane l of `wi` holds the weight of edge 32k + l of the window the issue
  // side is in (GCN: nsrc[u], loaded when the window's indices become current,
  // 32 edges after they were requested; explicit: edge_w[beg + e], coalesced);
  // the consume side takes the window over (`wc`) when it reaches it, at most
  // S edges later, and broadcasts edge e's weight with one shuffle
  auto wload = [&](int32_t e_base, int32_t u_lane) -> float {
    if (!has_w || e_base + lane >= len) return 1.0f;
    return weight == GNN_W_GCN ? __ldg(p.g.nsrc + u_lane) : ld_stream_f32(p.edge_w + beg + e_base + lane);
  };
  int32_t cur = lane < len ? ld_stream_i32(idx + lane) : 0;
  int32_t nxt = 32 + lane < len ? ld_stream_i32(idx + 32 + lane) : 0;
  float wi = wload(0, cur);
  float wc = wi;
  // issue edges e0 .. e0+U-1 (e0 % U == 0) as one commit group; indices from
  // the 32-entry window `cur` (refilled from `nxt` at multiples of 32); a
  // batch wholly inside the group needs no per-edge checks (FULL), the last
  // ones copy nothing for edges past the end
  auto issue = [&](int32_t e0, auto full) {
    if ((e0 & 31) == 0 && e0 >= 32) {
      cur = nxt;
      nxt = e0 + 32 + lane < len ? ld_stream_i32(idx + e0 + 32 + lane) : 0;
      wi = wload(e0, cur);
    }
#pragma unroll
    for (int j = 0; j < U; ++j) {
      const int32_t e = e0 + j;
      const uint32_t u = (uint32_t)__shfl_sync(0xffffffffu, cur, (e0 & 31) + j);
      const uint32_t sw = slot_w + (uint32_t)(j * SLOT * 4);
      const char *src = xl + (uint64_t)u * ldxb;
#pragma unroll
      for (int n = 0; n < NV; ++n) {
        if constexpr (decltype(full)::value)
          cp_async16_if(sw + my_off + (uint32_t)(n * 512), src + n * 512, lv[n]);
        else
          cp_async16_if(sw + my_off + (uint32_t)(n * 512), src + n * 512, e < len ? lv[n] : 0u);
      }
    }
    cp_commit();
    slot_i += U;
    if (slot_i == S) {
      slot_i = 0;
      slot_w = ring_s;
    } else {
      slot_w += (uint32_t)(U * SLOT * 4);
    }
  };
  auto issue_any = [&](int32_t e0) {
    if (e0 + U <= len) issue(e0, std::true_type{});
    else issue(e0, std::false_type{});
  };
#pragma unroll
  for (int q = 0; q < NG; ++q) issue_any(q * U);
  const float *rd = ring;
  int rd_i = 0;
  auto consume = [&](int32_t e0, int j) {
    const float *sl = rd + j * SLOT;
    const float w = has_w ? __shfl_sync(0xffffffffu, wc, (e0 & 31) + j) : 1.0f;
#pragma unroll
    for (int n = 0; n < NV; ++n) {
      const float4 x4 = *reinterpret_cast<const float4 *>(sl + n * 128 + lane * VEC);
      const float v[4] = {x4.x, x4.y, x4.z, x4.w};
      if constexpr (MODE == M_MAX) {
#pragma unroll
        for (int i = 0; i < VEC; ++i) G.a[n][i] = fmaxf(G.a[n][i], w * v[i]);
      } else {
        fma_vec<VEC>(G.a[n], v, w);
      }
    }
  };
  for (int32_t e0 = 0; e0 < len; e0 += U) {
    // the issue side is at most S <= 32 edges ahead, so at a window start it
    // is still inside this window: `wi` holds this window's weights
    if ((e0 & 31) == 0) wc = wi;
    cp_wait<NG - 1>();
    __syncwarp();
    if (e0 + U <= len) {
#pragma unroll
      for (int j = 0; j < U; ++j) consume(e0, j);
    } else {
      for (int j = 0; j < len - e0; ++j) consume(e0, j);
    }
    __syncwarp();  // every lane has read the slots before they are refilled
    rd_i += U;
    if (rd_i == S) {
      rd_i = 0;
      rd = ring;
    } else {
      rd += U * SLOT;
    }
    issue_any(e0 + S);
  }
}

// Lean chain for GAT (same structure as group_chain_cp_lean): U = 4 edges per
// commit group, predicated 16-byte row copies, the H scores s_u[h] of each
// edge by 16-byte copies of lanes 0 .. H/4-1 (4-byte copies when H % 4 != 0)
// into the slot tail; each lane computes e and exp(e - m) for the head of each
// of its vectors (same expression and order as the register and gather4
// kernels: bit-identical).  A group whose softmax bound was too loose for
// some head is streamed a second time against its exact maxima (R9 GAT).
template <int NV, int S>
__device__ __forceinline__ void group_chain_cp_lean_gat(const KParams &p, const int32_t *idx, int32_t len,
                                                        int32_t row, int32_t c0, int lane, float *ring,
                                                        Part<M_GAT, 4, NV> &G) {
  constexpr int VEC = 4;
  constexpr int SLOT = cp_slot_floats<M_GAT, NV>();
  constexpr int U = (S % GNN_CP_U == 0) ? GNN_CP_U : (S % 2 == 0 ? 2 : 1);
  constexpr int NG = S / U;
  static_assert(32 % U == 0 && S <= 32, "U divides the 32-entry index window, S fits it");
  const uint32_t ring_s = (uint32_t)__cvta_generic_to_shared(ring);
  uint32_t lv[NV];
  bool valid[NV];
  int32_t head[NV];
  float tv[NV], nmb[NV], seen[NV];
  const bool one = len == 1;
#pragma unroll
  for (int n = 0; n < NV; ++n) {
    const int32_t f = c0 + (n * 32 + lane) * VEC;
    valid[n] = f < p.F;
    lv[n] = valid[n] ? 1u : 0u;
    head[n] = valid[n] ? f / p.Fh : 0;
    tv[n] = valid[n] ? __ldg(p.t + (int64_t)row * p.ldt + head[n]) : 0.0f;
    const float mb = valid[n] ? leaky_f(fkey_decode(__ldg(p.smax + head[n])) + tv[n], p.slope) : 0.0f;
    G.m[n] = mb;
    nmb[n] = -mb * kLog2e;
  }
  const char *xl = reinterpret_cast<const char *>(p.X + c0 + lane * VEC);
  const char *sxl = reinterpret_cast<const char *>(p.X + p.F);
  const uint32_t ldxb = (uint32_t)p.ldx * 4u;
  const uint32_t my_off = (uint32_t)(lane * VEC * 4);
  const bool s16 = (p.H & 3) == 0;
  const uint32_t sc_lane = s16 ? ((lane < (p.H >> 2)) ? 1u : 0u) : ((lane < p.H) ? 1u : 0u);
  const uint32_t sc_off = s16 ? (uint32_t)(lane * 16) : (uint32_t)(lane * 4);
#pragma unroll 1
  for (int pass = 0;; ++pass) {
#pragma unroll
    for (int n = 0; n < NV; ++n) {
      G.l[n] = 0.0f;
      seen[n] = -INFINITY;
#pragma unroll
      for (int i = 0; i < VEC; ++i) G.a[n][i] = 0.0f;
    }
    uint32_t slot_w = ring_s;
    int slot_i = 0;
    int32_t cur = lane < len ? ld_stream_i32(idx + lane) : 0;
    int32_t nxt = 32 + lane < len ? ld_stream_i32(idx + 32 + lane) : 0;
    auto issue = [&](int32_t e0) {
      if ((e0 & 31) == 0 && e0 >= 32) {
        cur = nxt;
        nxt = e0 + 32 + lane < len ? ld_stream_i32(idx + e0 + 32 + lane) : 0;
      }
#pragma unroll
      for (int j = 0; j < U; ++j) {
        const int32_t e = e0 + j;
        const uint32_t u = (uint32_t)__shfl_sync(0xffffffffu, cur, (e0 & 31) + j);
        const uint32_t sw = slot_w + (uint32_t)(j * SLOT * 4);
        const uint32_t live = e < len ? 1u : 0u;
        const char *src = xl + (uint64_t)u * ldxb;
#pragma unroll
        for (int n = 0; n < NV; ++n) cp_async16_if(sw + my_off + (uint32_t)(n * 512), src + n * 512, live & lv[n]);
        const char *ss = sxl + (uint64_t)u * ldxb + sc_off;
        if (s16) cp_async16_if(sw + (uint32_t)(NV * 512) + sc_off, ss, live & sc_lane);
        else cp_async4_if(sw + (uint32_t)(NV * 512) + sc_off, ss, live & sc_lane);
      }
      cp_commit();
      slot_i += U;
      if (slot_i == S) {
        slot_i = 0;
        slot_w = ring_s;
      } else {
        slot_w += (uint32_t)(U * SLOT * 4);
      }
    };
#pragma unroll
    for (int q = 0; q < NG; ++q) issue(q * U);
    const float *rd = ring;
    int rd_i = 0;
    auto consume = [&](int j) {
      const float *sl = rd + j * SLOT;
#pragma unroll
      for (int n = 0; n < NV; ++n) {
        const float4 x4 = *reinterpret_cast<const float4 *>(sl + n * 128 + lane * VEC);
        const float v[4] = {x4.x, x4.y, x4.z, x4.w};
        const float sco = leaky_f(sl[NV * 128 + head[n]] + tv[n], p.slope);
        seen[n] = fmaxf(seen[n], sco);
        const float ex = one ? 1.0f : ex2_f(fmaf(sco, kLog2e, nmb[n]));
        G.l[n] += ex;
        fma_vec<VEC>(G.a[n], v, ex);
      }
    };
    for (int32_t e0 = 0; e0 < len; e0 += U) {
      cp_wait<NG - 1>();
      __syncwarp();
      if (e0 + U <= len) {
#pragma unroll
        for (int j = 0; j < U; ++j) consume(j);
      } else {
        for (int j = 0; j < len - e0; ++j) consume(j);
      }
      __syncwarp();  // every lane has read the slots before they are refilled
      rd_i += U;
      if (rd_i == S) {
        rd_i = 0;
        rd = ring;
      } else {
        rd += U * SLOT;
      }
      issue(e0 + S);
    }
    cp_wait<0>();  // nothing of this pass is still landing in the ring
    if (one) {
#pragma unroll
      for (int n = 0; n < NV; ++n) G.m[n] = seen[n];
      break;
    }
    // bound too loose for some head of this warp: redo against the exact max (R9 GAT)
    bool loose = false;
#pragma unroll
    for (int n = 0; n < NV; ++n) loose |= valid[n] && !(G.m[n] - seen[n] <= kGatSlack);
    if (pass == 1 || !__any_sync(0xffffffffu, loose)) break;
#pragma unroll
    for (int n = 0; n < NV; ++n) {
      G.m[n] = seen[n];
      nmb[n] = -seen[n] * kLog2e;
    }
    __syncwarp();
  }
}

#ifndef GNN_CP_GAT_LEAN
#define GNN_CP_GAT_LEAN 1  // 0: the per-edge GAT chain below
#endif
template <int MODE, int NV, int S>
__device__ __forceinline__ void group_chain_cp(const KParams &p, const int32_t *idx, int32_t len, int32_t beg,
                                               int32_t row, int32_t c0, int lane, float *ring,
                                               Part<MODE, 4, NV> &G) {
  constexpr int VEC = 4;
  constexpr int SLOT = cp_slot_floats<MODE, NV>();
  if constexpr (MODE != M_GAT) {
#ifndef GNN_CP_LEGACY
    (void)row;
    group_chain_cp_lean<MODE, NV, S>(p, idx, len, beg, c0, lane, ring, G);
    return;
#endif
  } else if constexpr (GNN_CP_GAT_LEAN) {
    (void)beg;
    group_chain_cp_lean_gat<NV, S>(p, idx, len, row, c0, lane, ring, G);
    return;
  }
  part_init(G);
  const int weight = p.weight;
  const uint32_t ring_s = (uint32_t)__cvta_generic_to_shared(ring);
  bool valid[NV];
  int32_t head[NV];
  float tv[NV], nmb[NV], seen[NV];
  const bool one = MODE == M_GAT && len == 1;
#pragma unroll
  for (int n = 0; n < NV; ++n) {
    const int32_t f = c0 + (n * 32 + lane) * VEC;
    valid[n] = f < p.F;
    head[n] = 0;
    tv[n] = 0.0f;
    nmb[n] = 0.0f;
    seen[n] = -INFINITY;
    if constexpr (MODE == M_GAT) {
      head[n] = valid[n] ? f / p.Fh : 0;
      tv[n] = valid[n] ? __ldg(p.t + (int64_t)row * p.ldt + head[n]) : 0.0f;
      const float mb = valid[n] ? leaky_f(fkey_decode(__ldg(p.smax + head[n])) + tv[n], p.slope) : 0.0f;
      G.m[n] = mb;
      nmb[n] = -mb * kLog2e;
    }
  }
  const float *xl = p.X + c0 + lane * VEC;
  // issue the copies of edge e (source row u) into slot e % S; one commit group per edge
  auto issue = [&](int32_t u, int32_t e) {
    const uint32_t sl = ring_s + (uint32_t)((e % S) * SLOT * 4);
    if (e < len) {
#pragma unroll
      for (int n = 0; n < NV; ++n)
        if (valid[n]) cp_async16(sl + (uint32_t)((n * 128 + lane * VEC) * 4), xl + (int64_t)u * p.ldx + n * 128);
      if constexpr (MODE == M_GAT) {
        if (lane < p.H) cp_async4(sl + (uint32_t)((NV * 128 + lane) * 4), p.X + (int64_t)u * p.ldx + p.F + lane);
      } else {
        if (lane == 0) {
          if (weight == GNN_W_GCN) cp_async4(sl + (uint32_t)(NV * 128 * 4), p.g.nsrc + u);
          else if (weight == GNN_W_EDGE) cp_async4(sl + (uint32_t)(NV * 128 * 4), p.edge_w + beg + e);
        }
      }
    }
    cp_commit();
  };
#pragma unroll 1
  for (int pass = 0;; ++pass) {
    int32_t cur = lane < len ? ld_stream_i32(idx + lane) : 0;
    int32_t nxt = 32 + lane < len ? ld_stream_i32(idx + 32 + lane) : 0;
#pragma unroll
    for (int q = 0; q < S; ++q) issue(__shfl_sync(0xffffffffu, cur, q), q);
    for (int32_t e = 0; e < len; ++e) {
      cp_wait<S - 1>();
      __syncwarp();
      const float *sl = ring + (e % S) * SLOT;
      if constexpr (MODE == M_GAT) {
#pragma unroll
        for (int n = 0; n < NV; ++n) {
          if (!valid[n]) continue;
          const float4 x4 = *reinterpret_cast<const float4 *>(sl + n * 128 + lane * VEC);
          const float v[4] = {x4.x, x4.y, x4.z, x4.w};
          const float sco = leaky_f(sl[NV * 128 + head[n]] + tv[n], p.slope);
          seen[n] = fmaxf(seen[n], sco);
          const float ex = one ? 1.0f : ex2_f(fmaf(sco, kLog2e, nmb[n]));
          G.l[n] += ex;
          fma_vec<VEC>(G.a[n], v, ex);
        }
      } else {
        const float w = (weight == GNN_W_GCN || weight == GNN_W_EDGE) ? sl[NV * 128] : 1.0f;
#pragma unroll
        for (int n = 0; n < NV; ++n) {
          if (!valid[n]) continue;
          const float4 x4 = *reinterpret_cast<const float4 *>(sl + n * 128 + lane * VEC);
          const float v[4] = {x4.x, x4.y, x4.z, x4.w};
          if constexpr (MODE == M_MAX) {
#pragma unroll
            for (int i = 0; i < VEC; ++i) G.a[n][i] = fmaxf(G.a[n][i], w * v[i]);
          } else {
            fma_vec<VEC>(G.a[n], v, w);
          }
        }
      }
      __syncwarp();  // every lane has read slot e % S before it is refilled
      const int32_t pe = e + S;
      if ((pe & 31) == 0) {
        cur = nxt;
        nxt = pe + 32 + lane < len ? ld_stream_i32(idx + pe + 32 + lane) : 0;
      }
      issue(__shfl_sync(0xffffffffu, cur, pe & 31), pe);
    }
    if constexpr (MODE != M_GAT) {
      break;
    } else {
      if (one) {
#pragma unroll
        for (int n = 0; n < NV; ++n) G.m[n] = seen[n];
        break;
      }
      // bound too loose for some head of this warp: redo against the exact max (R9 GAT)
      bool loose = false;
#pragma unroll
      for (int n = 0; n < NV; ++n) loose |= valid[n] && !(G.m[n] - seen[n] <= kGatSlack);
      if (pass == 1 || !__any_sync(0xffffffffu, loose)) break;
#pragma unroll
      for (int n = 0; n < NV; ++n) {
        G.m[n] = seen[n];
        nmb[n] = -seen[n] * kLog2e;
        G.l[n] = 0.0f;
#pragma unroll
        for (int i = 0; i < VEC; ++i) G.a[n][i] = 0.0f;
      }
    }
  }
}

// merge the group partials of a long row in group order (R9), epilogue, store
template <int MODE, int VEC, int NV, int LANES>
__device__ __forceinline__ void merge_row(const KParams &p, const float *base, int32_t ngrp, int32_t row,
                                          int32_t deg, int32_t c0, int32_t ci, int lane) {
  Part<MODE, VEC, NV> A;
  part_init(A);
#pragma unroll
  for (int n = 0; n < NV; ++n) {
    const int32_t f = c0 + (n * LANES + lane) * VEC;
    if (f >= p.F) continue;
    for (int32_t q = 0; q < ngrp; ++q) {
      float b[VEC];
      ldv_cg<VEC>(base + (size_t)q * p.FW + f, b);
      if constexpr (is_att(MODE)) {
        const int32_t e = f / p.Fh + ci;  // (chunk, head) entry
        const float bm = __ldcg(base + (size_t)q * p.FW + p.F + e);
        const float bl = __ldcg(base + (size_t)q * p.FW + p.F + p.nmeta + e);
        if (q == 0) {
#pragma unroll
          for (int i = 0; i < VEC; ++i) A.a[n][i] = b[i];
          A.m[n] = bm;
          A.l[n] = bl;
        } else {
          gat_merge(A.m[n], A.l[n], A.a[n], bm, bl, b, VEC);
        }
      } else {
#pragma unroll
        for (int i = 0; i < VEC; ++i)
          A.a[n][i] = (q == 0) ? b[i] : (MODE == M_MAX ? fmaxf(A.a[n][i], b[i]) : A.a[n][i] + b[i]);
      }
    }
  }
  store_row<MODE, VEC, NV, LANES>(p, row, deg, c0, lane, A);
}

// one work unit = one neighbour group (NG: a group is the task of
// one computing unit).  A row with a single group is finished here (epilogue +
// store); the groups of a longer row leave their partials in the workspace and
// the last one to arrive merges them in group order (R9).
template <int MODE, int VEC, int NV, int LANES>
__device__ __forceinline__ void finish_unit(const KParams &p, const Part<MODE, VEC, NV> &G, int32_t row, int32_t beg,
                                            int32_t m, int32_t len, int32_t c0, int32_t ci, int lane, unsigned mask,
                                            const float *ndst_pre);

template <int MODE, int VEC, int NV, int LANES, int S = 0>
__device__ __forceinline__ void process_unit(const KParams &p, int4 d, int32_t len, int32_t c0, int32_t ci, int lane,
                                             unsigned mask, float *ring = nullptr) {
  const DevGraph &g = p.g;
  const int32_t tpos = d.x, beg = d.y, row = d.z, m = d.w;
  Part<MODE, VEC, NV> G;
  if constexpr (S > 0) {
    static_assert(VEC == 4 && LANES == 32 && MODE <= M_GAT, "cp.async chain: (4, 32, NV) mapping");
    group_chain_cp<MODE, NV, S>(p, g.colidx_t + tpos, len, beg, row, c0, lane, ring, G);
  } else if constexpr (MODE > M_GAT)
    group_chain_att<MODE, VEC, NV, LANES>(p, g.colidx_t + tpos, len, beg, row, c0, lane, mask, G);
  else
    group_chain<MODE, VEC, NV, LANES>(p, g.colidx_t + tpos, len, beg, row, c0, lane, mask, G, m);
  finish_unit<MODE, VEC, NV, LANES>(p, G, row, beg, m, len, c0, ci, lane, mask, nullptr);
}

// a finished group: a whole row -> epilogue + store (deg = len); a group of a
// longer row -> its partial to the workspace, the last group to arrive merges
// them in group order (R9)
template <int MODE, int VEC, int NV, int LANES>
__device__ __forceinline__ void finish_unit(const KParams &p, const Part<MODE, VEC, NV> &G, int32_t row, int32_t beg,
                                            int32_t m, int32_t len, int32_t c0, int32_t ci, int lane, unsigned mask,
                                            const float *ndst_pre) {
  const DevGraph &g = p.g;
  if (m < 0) {
    store_row<MODE, VEC, NV, LANES>(p, row, len, c0, lane, G, ndst_pre);
    return;
  }
  const int32_t rb = g.rowptr[row], re = g.rowptr[row + 1];
  const int32_t ng = g.ng;
  const int32_t ngrp = 1 + (re - rb - 1) / ng;
  const int32_t k = (beg - rb) / ng;
  // non-deterministic variant: partials meet in one accumulator row
  // by atomics -- sum / mean: float adds; max: atomicMax on order-preserving
  // keys (exact); GAT: a and l added against the shared exact row maximum
  const bool atomic_acc = !p.deterministic && (MODE == M_SUM || MODE == M_MAX || MODE == M_GAT);
  float *base = p.ws_part + (size_t)g.multi_slot[m] * p.FW;
  float *acc = p.ws_acc + (size_t)m * p.FW;
#pragma unroll
  for (int n = 0; n < NV; ++n) {
    const int32_t f = c0 + (n * LANES + lane) * VEC;
    if (f >= p.F) continue;
    if (atomic_acc) {
      if constexpr (MODE == M_MAX) {
#pragma unroll
        for (int i = 0; i < VEC; ++i) atomicMax(reinterpret_cast<uint32_t *>(acc) + f + i, fkey(G.a[n][i]));
      } else {
#pragma unroll
        for (int i = 0; i < VEC; ++i) atomicAdd(acc + f + i, G.a[n][i]);
        if constexpr (MODE == M_GAT) {
          if (f % p.Fh == 0) atomicAdd(acc + p.F + f / p.Fh, G.l[n]);  // heads never straddle chunks here
        }
      }
    } else {
      stv<VEC>(base + (size_t)k * p.FW + f, G.a[n]);
      if constexpr (is_att(MODE)) {
        // the softmax state of (chunk ci, head h), written by the lane holding
        // the head's first feature in this chunk (a head may straddle chunks;
        // each chunk keeps its own reference and sum)
        if (f % p.Fh == 0 || f == c0) {
          const int32_t e = f / p.Fh + ci;
          base[(size_t)k * p.FW + p.F + e] = G.m[n];
          base[(size_t)k * p.FW + p.F + p.nmeta + e] = G.l[n];
        }
      }
    }
  }
  __threadfence();
  __syncwarp(mask);
  int32_t *cnt = p.ws_cnt + (size_t)m * p.nch + ci;
  int last = 0;
  if (lane == 0) last = atomicAdd(cnt, 1) == ngrp - 1;
  last = __shfl_sync(mask, last, 0, LANES);
  if (!last) return;
  __threadfence();
  if (atomic_acc) {
    Part<MODE, VEC, NV> A;
    part_init(A);
#pragma unroll
    for (int n = 0; n < NV; ++n) {
      const int32_t f = c0 + (n * LANES + lane) * VEC;
      if (f >= p.F) continue;
      ldv_cg<VEC>(acc + f, A.a[n]);
      if constexpr (MODE == M_MAX) {
#pragma unroll
        for (int i = 0; i < VEC; ++i) A.a[n][i] = fkey_decode(__float_as_uint(A.a[n][i]));
      }
      if constexpr (MODE == M_GAT) A.l[n] = __ldcg(acc + p.F + f / p.Fh);
    }
    store_row<MODE, VEC, NV, LANES>(p, row, re - rb, c0, lane, A);
  } else {
    merge_row<MODE, VEC, NV, LANES>(p, base, ngrp, row, re - rb, c0, ci, lane);
  }
  if (lane == 0) *cnt = 0;  // leave the counter at 0 for the next call
}

#ifndef GNN_AGG_MINB
#define GNN_AGG_MINB 4
#endif
#ifndef GNN_AGG_MINB_GAT
#define GNN_AGG_MINB_GAT 4
#endif
#ifndef GNN_AGG_MINB_CP
#define GNN_AGG_MINB_CP 4
#endif
// slots per warp of the cp.async ring (S > 0 selects the cp.async chain)
#ifndef GNN_CP_S1
#define GNN_CP_S1 12  // NV = 1: rows <= 128 features
#endif
#ifndef GNN_CP_S2
#define GNN_CP_S2 8  // NV = 2: rows <= 256 features (C3 F=256 GCN, same box: S = 4 / 6 / 8 / 12 -> 9.7-9.8 / 10.0-10.1 / 9.2-9.5 / 9.65 ms)
#endif
template <int MODE, int VEC, int NV, int LANES, int S = 0>
#ifndef GNN_AGG_MINB_CP2
#define GNN_AGG_MINB_CP2 3  // NV = 2 rings (8 slots of 1 KB per warp) fit 3 CTAs per SM: 80 registers, no spills
#endif
__global__ void __launch_bounds__(256, S > 0 ? (NV >= 2 ? GNN_AGG_MINB_CP2 : GNN_AGG_MINB_CP)
                                             : (vec_score(MODE) ? 2 : (is_att(MODE) ? GNN_AGG_MINB_GAT : GNN_AGG_MINB)))
    k_aggregate(const KParams p) {
  constexpr int CW = LANES * VEC * NV;
  extern __shared__ __align__(16) float cp_smem[];
  const int tid = threadIdx.x;
  const int lane = tid & (LANES - 1);
  const unsigned mask =
      LANES == 32 ? 0xffffffffu : (((1u << LANES) - 1u) << ((tid & 31) & ~(LANES - 1)));
  const DevGraph &g = p.g;
  if ((int32_t)blockIdx.x >= p.n_persist) {
    // zero-fill rows without in-edges (R3-i): 32 rows per block (kept as they are when accumulating)
    if (p.accum) return;
    const int64_t r0 = (int64_t)(blockIdx.x - p.n_persist) * 32;
    for (int64_t r = r0; r < r0 + 32 && r < g.n_empty; ++r) {
      float *y = p.Y + (int64_t)g.empty_rows[r] * p.ldy;
      for (int f = tid; f < p.F; f += blockDim.x) y[f] = 0.0f;
    }
    return;
  }
  const int32_t nunits = g.n_units;
  int32_t ci = 0;
  // load-balance trace state lives in shared memory (one slot per worker), so
  // the untraced kernel carries no extra registers across the unit loop
  __shared__ unsigned long long trace_sh[256 / LANES][3];  // t_unit, busy, n_done
  unsigned long long *const tr = trace_sh[tid / LANES];
  unsigned long long t_start = 0;
  if (p.trace) {
    t_start = gtimer();
    if (lane == 0) tr[1] = tr[2] = 0ull;
  }
  for (int32_t c0 = 0; c0 < p.F; c0 += CW, ++ci) {
    int32_t *ctr = p.ws_unit + ci;
    // the next unit (id and descriptor) is claimed while the current one streams
    int32_t u = 0;
    if (lane == 0) u = atomicAdd(ctr, 1);
    u = __shfl_sync(mask, u, 0, LANES);
    int4 d = make_int4(0, 0, 0, -1);
    int32_t dnx = 0;
    if (u < nunits) {
      d = __ldg(g.unit_desc + u);
      dnx = __ldg(&g.unit_desc[u + 1].x);
    }
    while (u < nunits) {
      if (p.trace && lane == 0) tr[0] = gtimer();
      int32_t un = 0;
      if (lane == 0) un = atomicAdd(ctr, 1);
      un = __shfl_sync(mask, un, 0, LANES);
      int4 dn = make_int4(0, 0, 0, -1);
      int32_t dnxn = 0;
      if (un < nunits) {
        dn = __ldg(g.unit_desc + un);
        dnxn = __ldg(&g.unit_desc[un + 1].x);
      }
      if constexpr (S > 0)
        process_unit<MODE, VEC, NV, LANES, S>(p, d, dnx - d.x, c0, ci, lane, mask,
                                              cp_smem + (tid >> 5) * S * cp_ring_slot<MODE, NV>(p.F));
      else
        process_unit<MODE, VEC, NV, LANES>(p, d, dnx - d.x, c0, ci, lane, mask);
      if (p.trace && lane == 0) {
        tr[1] += gtimer() - tr[0];
        tr[2] += 1ull;
      }
      u = un;
      d = dn;
      dnx = dnxn;
    }
  }
  if (p.trace && lane == 0) {
    const unsigned long long busy = tr[1];
    atomicAdd(p.trace + 0, busy);
    atomicAdd(p.trace + 1, 1ull);
    atomicMin(p.trace + 2, t_start);
    atomicMax(p.trace + 3, gtimer());
    atomicAdd(p.trace + 4, tr[2]);
    atomicMax(p.trace + 5, busy);
  }
}

// GAT, a group whose softmax bound was too loose (R9 GAT): recompute it
// against its exact maximum with direct loads (rare path); 32 lanes, lane's
// vector n at features c0 + (n * 32 + lane) * VEC
template <int VEC, int NV>
__device__ __forceinline__ void gat_recompute_v(const KParams &p, int32_t tpos, int32_t len, int32_t c0, int lane,
                                                const bool (&valid)[NV], const int32_t (&head)[NV],
                                                const float (&tv)[NV], Part<M_GAT, VEC, NV> &G, float (&seen)[NV]) {
  const int32_t *idx = p.g.colidx_t + tpos;
  float nmb[NV];
#pragma unroll
  for (int n = 0; n < NV; ++n) {
    G.m[n] = seen[n];
    nmb[n] = -seen[n] * kLog2e;
    G.l[n] = 0.0f;
#pragma unroll
    for (int i = 0; i < VEC; ++i) G.a[n][i] = 0.0f;
  }
  const float *xl = p.X + c0 + lane * VEC;
  for (int32_t e = 0; e < len; ++e) {
    const int32_t u = ld_stream_i32(idx + e);
#pragma unroll
    for (int n = 0; n < NV; ++n) {
      if (!valid[n]) continue;
      float v[VEC];
      ldv<VEC>(xl + (int64_t)u * p.ldx + n * 32 * VEC, v);
      const float sco = leaky_f(__ldg(p.X + (int64_t)u * p.ldx + p.F + head[n]) + tv[n], p.slope);
      const float ex = ex2_f(fmaf(sco, kLog2e, nmb[n]));
      G.l[n] += ex;
      fma_vec<VEC>(G.a[n], v, ex);
    }
  }
}

// ---------------------------------------------------------------------------
// launch templates
// ---------------------------------------------------------------------------
struct Mapping {
  int vec, lanes, nv;
  int cp = 0;  // 1: the cp.async-staged chain with the (4, 32, nv) mapping; 2: the TMA gather4 streaming kernel
};
int num_sms();

template <typename KFN>
cudaError_t launch_persistent(KFN fn, int &occ, const KParams &kp_in, int32_t units, int cw, int lanes,
                                     int threads, cudaStream_t s, size_t smem = 0, size_t smem_attr = 0) {
  if (occ == 0) {
    if (smem > 0) {  // cp.async ring: shared memory first (attribute: the largest ring this kernel takes)
      cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)std::max(smem, smem_attr));
      cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    } else {
      cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, 0);  // all of it to L1
    }
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, threads, smem);
    if (occ <= 0) occ = 1;
  }
  KParams kp = kp_in;
  kp.nch = (kp.F + cw - 1) / cw;
  const int64_t workers_per_cta = threads / lanes;
  // A/B knob: cap on resident CTAs per SM (fewer concurrent groups = a narrower
  // window of the task order in flight = more L2 reuse, fewer rows in flight)
  static int cap = -1;
  if (cap < 0) {
    const char *e = getenv("GNN_AGG_CTAS_PER_SM");
    cap = e ? atoi(e) : 0;
  }
  const int occ_used = (cap > 0 && cap < occ) ? cap : occ;
  kp.n_persist = (int32_t)std::min<int64_t>((int64_t)num_sms() * occ_used,
                                            std::max<int64_t>(1, (units + workers_per_cta - 1) / workers_per_cta));
  if (kp.nch > kp.n_unit_ctr) return cudaErrorInvalidValue;  // mapping wider than the workspace sizing
  cudaError_t e = cudaMemsetAsync(kp.ws_unit, 0, sizeof(int32_t) * (size_t)kp.n_unit_ctr, s);
  if (e == cudaSuccess && kp.g.n_multi > 0)
    e = cudaMemsetAsync(kp.ws_cnt, 0, sizeof(int32_t) * (size_t)kp.g.n_multi * kp.nch, s);
  if (e == cudaSuccess && kp.g.n_multi > 0 && !kp.deterministic)  // max keys: 0 is below every key
    e = cudaMemsetAsync(kp.ws_acc, 0, sizeof(float) * (size_t)kp.g.n_multi * kp.FW, s);
  if (e != cudaSuccess) return e;
  if (e == cudaSuccess && kp.trace) {
    e = cudaMemsetAsync(kp.trace, 0, 8 * sizeof(unsigned long long), s);
    if (e == cudaSuccess) e = cudaMemsetAsync(kp.trace + 2, 0xff, sizeof(unsigned long long), s);
  }
  if (e != cudaSuccess) return e;
  const int64_t blocks = (int64_t)kp.n_persist + (kp.g.n_empty + 31) / 32;
  fn<<<(unsigned)blocks, threads, smem, s>>>(kp);
  count_launch();
  return cudaGetLastError();
}

template <int MODE, int VEC, int NV, int LANES>
cudaError_t launch_one(const KParams &kp, int threads, cudaStream_t s) {
  constexpr int CW = LANES * VEC * NV;
  static int occ = 0;
  return launch_persistent(k_aggregate<MODE, VEC, NV, LANES>, occ, kp, kp.g.n_units, CW, LANES, threads, s);
}

// the cp.async-staged kernel: (4, 32, NV) mapping, S ring slots per warp
template <int MODE, int NV>
cudaError_t launch_cp(const KParams &kp, int threads, cudaStream_t s) {
  constexpr int S = NV == 1 ? GNN_CP_S1 : GNN_CP_S2;
  constexpr int CW = 32 * 4 * NV;
  const size_t smem = sizeof(float) * ((size_t)(threads / 32) * S * cp_ring_slot<MODE, NV>(kp.F) + NV * 128);
  // the ring size depends on F: occupancy (and the dynamic shared-memory
  // attribute, set when occ == 0) cached per ring size
  static size_t occ_smem[8] = {0};
  static int occ_val[8] = {0};
  int slot = 0;
  while (slot < 8 && occ_smem[slot] != 0 && occ_smem[slot] != smem) ++slot;
  if (slot == 8) slot = 7;  // more sizes than slots: recompute in the last one
  if (occ_smem[slot] != smem) {
    occ_smem[slot] = smem;
    occ_val[slot] = 0;
  }
  const size_t smem_max = sizeof(float) * ((size_t)(threads / 32) * S * cp_slot_floats<MODE, NV>() + NV * 128);
  return launch_persistent(k_aggregate<MODE, 4, NV, 32, S>, occ_val[slot], kp, kp.g.n_units, CW, 32, threads, s,
                           smem, smem_max);
}

template <int MODE, int VEC>
cudaError_t dispatch_lanes(const KParams &kp, const Mapping &m, int threads, cudaStream_t s) {
  switch (m.lanes) {
    case 4: return launch_one<MODE, VEC, 1, 4>(kp, threads, s);
    case 8:
      if constexpr (VEC >= 4) {
        if (m.nv == 4) return launch_one<MODE, VEC, 4, 8>(kp, threads, s);
      }
      return launch_one<MODE, VEC, 1, 8>(kp, threads, s);
    case 16:
      if constexpr (VEC >= 2) {
        if (m.nv == 2) return launch_one<MODE, VEC, 2, 16>(kp, threads, s);
      }
      return launch_one<MODE, VEC, 1, 16>(kp, threads, s);
    default:
      if (m.nv == 1) return launch_one<MODE, VEC, 1, 32>(kp, threads, s);
      if (m.nv == 2) return launch_one<MODE, VEC, 2, 32>(kp, threads, s);
      if constexpr (VEC < 8) return launch_one<MODE, VEC, 4, 32>(kp, threads, s);
      return cudaErrorInvalidValue;
  }
}

template <int MODE>
cudaError_t dispatch_vec(const KParams &kp, const Mapping &m, int threads, cudaStream_t s) {
  if constexpr (MODE <= M_GAT) {
    if (m.cp) return m.nv == 1 ? launch_cp<MODE, 1>(kp, threads, s) : launch_cp<MODE, 2>(kp, threads, s);
  }
#ifdef GNN_DEV_SUBSET  // dev builds: only the C5 bench instantiations (fast compile)
  if (m.lanes == 32 && m.nv == 1 && m.vec == 8) return launch_one<MODE, 8, 1, 32>(kp, threads, s);
  if (m.lanes == 32 && m.nv == 1 && m.vec == 4) return launch_one<MODE, 4, 1, 32>(kp, threads, s);
  if (m.lanes == 16 && m.nv == 2 && m.vec == 4) return launch_one<MODE, 4, 2, 16>(kp, threads, s);
  if (m.lanes == 8 && m.nv == 4 && m.vec == 4) return launch_one<MODE, 4, 4, 8>(kp, threads, s);
  if (m.lanes == 16 && m.nv == 2 && m.vec == 8) return launch_one<MODE, 8, 2, 16>(kp, threads, s);
  if (m.lanes == 8 && m.nv == 4 && m.vec == 8) return launch_one<MODE, 8, 4, 8>(kp, threads, s);
  return cudaErrorInvalidValue;
#else
  switch (m.vec) {
    case 8: return dispatch_lanes<MODE, 8>(kp, m, threads, s);
    case 4: return dispatch_lanes<MODE, 4>(kp, m, threads, s);
    case 2: return dispatch_lanes<MODE, 2>(kp, m, threads, s);
    default: return dispatch_lanes<MODE, 1>(kp, m, threads, s);
  }
#endif
}

cudaError_t dispatch_sum(const KParams &kp, const Mapping &m, int threads, cudaStream_t s);
bool g4_admissible(const KParams &kp, int32_t n_src);
cudaError_t launch_row_score_max(const KParams &kp, cudaStream_t s);
cudaError_t launch_g4(const KParams &kp, int32_t n_src, cudaStream_t s);
cudaError_t dispatch_max(const KParams &kp, const Mapping &m, int threads, cudaStream_t s);
cudaError_t dispatch_gat(const KParams &kp, const Mapping &m, int threads, cudaStream_t s);
cudaError_t dispatch_att(const KParams &kp, const Mapping &m, int threads, cudaStream_t s);

}  // namespace gnn
