// k_graph.cu — sm_100a graph kernels of libgnn.so:
//   a1 degrees / GCN normalisers, a2 MinHash signatures, a6/a7/a8/a9 the
//   aggregation kernel family (sum, mean, max, fused GAT) with neighbor
//   grouping, feature-length-adaptive lane mapping and split-row combine.
//
// Paper: Huang et al., PPoPP'21 (PAPER.md P:<line>).  Design: DESIGN.md §5.
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include <algorithm>

#include "gnn_internal.h"

namespace gnn {

// ---------------------------------------------------------------------------
// a1: degrees and GCN normalisers (Table 2 GCN P:263-269, reading R1):
// d_out(u) = #CSR entries equal to u (integer atomics: exact, order-free),
// nsrc = 1/sqrtf(d_out), ndst = 1/sqrtf(d_in), 0 for degree 0.  IEEE sqrt
// and div (no fast-math) so the values are bit-identical to the host formula.
// ---------------------------------------------------------------------------
__global__ void k_count_out(const int32_t *__restrict__ colidx, int64_t nnz, int32_t *d_out) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nnz;
       k += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(d_out + colidx[k], 1);
}

__global__ void k_normalisers(const int32_t *__restrict__ rowptr, const int32_t *__restrict__ d_out,
                              int64_t n, int64_t n_src, float *nsrc, float *ndst) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (n > n_src ? n : n_src);
       i += (int64_t)gridDim.x * blockDim.x) {
    if (i < n_src) {
      int32_t d = d_out[i];
      nsrc[i] = d > 0 ? 1.0f / sqrtf((float)d) : 0.0f;
    }
    if (i < n) {
      int32_t d = rowptr[i + 1] - rowptr[i];
      ndst[i] = d > 0 ? 1.0f / sqrtf((float)d) : 0.0f;
    }
  }
}

cudaError_t launch_degrees(const int32_t *rowptr, const int32_t *colidx, int64_t n, int64_t n_src,
                           int64_t nnz, const int32_t *src_degree_override, int32_t *d_out_tmp,
                           float *nsrc, float *ndst, cudaStream_t s) {
  const int32_t *dout = src_degree_override;
  if (!dout) {
    cudaError_t e = cudaMemsetAsync(d_out_tmp, 0, sizeof(int32_t) * (size_t)(n_src > 0 ? n_src : 1), s);
    if (e != cudaSuccess) return e;
    if (nnz > 0) {
      int blocks = (int)std::min<int64_t>((nnz + 255) / 256, 148 * 16);
      k_count_out<<<blocks, 256, 0, s>>>(colidx, nnz, d_out_tmp);
      count_launch();
    }
    dout = d_out_tmp;
  }
  int64_t m = std::max<int64_t>(std::max(n, n_src), 1);
  int blocks = (int)std::min<int64_t>((m + 255) / 256, 148 * 16);
  k_normalisers<<<blocks, 256, 0, s>>>(rowptr, dout, n, n_src, nsrc, ndst);
  count_launch();
  return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// a2 step 1: Min-Hashing (reading R7).  One warp per row, lane k
// owns hash k: sig[v][k] = min over u in N(v) of fmix64(u + c_k).  Integer
// only -> bit-exact with the oracle.  K <= 64 (two salts per lane above 32).
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint64_t fmix64_dev(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

__global__ void k_minhash(const int32_t *__restrict__ rowptr, const int32_t *__restrict__ colidx,
                          int64_t n, int32_t K, const uint64_t *__restrict__ salts, uint64_t *sig) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const uint64_t c0 = lane < K ? salts[lane] : 0, c1 = lane + 32 < K ? salts[lane + 32] : 0;
  for (int64_t v = warp; v < n; v += nwarps) {
    const int32_t beg = rowptr[v], end = rowptr[v + 1];
    uint64_t m0 = ~0ULL, m1 = ~0ULL;
    for (int32_t base = beg; base < end; base += 32) {
      const int32_t cnt = min(32, end - base);
      const uint32_t mine = lane < cnt ? (uint32_t)__ldg(colidx + base + lane) : 0u;
      for (int32_t j = 0; j < cnt; ++j) {
        const uint64_t u = (uint64_t)__shfl_sync(0xffffffffu, mine, j);
        const uint64_t h0 = fmix64_dev(u + c0);
        m0 = h0 < m0 ? h0 : m0;
        if (K > 32) {
          const uint64_t h1 = fmix64_dev(u + c1);
          m1 = h1 < m1 ? h1 : m1;
        }
      }
    }
    if (lane < K) sig[v * K + lane] = m0;
    if (lane + 32 < K) sig[v * K + lane + 32] = m1;
  }
}

cudaError_t launch_minhash(const int32_t *rowptr, const int32_t *colidx, int64_t n, int32_t K,
                           uint64_t seed, uint64_t *sig, cudaStream_t s) {
  // salts c_k = k-th SplitMix64 output from `seed` (same stream as the oracle's
  // definition; computed here independently)
  uint64_t salts_h[64];
  uint64_t st = seed;
  for (int k = 0; k < K; ++k) {
    st += 0x9E3779B97F4A7C15ULL;
    uint64_t z = st;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    salts_h[k] = z ^ (z >> 31);
  }
  uint64_t *salts_d = nullptr;
  cudaError_t e = cudaMalloc(&salts_d, sizeof(uint64_t) * 64);
  if (e != cudaSuccess) return e;
  e = cudaMemcpyAsync(salts_d, salts_h, sizeof(uint64_t) * K, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess && n > 0) {
    int blocks = (int)std::min<int64_t>((n * 32 + 255) / 256, 148 * 32);
    k_minhash<<<blocks, 256, 0, s>>>(rowptr, colidx, n, K, salts_d, sig);
    count_launch();
    e = cudaGetLastError();
  }
  cudaError_t e2 = cudaStreamSynchronize(s);
  cudaFree(salts_d);
  return e != cudaSuccess ? e : e2;
}

// ---------------------------------------------------------------------------
// a6/a7/a8/a9: the aggregation kernel family.
//
// Mapping (a4, feature-length-adaptive): a "worker"
// is LANES consecutive lanes (LANES in {4, 8, 16, 32}); each lane owns NV
// vectors of VEC consecutive features (VEC in {1,2,4,8}; VEC = 8 is one
// 256-bit LDG per lane).  Chunk width CW = LANES*VEC*NV features; wider rows
// loop over chunks.  One CTA processes one plan tile (<= T neighbor groups,
// P:855-884) per launch block; workers take groups round-robin.
//
// Per group: indices are loaded LANES at a time (one coalesced load), then
// broadcast with sub-warp shuffles; U source rows are in flight per worker.
// Group partial = sequential fp32 chain in CSR order (reading R9).
// Single-group rows finish in the worker (epilogue + store).  Multi-group
// rows inside one tile are combined in shared memory in group order (TB-level
// data-visible-range adapter).  Rows spanning several tiles write
// per-group partials to the workspace; the last-arriving CTA (per-row counter)
// merges them in group order (P:885-894 with a fixed order) and applies the
// postponed epilogue (linear property).
// ---------------------------------------------------------------------------
enum { M_SUM = 0, M_MEAN = 1, M_MAX = 2, M_GAT = 3 };
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
  int32_t *ws_unit;  // work-unit counters (one per feature chunk), zeroed per call
  float *ws_acc;   // [n_multi][FW] atomic accumulators (deterministic == 0)
  float *ws_part;  // [multi slots][FW] per-group partials (deterministic)
  int32_t *ws_cnt; // [n_multi][nch] arrival counters
  int32_t FW;      // F (+ 2H for GAT)
  int32_t deterministic;
  int32_t nch;        // feature chunks per row (arrival counters per multi-unit row)
  int32_t n_persist;  // persistent CTAs
};

template <int VEC>
__device__ __forceinline__ void ldv(const float *p, float (&v)[VEC]) {
  if constexpr (VEC == 8) {
    asm volatile("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]),
                   "=f"(v[6]), "=f"(v[7])
                 : "l"(p));
  } else if constexpr (VEC == 4) {
    float4 x = __ldg(reinterpret_cast<const float4 *>(p));
    v[0] = x.x; v[1] = x.y; v[2] = x.z; v[3] = x.w;
  } else if constexpr (VEC == 2) {
    float2 x = __ldg(reinterpret_cast<const float2 *>(p));
    v[0] = x.x; v[1] = x.y;
  } else {
    v[0] = __ldg(p);
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

// streaming index load: read once, do not keep in L1
__device__ __forceinline__ int32_t ld_stream_i32(const int32_t *p) {
  int32_t r;
  asm volatile("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ float ld_stream_f32(const float *p) {
  float r;
  asm volatile("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(r) : "l"(p));
  return r;
}

// fixed ReLU: y > 0 ? y : +0 (matches the oracle replica, R9)
__device__ __forceinline__ float relu_f(float y) { return y > 0.0f ? y : 0.0f; }

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
    if constexpr (MODE == M_GAT) {
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
  if (mode == M_GAT) {
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

template <int MODE, int VEC, int NV, int LANES>
__device__ __forceinline__ void store_row(const KParams &p, int32_t row, int32_t deg, int32_t c0,
                                          int lane, const Part<MODE, VEC, NV> &P) {
  const float ndst = (MODE != M_GAT && scales_dst(p.weight)) ? __ldg(p.g.ndst + row) : 1.0f;
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
    stv<VEC>(p.Y + (int64_t)row * p.ldy + f, y);
  }
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

// ---------------------------------------------------------------------------
// v8 work distribution (measured: scripts/stream_bench_k.cu): persistent
// workers grab work units in task (LAS) order through one atomic counter, so
// the units in flight across the GPU are consecutive in the schedule and share
// their source rows in L2; load balance is dynamic (NG's goal,
// P:855-884) with no CTA barrier.  A unit is a whole row (<= R groups) or an
// R-group slice of a longer row; its source indices are read from the
// task-ordered colidx_t (one contiguous stream per unit).
// ---------------------------------------------------------------------------

// one neighbour group: fresh fp32 chain in CSR order (R9); indices from the
// task-ordered stream, LANES at a time, U source rows in flight per worker
template <int MODE, int VEC, int NV, int LANES>
__device__ __forceinline__ void group_chain(const KParams &p, const int32_t *idx, int32_t len, int32_t beg,
                                            int32_t row, int32_t c0, int lane, unsigned mask,
                                            Part<MODE, VEC, NV> &G) {
  constexpr int FPL = VEC * NV;
  constexpr int U = FPL >= 32 ? 1 : (32 / FPL > 8 ? 8 : 32 / FPL);
  part_init(G);
  const int weight = p.weight;
  const float *xl = p.X + c0 + lane * VEC;
  bool valid[NV];
  int32_t head[NV];
  float tv[NV];
#pragma unroll
  for (int n = 0; n < NV; ++n) {
    const int32_t f = c0 + (n * LANES + lane) * VEC;
    valid[n] = f < p.F;
    head[n] = 0;
    tv[n] = 0.0f;
    if constexpr (MODE == M_GAT) {
      head[n] = valid[n] ? f / p.Fh : 0;
      tv[n] = valid[n] ? __ldg(p.t + (int64_t)row * p.ldt + head[n]) : 0.0f;
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
            // online softmax (R9 GAT): one exp per edge and head
#pragma unroll
            for (int n = 0; n < NV; ++n) {
              if (!valid[n]) continue;
              float sco = sc[q][n] + tv[n];
              sco = sco > 0.0f ? sco : p.slope * sco;  // LeakyReLU (Table 2 GAT)
              const float d = sco - G.m[n];
              const float ex = __expf(-fabsf(d));
              const bool up = d > 0.0f;
#pragma unroll
              for (int i = 0; i < VEC; ++i)
                G.a[n][i] = fmaf(up ? G.a[n][i] : v[q][n][i], ex, up ? v[q][n][i] : G.a[n][i]);
              G.l[n] = fmaf(up ? G.l[n] : 1.0f, ex, up ? 1.0f : G.l[n]);
              G.m[n] = up ? sco : G.m[n];
            }
          } else {
            const float w = __shfl_sync(mask, my_w, e, LANES);
#pragma unroll
            for (int n = 0; n < NV; ++n) {
              if (!valid[n]) continue;
#pragma unroll
              for (int i = 0; i < VEC; ++i) {
                if constexpr (MODE == M_MAX) G.a[n][i] = fmaxf(G.a[n][i], w * v[q][n][i]);
                else G.a[n][i] = fmaf(w, v[q][n][i], G.a[n][i]);
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
}

// merge the group partials of a long row in group order (R9), epilogue, store
template <int MODE, int VEC, int NV, int LANES>
__device__ __forceinline__ void merge_row(const KParams &p, const float *base, int32_t ngrp, int32_t row,
                                          int32_t deg, int32_t c0, int lane) {
  Part<MODE, VEC, NV> A;
  part_init(A);
#pragma unroll
  for (int n = 0; n < NV; ++n) {
    const int32_t f = c0 + (n * LANES + lane) * VEC;
    if (f >= p.F) continue;
    for (int32_t q = 0; q < ngrp; ++q) {
      float b[VEC];
      ldv_cg<VEC>(base + (size_t)q * p.FW + f, b);
      if constexpr (MODE == M_GAT) {
        const float bm = __ldcg(base + (size_t)q * p.FW + p.F + f / p.Fh);
        const float bl = __ldcg(base + (size_t)q * p.FW + p.F + p.H + f / p.Fh);
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
__device__ __forceinline__ void process_unit(const KParams &p, int4 d, int32_t len, int32_t c0, int32_t ci, int lane,
                                             unsigned mask) {
  const DevGraph &g = p.g;
  const int32_t tpos = d.x, beg = d.y, row = d.z, m = d.w;
  Part<MODE, VEC, NV> G;
  group_chain<MODE, VEC, NV, LANES>(p, g.colidx_t + tpos, len, beg, row, c0, lane, mask, G);
  const int32_t rb = g.rowptr[row], re = g.rowptr[row + 1];
  if (m < 0) {
    store_row<MODE, VEC, NV, LANES>(p, row, re - rb, c0, lane, G);
    return;
  }
  const int32_t ng = g.ng;
  const int32_t ngrp = 1 + (re - rb - 1) / ng;
  const int32_t k = (beg - rb) / ng;
  const bool atomic_acc = !p.deterministic && MODE == M_SUM;
  float *base = p.ws_part + (size_t)g.multi_slot[m] * p.FW;
  float *acc = p.ws_acc + (size_t)m * p.FW;
#pragma unroll
  for (int n = 0; n < NV; ++n) {
    const int32_t f = c0 + (n * LANES + lane) * VEC;
    if (f >= p.F) continue;
    if (atomic_acc) {
#pragma unroll
      for (int i = 0; i < VEC; ++i) atomicAdd(acc + f + i, G.a[n][i]);
    } else {
      stv<VEC>(base + (size_t)k * p.FW + f, G.a[n]);
      if constexpr (MODE == M_GAT) {
        if (f % p.Fh == 0) {
          base[(size_t)k * p.FW + p.F + f / p.Fh] = G.m[n];
          base[(size_t)k * p.FW + p.F + p.H + f / p.Fh] = G.l[n];
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
      if (f < p.F) ldv_cg<VEC>(acc + f, A.a[n]);
    }
    store_row<MODE, VEC, NV, LANES>(p, row, re - rb, c0, lane, A);
  } else {
    merge_row<MODE, VEC, NV, LANES>(p, base, ngrp, row, re - rb, c0, lane);
  }
  if (lane == 0) *cnt = 0;  // leave the counter at 0 for the next call
}

#ifndef GNN_AGG_MINB
#define GNN_AGG_MINB 4
#endif
template <int MODE, int VEC, int NV, int LANES>
__global__ void __launch_bounds__(256, MODE == M_GAT ? GNN_AGG_MINB - 1 : GNN_AGG_MINB) k_aggregate(const KParams p) {
  constexpr int CW = LANES * VEC * NV;
  const int tid = threadIdx.x;
  const int lane = tid & (LANES - 1);
  const unsigned mask =
      LANES == 32 ? 0xffffffffu : (((1u << LANES) - 1u) << ((tid & 31) & ~(LANES - 1)));
  const DevGraph &g = p.g;
  if ((int32_t)blockIdx.x >= p.n_persist) {
    // zero-fill rows without in-edges (R3-i): 32 rows per block
    const int64_t r0 = (int64_t)(blockIdx.x - p.n_persist) * 32;
    for (int64_t r = r0; r < r0 + 32 && r < g.n_empty; ++r) {
      float *y = p.Y + (int64_t)g.empty_rows[r] * p.ldy;
      for (int f = tid; f < p.F; f += blockDim.x) y[f] = 0.0f;
    }
    return;
  }
  const int32_t nunits = g.n_units;
  int32_t ci = 0;
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
      int32_t un = 0;
      if (lane == 0) un = atomicAdd(ctr, 1);
      un = __shfl_sync(mask, un, 0, LANES);
      int4 dn = make_int4(0, 0, 0, -1);
      int32_t dnxn = 0;
      if (un < nunits) {
        dn = __ldg(g.unit_desc + un);
        dnxn = __ldg(&g.unit_desc[un + 1].x);
      }
      process_unit<MODE, VEC, NV, LANES>(p, d, dnx - d.x, c0, ci, lane, mask);
      u = un;
      d = dn;
      dnx = dnxn;
    }
  }
}

// ---------------------------------------------------------------------------
// host dispatch
// ---------------------------------------------------------------------------
static bool aligned(const void *ptr, int bytes) {
  return ptr == nullptr || (reinterpret_cast<uintptr_t>(ptr) % (uintptr_t)bytes) == 0;
}

struct Mapping {
  int vec, lanes, nv;
};

// feature chunks one call may sweep (sizes the per-chunk counters): the
// automatic rule needs <= ceil(F/32); an override up to 8
static int32_t max_chunks(int32_t F) { return std::max<int32_t>(8, (F + 31) / 32); }

// process-wide mapping override (gnn_set_agg_mapping; the tuner hook)
static Mapping g_override{0, 0, 0};

bool set_agg_mapping(int32_t vec, int32_t lanes, int32_t nv) {
  if (vec == 0 && lanes == 0 && nv == 0) {
    g_override = Mapping{0, 0, 0};
    return true;
  }
  const bool vec_ok = vec == 1 || vec == 2 || vec == 4 || vec == 8;
  const bool lanes_ok = lanes == 4 || lanes == 8 || lanes == 16 || lanes == 32;
  const bool nv_ok = nv == 1 || ((nv == 2 || nv == 4) && lanes == 32 && !(vec == 8 && nv == 4));
  if (!vec_ok || !lanes_ok || !nv_ok) return false;
  g_override = Mapping{vec, lanes, nv};
  return true;
}

static bool vec_admissible(const AggArgs &a, int32_t fh_or_0, int v) {
  bool ok = a.F % v == 0 && a.ldx % v == 0 && a.ldy % v == 0 && aligned(a.X, 4 * v) && aligned(a.Y, 4 * v);
  if (a.add_row) ok = ok && a.ld_add % v == 0 && aligned(a.add_row, 4 * v);
  if (fh_or_0) ok = ok && fh_or_0 % v == 0;
  return ok;
}

// a4: feature-length-adaptive mapping rule
static Mapping choose_mapping(const AggArgs &a, int32_t fh_or_0) {
  Mapping m{1, 4, 1};
  if (g_override.vec != 0 && vec_admissible(a, fh_or_0, g_override.vec)) {
    // GAT: a chunk must hold whole heads (the softmax state is per head)
    const int cw = g_override.vec * g_override.lanes * g_override.nv;
    const bool heads_ok = !fh_or_0 || cw >= a.F || cw % fh_or_0 == 0;
    if (heads_ok && (a.F + cw - 1) / cw <= max_chunks(a.F)) return g_override;
  }
  const int cands[4] = {8, 4, 2, 1};
  for (int v : cands) {
    if (vec_admissible(a, fh_or_0, v)) {
      m.vec = v;
      break;
    }
  }
  const int nvec = a.F / m.vec;  // vectors per row
  int lanes = 4;
  while (lanes < nvec && lanes < 32) lanes *= 2;
  m.lanes = lanes;
  m.nv = 1;
  if (lanes == 32) {
    const int max_nv = m.vec == 8 ? 2 : 4;
    while (m.nv < max_nv && 32 * m.nv < nvec) m.nv *= 2;
  }
  return m;
}


// layout: [unit counters (256 B)][row counters n_multi x nch | pad 256][acc n_multi x FW][slots x FW]
size_t agg_workspace_bytes(const gnn_plan_s *p, int mode, int32_t F, int32_t H) {
  const size_t FW = (size_t)F + (mode == M_GAT ? 2 * (size_t)H : 0);
  size_t b = 256;
  size_t c = sizeof(int32_t) * (size_t)p->n_multi * max_chunks(F);
  b += (c + 255) & ~(size_t)255;
  return b + sizeof(float) * ((size_t)p->multi_slots + (size_t)p->n_multi) * FW;
}

static int num_sms() {
  static int n = 0;
  if (n == 0) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

template <int MODE, int VEC, int NV, int LANES>
static cudaError_t launch_one(const KParams &kp_in, int threads, cudaStream_t s) {
  auto fn = k_aggregate<MODE, VEC, NV, LANES>;
  static int occ = 0;  // resident CTAs per SM for this instantiation
  if (occ == 0) {
    cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, 0);  // all of it to L1
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, threads, 0);
    if (occ <= 0) occ = 1;
  }
  KParams kp = kp_in;
  constexpr int CW = LANES * VEC * NV;
  kp.nch = (kp.F + CW - 1) / CW;
  const int64_t workers_per_cta = threads / LANES;
  kp.n_persist = (int32_t)std::min<int64_t>((int64_t)num_sms() * occ,
                                            std::max<int64_t>(1, (kp.g.n_units + workers_per_cta - 1) / workers_per_cta));
  cudaError_t e = cudaMemsetAsync(kp.ws_unit, 0, 256, s);
  if (e == cudaSuccess && kp.g.n_multi > 0)
    e = cudaMemsetAsync(kp.ws_cnt, 0, sizeof(int32_t) * (size_t)kp.g.n_multi * kp.nch, s);
  if (e == cudaSuccess && kp.g.n_multi > 0 && !kp.deterministic && MODE == M_SUM)
    e = cudaMemsetAsync(kp.ws_acc, 0, sizeof(float) * (size_t)kp.g.n_multi * kp.FW, s);
  if (e != cudaSuccess) return e;
  const int64_t blocks = (int64_t)kp.n_persist + (kp.g.n_empty + 31) / 32;
  fn<<<(unsigned)blocks, threads, 0, s>>>(kp);
  count_launch();
  return cudaGetLastError();
}

template <int MODE, int VEC>
static cudaError_t dispatch_lanes(const KParams &kp, const Mapping &m, int threads, cudaStream_t s) {
  switch (m.lanes) {
    case 4: return launch_one<MODE, VEC, 1, 4>(kp, threads, s);
    case 8: return launch_one<MODE, VEC, 1, 8>(kp, threads, s);
    case 16: return launch_one<MODE, VEC, 1, 16>(kp, threads, s);
    default:
      if (m.nv == 1) return launch_one<MODE, VEC, 1, 32>(kp, threads, s);
      if (m.nv == 2) return launch_one<MODE, VEC, 2, 32>(kp, threads, s);
      if constexpr (VEC < 8) return launch_one<MODE, VEC, 4, 32>(kp, threads, s);
      return cudaErrorInvalidValue;
  }
}

template <int MODE>
static cudaError_t dispatch_vec(const KParams &kp, const Mapping &m, int threads, cudaStream_t s) {
  switch (m.vec) {
    case 8: return dispatch_lanes<MODE, 8>(kp, m, threads, s);
    case 4: return dispatch_lanes<MODE, 4>(kp, m, threads, s);
    case 2: return dispatch_lanes<MODE, 2>(kp, m, threads, s);
    default: return dispatch_lanes<MODE, 1>(kp, m, threads, s);
  }
}

gnn_status launch_aggregate(const gnn_plan_s *p, const AggArgs &a, void *ws, size_t ws_bytes, cudaStream_t s) {
  if (a.F <= 0) return GNN_OK;
  const int mode = a.mode;
  const size_t need = agg_workspace_bytes(p, mode, a.F, a.H);
  if (ws == nullptr || ws_bytes < need) {
    set_error("workspace too small: need " + std::to_string(need) + " bytes");
    return GNN_ERR_WORKSPACE;
  }
  KParams kp{};
  kp.g = p->dg;
  kp.mode = mode;
  kp.weight = a.weight;
  kp.edge_w = a.edge_w;
  kp.X = a.X;
  kp.ldx = a.ldx;
  kp.F = a.F;
  kp.Y = a.Y;
  kp.ldy = a.ldy;
  kp.add_row = a.add_row;
  kp.ld_add = a.ld_add;
  kp.relu = a.relu;
  kp.t = a.t;
  kp.ldt = a.ldt;
  kp.H = a.H;
  kp.Fh = a.Fh;
  kp.slope = a.slope;
  kp.FW = a.F + (mode == M_GAT ? 2 * a.H : 0);
  kp.deterministic = a.deterministic;
  char *w = reinterpret_cast<char *>(ws);
  kp.ws_unit = reinterpret_cast<int32_t *>(w);
  const size_t cnt_bytes = (sizeof(int32_t) * (size_t)p->n_multi * max_chunks(a.F) + 255) & ~(size_t)255;
  kp.ws_cnt = reinterpret_cast<int32_t *>(w + 256);
  kp.ws_acc = reinterpret_cast<float *>(w + 256 + cnt_bytes);
  kp.ws_part = kp.ws_acc + (size_t)p->n_multi * kp.FW;
  const Mapping m = choose_mapping(a, mode == M_GAT ? a.Fh : 0);
  const int threads = 256;
  cudaError_t e;
  switch (mode) {
    case M_SUM:
    case M_MEAN: e = dispatch_vec<M_SUM>(kp, m, threads, s); break;
    case M_MAX: e = dispatch_vec<M_MAX>(kp, m, threads, s); break;
    default: e = dispatch_vec<M_GAT>(kp, m, threads, s); break;
  }
  return cuda_status(e, "aggregate launch");
}

// ---------------------------------------------------------------------------
// small weight-preparation kernels (run once per layer call, O(f_in * H*Fh))
// ---------------------------------------------------------------------------
// Wext[:, 0:HF] = W; Wext[:, HF + h] = W_h . a_src_h; Wext[:, HF + H + h] = W_h . a_dst_h
__global__ void k_gat_weights(const float *W, const float *a_src, const float *a_dst, int32_t f_in,
                              int32_t H, int32_t Fh, float *Wext, int32_t ldwe) {
  const int32_t HF = H * Fh;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (int64_t)f_in * ldwe;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = (int32_t)(i / ldwe), c = (int32_t)(i % ldwe);
    float v = 0.0f;
    if (c < HF) {
      v = W[(int64_t)r * HF + c];
    } else if (c < HF + 2 * H) {
      const int32_t h = (c - HF) % H;
      const float *a = (c < HF + H) ? a_src : a_dst;
      for (int32_t f = 0; f < Fh; ++f) v = fmaf(W[(int64_t)r * HF + h * Fh + f], a[h * Fh + f], v);
    }
    Wext[i] = v;
  }
}

cudaError_t launch_gat_weights(const float *W, const float *a_src, const float *a_dst, int32_t f_in,
                               int32_t H, int32_t Fh, float *Wext, int32_t ldwe, cudaStream_t s) {
  const int64_t tot = (int64_t)f_in * ldwe;
  const int blocks = (int)std::max<int64_t>(1, std::min<int64_t>((tot + 255) / 256, 1024));
  k_gat_weights<<<blocks, 256, 0, s>>>(W, a_src, a_dst, f_in, H, Fh, Wext, ldwe);
  count_launch();
  return cudaGetLastError();
}

// Wpq [f_in, 2 f_out]: column o < f_out = theta[o, :], column f_out + o = (phi - theta)[o, :];
// bpq [2 f_out] = [0 | b]
__global__ void k_edgeconv_weights(const float *theta, const float *phi, const float *bias,
                                   int32_t f_in, int32_t f_out, float *Wpq, float *bpq) {
  const int32_t ld = 2 * f_out;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (int64_t)f_in * ld;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = (int32_t)(i / ld), c = (int32_t)(i % ld);
    Wpq[i] = c < f_out ? theta[(int64_t)c * f_in + r]
                       : phi[(int64_t)(c - f_out) * f_in + r] - theta[(int64_t)(c - f_out) * f_in + r];
  }
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < ld;
       i += (int64_t)gridDim.x * blockDim.x)
    bpq[i] = (i < f_out || bias == nullptr) ? 0.0f : bias[i - f_out];
}

cudaError_t launch_edgeconv_weights(const float *theta, const float *phi, const float *bias,
                                    int32_t f_in, int32_t f_out, float *Wpq, float *bpq,
                                    cudaStream_t s) {
  const int64_t tot = (int64_t)f_in * 2 * f_out;
  const int blocks = (int)std::max<int64_t>(1, std::min<int64_t>((tot + 255) / 256, 1024));
  k_edgeconv_weights<<<blocks, 256, 0, s>>>(theta, phi, bias, f_in, f_out, Wpq, bpq);
  count_launch();
  return cudaGetLastError();
}

}  // namespace gnn
