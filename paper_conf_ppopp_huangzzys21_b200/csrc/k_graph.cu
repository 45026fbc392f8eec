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
  float *ws_acc;   // [n_multi][FW] atomic accumulators (deterministic == 0)
  float *ws_part;  // [multi slots][FW] per-group partials (deterministic)
  int32_t *ws_cnt; // [n_multi][nch] arrival counters
  int32_t FW;      // F (+ 2H for GAT)
  int32_t deterministic;
  int32_t nch;  // feature chunks per row (arrival counters per multi-group row)
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

// Chain over CSR entries [beg, end) of destination `row`, neighbour groups
// of ng entries starting at beg (R9): a fresh fp32 group partial G runs in CSR
// order and is folded into the row accumulator A at every group boundary
// (A = G for the first group, then A = A (+) G).  One rolling register ring
// keeps U source rows in flight per worker across group boundaries; the next
// batch of LANES indices is requested before the current batch is consumed.
template <int MODE, int VEC, int NV, int LANES>
__device__ __forceinline__ void row_chain(const KParams &p, int32_t beg, int32_t end, int32_t row, int32_t c0,
                                          int lane, unsigned mask, Part<MODE, VEC, NV> &A) {
  constexpr int FPL = VEC * NV;  // floats per lane per source row
  constexpr int U = FPL >= 32 ? 1 : (32 / FPL > 8 ? 8 : 32 / FPL);
  const int32_t ng = p.g.ng;
  Part<MODE, VEC, NV> G;
  part_init(G);
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
  const int weight = p.weight;
  auto load_idx = [&](int32_t k, int32_t cnt, int32_t &u, float &w) {
    u = 0;
    w = 1.0f;
    if (lane < cnt) {
      u = ld_stream_i32(p.g.colidx + k + lane);
      if constexpr (MODE != M_GAT) {
        if (weight == GNN_W_GCN) w = __ldg(p.g.nsrc + u);
        else if (weight == GNN_W_EDGE) w = ld_stream_f32(p.edge_w + k + lane);
      }
    }
  };
  float v[U][NV][VEC];
  float sc[U][NV];
  auto load_row = [&](int q, int32_t u) {
    const float *xr = p.X + (int64_t)u * p.ldx;
#pragma unroll
    for (int n = 0; n < NV; ++n) {
      if (valid[n]) ldv<VEC>(xr + c0 + (n * LANES + lane) * VEC, v[q][n]);
      if constexpr (MODE == M_GAT) sc[q][n] = valid[n] ? __ldg(xr + p.F + head[n]) : 0.0f;
    }
  };
  int32_t k = beg;
  int32_t cnt = min(LANES, end - k);
  int32_t my_u;
  float my_w;
  load_idx(k, cnt, my_u, my_w);
  int32_t next_fold = (end - beg > ng) ? beg + ng : end;  // absolute index ending the current group
  bool first = true;
  for (;;) {
    const int32_t kn = k + LANES;
    const int32_t cnt_n = kn < end ? min(LANES, end - kn) : 0;
    int32_t nx_u;
    float nx_w;
    load_idx(kn, cnt_n, nx_u, nx_w);
#pragma unroll
    for (int q = 0; q < U; ++q)
      if (q < cnt) load_row(q, __shfl_sync(mask, my_u, q, LANES));
    for (int32_t j = 0; j < cnt; j += U) {
#pragma unroll
      for (int q = 0; q < U; ++q) {
        const int32_t e = j + q;
        if (e < cnt) {
          if constexpr (MODE == M_GAT) {
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
          if (e + U < cnt) load_row(q, __shfl_sync(mask, my_u, e + U, LANES));
          if (k + e + 1 == next_fold) {  // group boundary: fold G into A, restart G
            if (first) {
              A = G;
              first = false;
            } else {
              part_combine<MODE, VEC, NV>(A, G);
            }
            part_init(G);
            next_fold = (end - next_fold > ng) ? next_fold + ng : end;
          }
        }
      }
    }
    if (cnt_n == 0) break;
    k = kn;
    cnt = cnt_n;
    my_u = nx_u;
    my_w = nx_w;
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

// a9: a group of a multi-group row.  Deterministic: the group partial goes to
// its workspace slot; the worker that completes the row's last group merges
// all partials in group order (R9) and applies the postponed epilogue
// (P:970-986).  Atomic variant (sum/mean): partials are added into one
// accumulator row and the last worker applies the epilogue.
template <int MODE, int VEC, int NV, int LANES>
__device__ __forceinline__ void multi_group_combine(const KParams &p, int32_t m, int32_t row, int32_t rb, int32_t re,
                                                    int32_t beg, int32_t c0, int32_t ci, int lane, unsigned mask,
                                                    const Part<MODE, VEC, NV> &P) {
  const int32_t ng = p.g.ng;
  const int32_t ngrp = 1 + (re - rb - 1) / ng;
  const int32_t k = (beg - rb) / ng;
  const bool atomic_acc = !p.deterministic && MODE == M_SUM;
  float *base = p.ws_part + (size_t)p.g.multi_slot[m] * p.FW;
  float *acc = p.ws_acc + (size_t)m * p.FW;
#pragma unroll
  for (int n = 0; n < NV; ++n) {
    const int32_t f = c0 + (n * LANES + lane) * VEC;
    if (f >= p.F) continue;
    if (atomic_acc) {
#pragma unroll
      for (int i = 0; i < VEC; ++i) atomicAdd(acc + f + i, P.a[n][i]);
    } else {
      stv<VEC>(base + (size_t)k * p.FW + f, P.a[n]);
      if constexpr (MODE == M_GAT) {
        if (f % p.Fh == 0) {
          base[(size_t)k * p.FW + p.F + f / p.Fh] = P.m[n];
          base[(size_t)k * p.FW + p.F + p.H + f / p.Fh] = P.l[n];
        }
      }
    }
  }
  __threadfence();
  __syncwarp(mask);
  int last = 0;
  int32_t *cnt = p.ws_cnt + (size_t)m * p.nch + ci;
  if (lane == 0) last = atomicAdd(cnt, 1) == ngrp - 1;
  last = __shfl_sync(mask, last, 0, LANES);
  if (!last) return;
  __threadfence();
  Part<MODE, VEC, NV> A;
  part_init(A);
#pragma unroll
  for (int n = 0; n < NV; ++n) {
    const int32_t f = c0 + (n * LANES + lane) * VEC;
    if (f >= p.F) continue;
    if (atomic_acc) {
      ldv_cg<VEC>(acc + f, A.a[n]);
      continue;
    }
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
  store_row<MODE, VEC, NV, LANES>(p, row, re - rb, c0, lane, A);
  if (lane == 0) *cnt = 0;  // leave the counter at 0 for the next call
}

#ifndef GNN_AGG_MINB
#define GNN_AGG_MINB 4
#endif
// One CTA per tile of T consecutive groups in task order (a LAS cluster stays
// on one SM); groups round-robin over the CTA's workers (NG load
// balance).  No shared memory and no CTA barrier on the hot path.
template <int MODE, int VEC, int NV, int LANES>
__global__ void __launch_bounds__(256, MODE == M_GAT ? GNN_AGG_MINB - 1 : GNN_AGG_MINB) k_aggregate(const KParams p) {
  constexpr int CW = LANES * VEC * NV;
  const int tid = threadIdx.x;
  const int lane = tid & (LANES - 1);
  const int wk = tid / LANES;
  const int nwk = blockDim.x / LANES;
  const unsigned mask =
      LANES == 32 ? 0xffffffffu : (((1u << LANES) - 1u) << ((tid & 31) & ~(LANES - 1)));
  const DevGraph &g = p.g;
  if ((int32_t)blockIdx.x >= g.n_tiles) {
    // zero-fill rows without in-edges (R3-i): 32 rows per block
    const int64_t r0 = (int64_t)(blockIdx.x - g.n_tiles) * 32;
    for (int64_t r = r0; r < r0 + 32 && r < g.n_empty; ++r) {
      float *y = p.Y + (int64_t)g.empty_rows[r] * p.ldy;
      for (int f = tid; f < p.F; f += blockDim.x) y[f] = 0.0f;
    }
    return;
  }
  const int32_t gb = (int32_t)blockIdx.x * g.T;
  const int32_t ngr = min(g.T, g.n_groups - gb);
  int32_t ci = 0;
  for (int32_t c0 = 0; c0 < p.F; c0 += CW, ++ci) {
    for (int32_t j = wk; j < ngr; j += nwk) {
      const int32_t gi = gb + j;
      const int32_t row = g.grp_row[gi], beg = g.grp_beg[gi];
      const int32_t rb = g.rowptr[row], re = g.rowptr[row + 1];
      const int32_t end = (re - beg > g.ng) ? beg + g.ng : re;
      Part<MODE, VEC, NV> P;
      row_chain<MODE, VEC, NV, LANES>(p, beg, end, row, c0, lane, mask, P);  // exactly one group
      const int32_t m = g.grp_multi[gi];
      if (m < 0) store_row<MODE, VEC, NV, LANES>(p, row, re - rb, c0, lane, P);
      else multi_group_combine<MODE, VEC, NV, LANES>(p, m, row, rb, re, beg, c0, ci, lane, mask, P);
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

// a4: feature-length-adaptive mapping rule
static Mapping choose_mapping(const AggArgs &a, int32_t fh_or_0) {
  Mapping m{1, 4, 1};
  const int cands[4] = {8, 4, 2, 1};
  for (int v : cands) {
    bool ok = a.F % v == 0 && a.ldx % v == 0 && a.ldy % v == 0 && aligned(a.X, 4 * v) && aligned(a.Y, 4 * v);
    if (a.add_row) ok = ok && a.ld_add % v == 0 && aligned(a.add_row, 4 * v);
    if (fh_or_0) ok = ok && fh_or_0 % v == 0;
    if (ok) {
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

static int32_t max_chunks(int32_t F) { return F <= 128 ? 1 : (F + 31) / 32; }

size_t agg_workspace_bytes(const gnn_plan_s *p, int mode, int32_t F, int32_t H) {
  if (p->n_multi == 0) return 0;
  const size_t FW = (size_t)F + (mode == M_GAT ? 2 * (size_t)H : 0);
  size_t b = sizeof(int32_t) * (size_t)p->n_multi * max_chunks(F);
  b = (b + 255) & ~(size_t)255;
  return b + sizeof(float) * ((size_t)p->multi_slots + (size_t)p->n_multi) * FW;
}

template <int MODE, int VEC, int NV, int LANES>
static cudaError_t launch_one(const KParams &kp_in, int threads, size_t smem, int64_t blocks, cudaStream_t s) {
  auto fn = k_aggregate<MODE, VEC, NV, LANES>;
  static bool configured = false;  // per instantiation
  if (!configured) {
    // no shared memory on the hot path: the unified array goes to L1, which
    // serves the source rows a LAS cluster (one tile, one SM) shares
    cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, 0);
    configured = true;
  }
  KParams kp = kp_in;
  constexpr int CW = LANES * VEC * NV;
  kp.nch = (kp.F + CW - 1) / CW;
  if (kp.g.n_multi > 0) {
    cudaError_t e = cudaMemsetAsync(kp.ws_cnt, 0, sizeof(int32_t) * (size_t)kp.g.n_multi * kp.nch, s);
    if (e == cudaSuccess && !kp.deterministic && MODE == M_SUM)
      e = cudaMemsetAsync(kp.ws_acc, 0, sizeof(float) * (size_t)kp.g.n_multi * kp.FW, s);
    if (e != cudaSuccess) return e;
  }
  if (blocks == 0) return cudaSuccess;
  fn<<<(unsigned)blocks, threads, smem, s>>>(kp);
  count_launch();
  return cudaGetLastError();
}

template <int MODE, int VEC>
static cudaError_t dispatch_lanes(const KParams &kp, const Mapping &m, int threads, size_t smem, int64_t blocks,
                                  cudaStream_t s) {
  switch (m.lanes) {
    case 4: return launch_one<MODE, VEC, 1, 4>(kp, threads, smem, blocks, s);
    case 8: return launch_one<MODE, VEC, 1, 8>(kp, threads, smem, blocks, s);
    case 16: return launch_one<MODE, VEC, 1, 16>(kp, threads, smem, blocks, s);
    default:
      if (m.nv == 1) return launch_one<MODE, VEC, 1, 32>(kp, threads, smem, blocks, s);
      if (m.nv == 2) return launch_one<MODE, VEC, 2, 32>(kp, threads, smem, blocks, s);
      if constexpr (VEC < 8) return launch_one<MODE, VEC, 4, 32>(kp, threads, smem, blocks, s);
      return cudaErrorInvalidValue;
  }
}

template <int MODE>
static cudaError_t dispatch_vec(const KParams &kp, const Mapping &m, int threads, size_t smem, int64_t blocks,
                                cudaStream_t s) {
  switch (m.vec) {
    case 8: return dispatch_lanes<MODE, 8>(kp, m, threads, smem, blocks, s);
    case 4: return dispatch_lanes<MODE, 4>(kp, m, threads, smem, blocks, s);
    case 2: return dispatch_lanes<MODE, 2>(kp, m, threads, smem, blocks, s);
    default: return dispatch_lanes<MODE, 1>(kp, m, threads, smem, blocks, s);
  }
}

gnn_status launch_aggregate(const gnn_plan_s *p, const AggArgs &a, void *ws, size_t ws_bytes, cudaStream_t s) {
  if (a.F <= 0) return GNN_OK;
  const int mode = a.mode;
  const size_t need = agg_workspace_bytes(p, mode, a.F, a.H);
  if (p->n_multi > 0 && (ws == nullptr || ws_bytes < need)) {
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
  if (p->n_multi > 0) {
    // layout: [counters n_multi x nch int32 | pad to 256 B][accumulators n_multi x FW][slots x FW]
    const size_t cnt_bytes = (sizeof(int32_t) * (size_t)p->n_multi * max_chunks(a.F) + 255) & ~(size_t)255;
    kp.ws_cnt = reinterpret_cast<int32_t *>(ws);
    kp.ws_acc = reinterpret_cast<float *>(reinterpret_cast<char *>(ws) + cnt_bytes);
    kp.ws_part = kp.ws_acc + (size_t)p->n_multi * kp.FW;
  }
  const Mapping m = choose_mapping(a, mode == M_GAT ? a.Fh : 0);
  const int threads = std::min(256, std::max(32, p->T * m.lanes));
  const size_t smem = 0;
  const int64_t blocks = (int64_t)p->dg.n_tiles + (p->dg.n_empty + 31) / 32;
  cudaError_t e;
  switch (mode) {
    case M_SUM:
    case M_MEAN: e = dispatch_vec<M_SUM>(kp, m, threads, smem, blocks, s); break;
    case M_MAX: e = dispatch_vec<M_MAX>(kp, m, threads, smem, blocks, s); break;
    default: e = dispatch_vec<M_GAT>(kp, m, threads, smem, blocks, s); break;
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
