// k_lstm.cu — NEXT-3: GraphSAGE-LSTM with sparse fetching and redundancy
// bypassing (Huang et al., PPoPP'21, §4.3, Fig 6; reading R13).
//
// Redundancy bypass: the input transform of every cell,
// W_{i,f,z,o} x_u, is computed once per node by the tensor-core GEMM
// GS = X [W_ihᵀ | W_selfᵀ] + [b_ih + b_hh | b]  (gates interleaved per hidden
// unit: column 4j+g = gate g of unit j), O(N) instead of O(N·T).
// Sparse fetching: cell t of center node v reads the row
// GS[u_t] of its t-th sampled neighbour by index inside the cell kernel —
// one 512 B row, one 16 B vector per lane — while the recurrent product
// R h_{t-1} and the element-wise cell run in registers; the neighbour
// feature matrix is never materialised.
//
// k_sage_lstm: one warp = NB center nodes, lane j = hidden unit j (F = 32).
// Rᵀ (16 KB, [k][j] float4 of the four gates) and W_neighᵀ stay in shared
// memory; h_{t-1} of each node sits in a per-warp shared buffer and is read
// as broadcast float4s.  The next cell's rows are fetched while the current
// cell computes.  After T cells the SAGE combine y = S_v + W_neigh h_T
// (S_v = x_v W_selfᵀ + b from the same GEMM) is the epilogue.  Rows are
// processed in the plan's task (LAS) order so that neighbouring center nodes
// share their sampled rows in L2.
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>

#include "gnn_internal.h"

namespace gnn {

int num_sms();

constexpr int kLstmF = 32;   // hidden units (32 in / 32 out)
constexpr int kLstmNB = 4;   // center nodes per warp (amortises the shared-memory weight reads)
constexpr int kLstmWarps = 8;
#ifndef GNN_LSTM_MINB
#define GNN_LSTM_MINB 3  // 3 CTAs per SM (4 measured slower: 64 registers spill, 10.1 vs 9.4 ms)
#endif

__device__ __forceinline__ uint64_t fmix64_s(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

// reading R13: sample t of row v = colidx[rowptr[v] + fmix64(seed + (vT + t + 1) * golden) mod d_v]
__global__ void k_sample_neighbors(const int32_t *__restrict__ rowptr, const int32_t *__restrict__ colidx,
                                   int64_t n, int32_t T, uint64_t seed, int32_t *table) {
  const int64_t tot = n * (int64_t)T;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < tot; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t v = i / T;
    const int32_t rb = rowptr[v], d = rowptr[v + 1] - rb;
    int32_t u = -1;
    if (d > 0) {
      const uint64_t h = fmix64_s(seed + (uint64_t)(i + 1) * 0x9E3779B97F4A7C15ULL);
      u = colidx[rb + (int32_t)(h % (uint64_t)d)];
    }
    table[i] = u;
  }
}

cudaError_t launch_sample_neighbors(const gnn_plan_s *p, int32_t T, uint64_t seed, int32_t *table, cudaStream_t s) {
  const int64_t tot = p->n * (int64_t)T;
  if (tot == 0) return cudaSuccess;
  const int blocks = (int)std::min<int64_t>((tot + 255) / 256, (int64_t)148 * 16);
  k_sample_neighbors<<<blocks, 256, 0, s>>>(p->dg.rowptr, p->dg.colidx, p->n, T, seed, table);
  count_launch();
  return cudaGetLastError();
}

// Wcat [f_in, 4F + F_out]: Wcat[k][4j+g] = W_ih[gF + j][k], Wcat[k][4F + o] = W_self[o][k];
// bcat[4j+g] = b_ih[gF+j] + b_hh[gF+j], bcat[4F+o] = bias[o]
__global__ void k_lstm_weights(const float *W_ih, const float *b_ih, const float *b_hh, const float *W_self,
                               const float *bias, int32_t f_in, int32_t F, int32_t F_out, float *Wcat, float *bcat) {
  const int32_t ld = 4 * F + F_out;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (int64_t)(f_in + 1) * ld;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = (int32_t)(i / ld), c = (int32_t)(i % ld);
    float v;
    if (c < 4 * F) {
      const int32_t j = c >> 2, g = c & 3;
      v = r < f_in ? W_ih[(int64_t)(g * F + j) * f_in + r] : b_ih[g * F + j] + b_hh[g * F + j];
    } else {
      const int32_t o = c - 4 * F;
      v = r < f_in ? W_self[(int64_t)o * f_in + r] : (bias ? bias[o] : 0.0f);
    }
    if (r < f_in) Wcat[i] = v;
    else bcat[c] = v;
  }
}

cudaError_t launch_lstm_weights(const float *W_ih, const float *b_ih, const float *b_hh, const float *W_self,
                                const float *bias, int32_t f_in, int32_t F, int32_t F_out, float *Wcat,
                                float *bcat, cudaStream_t s) {
  const int64_t tot = (int64_t)(f_in + 1) * (4 * F + F_out);
  const int blocks = (int)std::max<int64_t>(1, std::min<int64_t>((tot + 255) / 256, 1024));
  k_lstm_weights<<<blocks, 256, 0, s>>>(W_ih, b_ih, b_hh, W_self, bias, f_in, F, F_out, Wcat, bcat);
  count_launch();
  return cudaGetLastError();
}

struct LstmParams {
  const int32_t *table;
  int32_t T;
  const float *GS;
  int64_t ldg;
  const float *R;   // [4F, F] recurrent weights, gate blocks i, f, z, o
  const float *Wn;  // [F_out, F]
  int32_t F_out;
  float *Y;
  int64_t ldy;
  const int32_t *order;  // task order of the rows (plan perm)
  int64_t n;
};

// sigmoid / tanh from ex2.approx and rcp.approx (2 MUFU each, no IEEE division sequence)
__device__ __forceinline__ float rcp_s(float x) {
  float r;
  asm("rcp.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
__device__ __forceinline__ float ex2_s(float x) {
  float r;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
// (reciprocal by Newton iterations on the FMA pipe measured slower, 10.8 vs
// 9.8 ms: the cells are issue-bound, not MUFU-bound)
__device__ __forceinline__ float rcp_sel(float x) { return rcp_s(x); }
__device__ __forceinline__ float sigm(float x) { return rcp_sel(1.0f + ex2_s(fminf(-1.4426950408889634f * x, 64.0f))); }
__device__ __forceinline__ float tanh_f(float x) {
  return fmaf(2.0f, rcp_sel(1.0f + ex2_s(fminf(-2.8853900817779268f * x, 64.0f))), -1.0f);
}

__global__ void __launch_bounds__(kLstmWarps * 32, GNN_LSTM_MINB) k_sage_lstm(const LstmParams p) {
  constexpr int F = kLstmF, NB = kLstmNB;
  __shared__ float4 Rt[F][F];                // Rt[k][j] = (R_i, R_f, R_z, R_o)[j][k]
  __shared__ float Wnt[F][F + 1];            // Wnt[j][o] = W_neigh[o][j]
  __shared__ __align__(16) float hb[kLstmWarps][NB][F];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (int i = tid; i < F * F; i += blockDim.x) {
    const int k = i / F, j = i % F;
    Rt[k][j] = make_float4(p.R[(0 * F + j) * F + k], p.R[(1 * F + j) * F + k], p.R[(2 * F + j) * F + k],
                           p.R[(3 * F + j) * F + k]);
    const int jj = i / F, o = i % F;
    Wnt[jj][o] = o < p.F_out ? p.Wn[o * F + jj] : 0.0f;
  }
  __syncthreads();
  const int T = p.T;
  for (int64_t base = ((int64_t)blockIdx.x * kLstmWarps + warp) * NB; base < p.n;
       base += (int64_t)gridDim.x * kLstmWarps * NB) {
    int32_t v[NB], tab[NB];
    bool has[NB];
#pragma unroll
    for (int n = 0; n < NB; ++n) {
      const bool act = base + n < p.n;
      v[n] = act ? (p.order ? __ldg(p.order + base + n) : (int32_t)(base + n)) : -1;
      tab[n] = (act && lane < T) ? __ldg(p.table + (int64_t)v[n] * T + lane) : -1;
      has[n] = __shfl_sync(0xffffffffu, tab[n], 0) >= 0;
      hb[warp][n][lane] = 0.0f;
    }
    float c[NB];
    float4 cur[NB], nxt[NB];
#pragma unroll
    for (int n = 0; n < NB; ++n) {
      c[n] = 0.0f;
      const int32_t u = __shfl_sync(0xffffffffu, tab[n], 0);
      cur[n] = u >= 0 ? __ldg(reinterpret_cast<const float4 *>(p.GS + (int64_t)u * p.ldg) + lane)
                      : make_float4(0.f, 0.f, 0.f, 0.f);
    }
    __syncwarp();
    for (int t = 0; t < T; ++t) {
      // sparse fetch of the next cell's rows while this cell computes
#pragma unroll
      for (int n = 0; n < NB; ++n) {
        const int32_t u = t + 1 < T ? __shfl_sync(0xffffffffu, tab[n], t + 1) : -1;
        nxt[n] = u >= 0 ? __ldg(reinterpret_cast<const float4 *>(p.GS + (int64_t)u * p.ldg) + lane)
                        : make_float4(0.f, 0.f, 0.f, 0.f);
      }
      // gates = G[u_t] + R h_{t-1}  (k order, fp32 fma chain)
      float4 acc[NB];
#pragma unroll
      for (int n = 0; n < NB; ++n) acc[n] = cur[n];
#pragma unroll 2
      for (int k = 0; k < F; k += 4) {
        const float4 r0 = Rt[k][lane], r1 = Rt[k + 1][lane], r2 = Rt[k + 2][lane], r3 = Rt[k + 3][lane];
#pragma unroll
        for (int n = 0; n < NB; ++n) {
          const float4 h4 = *reinterpret_cast<const float4 *>(&hb[warp][n][k]);
          // the same fmaf chains as pairs of packed FMAs (FFMA2, bit-identical)
          fma2_bcast(acc[n].x, acc[n].y, r0.x, r0.y, h4.x);
          fma2_bcast(acc[n].z, acc[n].w, r0.z, r0.w, h4.x);
          fma2_bcast(acc[n].x, acc[n].y, r1.x, r1.y, h4.y);
          fma2_bcast(acc[n].z, acc[n].w, r1.z, r1.w, h4.y);
          fma2_bcast(acc[n].x, acc[n].y, r2.x, r2.y, h4.z);
          fma2_bcast(acc[n].z, acc[n].w, r2.z, r2.w, h4.z);
          fma2_bcast(acc[n].x, acc[n].y, r3.x, r3.y, h4.w);
          fma2_bcast(acc[n].z, acc[n].w, r3.z, r3.w, h4.w);
        }
      }
      __syncwarp();
      // element-wise cell (Fig 6): i, f, o sigmoid; z tanh; c = f c + i z; h = o tanh(c)
#pragma unroll
      for (int n = 0; n < NB; ++n) {
        if (!has[n]) continue;
        const float ig = sigm(acc[n].x), fg = sigm(acc[n].y), zg = tanh_f(acc[n].z), og = sigm(acc[n].w);
        c[n] = fmaf(fg, c[n], ig * zg);
        hb[warp][n][lane] = og * tanh_f(c[n]);
      }
#pragma unroll
      for (int n = 0; n < NB; ++n) cur[n] = nxt[n];
      __syncwarp();
    }
    // SAGE combine: y_v = S_v + W_neigh h_T(v)
#pragma unroll
    for (int n = 0; n < NB; ++n) {
      if (v[n] < 0 || lane >= p.F_out) continue;
      float y = __ldg(p.GS + (int64_t)v[n] * p.ldg + 4 * F + lane);
#pragma unroll 8
      for (int j = 0; j < F; ++j) y = fmaf(Wnt[j][lane], hb[warp][n][j], y);
      p.Y[(int64_t)v[n] * p.ldy + lane] = y;
    }
    __syncwarp();
  }
}

cudaError_t launch_sage_lstm(const gnn_plan_s *p, const int32_t *table, int32_t T, const float *GS, int64_t ldg,
                             const float *R, const float *Wn, int32_t F_out, float *Y, int64_t ldy, cudaStream_t s) {
  if (p->n == 0) return cudaSuccess;
  LstmParams kp{table, T, GS, ldg, R, Wn, F_out, Y, ldy, p->dg.perm, p->n};
  static int occ = 0;
  if (occ == 0) {
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_sage_lstm, kLstmWarps * 32, 0);
    if (occ <= 0) occ = 1;
  }
  const int64_t per_cta = (int64_t)kLstmWarps * kLstmNB;
  const int64_t blocks = std::min<int64_t>((p->n + per_cta - 1) / per_cta, (int64_t)num_sms() * occ);
  k_sage_lstm<<<(unsigned)blocks, kLstmWarps * 32, 0, s>>>(kp);
  count_launch();
  return cudaGetLastError();
}

}  // namespace gnn
