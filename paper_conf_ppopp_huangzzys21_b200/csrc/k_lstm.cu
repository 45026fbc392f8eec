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
#include "tc_common.cuh"

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
// 1/x for x in [1, 2^64] on the FMA pipe: integer seed (relative error < 1/8)
// and three Newton steps (error < (1/8)^8 ~ 6e-8).  The SIMT cells keep
// rcp.approx (measured: Newton 10.8 ms vs 9.8 ms — they are issue-bound, not
// MUFU-bound); the tensor-core cells use it (FMA pipe otherwise idle).
__device__ __forceinline__ float rcp_nr(float x) {
  float r = __int_as_float(0x7EF311C7 - __float_as_int(x));
  r = r * fmaf(-x, r, 2.0f);
  r = r * fmaf(-x, r, 2.0f);
  r = r * fmaf(-x, r, 2.0f);
  return r;
}
#ifndef GNN_LSTM_RCP_NR
#define GNN_LSTM_RCP_NR 0
#endif
__device__ __forceinline__ float rcp_sel(float x) { return GNN_LSTM_RCP_NR ? rcp_nr(x) : rcp_s(x); }
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

// ---------------------------------------------------------------------------
// k_sage_lstm_tc: the recurrent product on the tensor cores.  One CTA = 128
// center nodes (thread r = node r = TMEM lane r).  Per cell t >= 1 one thread
// issues D[128 x 128] = h_{t-1}[128 x 32] R^T[32 x 128] as 3xTF32
// tcgen05.mma (A = h split hi/lo, B = R split hi/lo, both K-major SW128 in
// shared memory; D in 128 TMEM columns, column 4j+g = gate g of unit j).
// Every thread then reads its node's 128 gate sums from TMEM (4 chunks of 32
// columns), adds the sparse-fetched row GS[u_t] (prefetched), runs the 32
// element-wise cells (c in registers) and writes h_t back into the A tiles
// for the next cell.  After T cells: y = S_v + W_neigh h_T (SIMT, W_neigh^T
// in shared memory).
// ---------------------------------------------------------------------------
namespace {
constexpr int kTcTileBytes = 128 * 128;  // 128 rows x 32 fp32 (one SW128 row each)

__device__ __forceinline__ float ex2_l(float x) {
  float r;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(x));
  return r;
}
constexpr float kL2e = 1.4426950408889634f;
// 2^x on the FMA pipe (the MUFU/XU pipe is the cells' bottleneck): x = r + f,
// r = round(x), f in [-0.5, 0.5]; 2^f by its degree-6 Taylor polynomial
// (relative error < 2e-7); 2^r added to the exponent bits.  |x| clamped to 126.
__device__ __forceinline__ float ex2_fma(float x) {
  x = fminf(fmaxf(x, -126.0f), 126.0f);
  const float big = x + 12582912.0f;  // 1.5 * 2^23: round to nearest integer in the low mantissa bits
  const float r = big - 12582912.0f;
  const float f = x - r;
  float q = 1.5403530393381606e-4f;
  q = fmaf(q, f, 1.3333558146428443e-3f);
  q = fmaf(q, f, 9.6181291076284772e-3f);
  q = fmaf(q, f, 5.5504108664821580e-2f);
  q = fmaf(q, f, 2.4022650695910071e-1f);
  q = fmaf(q, f, 6.9314718055994531e-1f);
  q = fmaf(q, f, 1.0f);
  return __int_as_float(__float_as_int(q) + ((__float_as_int(big) - 0x4B400000) << 23));
}
#ifndef GNN_LSTM_EX2_FMA
#define GNN_LSTM_EX2_FMA 1
#endif
__device__ __forceinline__ float ex2_sel(float x) { return GNN_LSTM_EX2_FMA ? ex2_fma(x) : ex2_l(x); }
// tensor-core cells: the FMA pipe is free, so both ex2 (polynomial) and the
// reciprocal (Newton) run there; arguments clamped to <= 64 (see rcp_nr)
__device__ __forceinline__ float sig_tc(float x) { return rcp_nr(1.0f + ex2_sel(fminf(-kL2e * x, 64.0f))); }
__device__ __forceinline__ float tanh_tc(float x) {
  return fmaf(2.0f, rcp_nr(1.0f + ex2_sel(fminf(-2.0f * kL2e * x, 64.0f))), -1.0f);
}
}  // namespace

constexpr int kTcGroups = 3;  // independent 128-node tiles per CTA (12 warps), sharing R and W_neigh

// named barrier of one 128-thread group
__device__ __forceinline__ void group_sync(int g) { asm volatile("bar.sync %0, 128;" ::"r"(g + 1) : "memory"); }

__global__ void __launch_bounds__(128 * kTcGroups, 1) k_sage_lstm_tc(const LstmParams p) {
  using namespace tc;
  constexpr int F = kLstmF;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t *smem = (uint8_t *)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  const int grp = threadIdx.x >> 7;          // this thread's group (tile)
  const int tid = threadIdx.x & 127, warp = tid >> 5;
  uint8_t *b_hi = smem, *b_lo = smem + kTcTileBytes;
  uint8_t *a_hi = smem + (2 + 2 * grp) * kTcTileBytes, *a_lo = a_hi + kTcTileBytes;
  float *Wnt = reinterpret_cast<float *>(smem + (2 + 2 * kTcGroups) * kTcTileBytes);  // Wnt[j*F + o] = W_neigh[o][j]
  __shared__ uint64_t mma_bar_all[kTcGroups];
  __shared__ uint32_t tmem_base_sh;
  uint64_t &mma_bar = mma_bar_all[grp];
  // B = R^T as K-major rows: row n = 4j + g holds R[g*F + j][0..31], split hi/lo
  for (int q = threadIdx.x; q < 128 * 8; q += blockDim.x) {
    const int n = q >> 3, c = q & 7;
    const int j = n >> 2, g = n & 3;
    const float *src = p.R + (int64_t)(g * F + j) * F + 4 * c;
    const float4 w = make_float4(src[0], src[1], src[2], src[3]);
    const float4 hi = make_float4(hi_of(w.x), hi_of(w.y), hi_of(w.z), hi_of(w.w));
    const float4 lo = make_float4(w.x - hi.x, w.y - hi.y, w.z - hi.z, w.w - hi.w);
    *reinterpret_cast<float4 *>(b_hi + sw128_off(n, c)) = hi;
    *reinterpret_cast<float4 *>(b_lo + sw128_off(n, c)) = lo;
  }
  for (int q = threadIdx.x; q < F * F; q += blockDim.x) {
    const int j = q / F, o = q % F;
    Wnt[q] = o < p.F_out ? p.Wn[o * F + j] : 0.0f;
  }
  if (threadIdx.x == 0) {
    for (int g = 0; g < kTcGroups; ++g) mbar_init(&mma_bar_all[g], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (threadIdx.x < 32) {  // 512 TMEM columns: 128 per group
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tmem_base_sh)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem_all = tmem_base_sh;
  const uint32_t tmem = tmem_all + 128u * grp;                   // this group's 128 accumulator columns
  const uint32_t taddr0 = tmem + ((uint32_t)(warp * 32) << 16);  // this warp's TMEM lane quadrant (warp id % 4)
  const uint32_t idesc = idesc_tf32(128);
  const int T = p.T;
  const int64_t ntiles = (p.n + 127) / 128;
  uint32_t phase = 0;
  for (int64_t tile = (int64_t)blockIdx.x * kTcGroups + grp; tile < ntiles; tile += (int64_t)gridDim.x * kTcGroups) {
    const int64_t idx = tile * 128 + tid;
    const bool act = idx < p.n;
    const int32_t v = act ? (p.order ? __ldg(p.order + idx) : (int32_t)idx) : -1;
    const int32_t *tab = p.table + (int64_t)(act ? v : 0) * T;
    int32_t u = act ? __ldg(tab) : -1;
    const bool has = u >= 0;
    float c[F];
#pragma unroll
    for (int j = 0; j < F; ++j) c[j] = 0.0f;
    // first gathered chunk of the current cell (prefetched one cell ahead)
    float4 g0[8];
    auto load_chunk = [&](int32_t uu, int q, float4 (&dst)[8]) {
      const float4 *src = reinterpret_cast<const float4 *>(p.GS + (int64_t)(uu >= 0 ? uu : 0) * p.ldg) + 8 * q;
#pragma unroll
      for (int i = 0; i < 8; ++i) dst[i] = uu >= 0 ? __ldg(src + i) : make_float4(0.f, 0.f, 0.f, 0.f);
    };
    load_chunk(u, 0, g0);
    for (int t = 0; t < T; ++t) {
      const int32_t un = (has && t + 1 < T) ? __ldg(tab + t + 1) : -1;
      if (t > 0 && tid == 0) {
        asm volatile("tcgen05.fence::after_thread_sync;");
        const uint32_t ah = smem_u32(a_hi), al = smem_u32(a_lo), bh = smem_u32(b_hi), bl = smem_u32(b_lo);
#pragma unroll
        for (int ks = 0; ks < 4; ++ks) {  // K = 32 in steps of 8 tf32 (32 B)
          const uint32_t ko = ks * 32;
          mma_tf32(tmem, sw128_desc(al + ko), sw128_desc(bh + ko), idesc, ks > 0 ? 1u : 0u);
          mma_tf32(tmem, sw128_desc(ah + ko), sw128_desc(bl + ko), idesc, 1u);
          mma_tf32(tmem, sw128_desc(ah + ko), sw128_desc(bh + ko), idesc, 1u);
        }
        mma_commit(&mma_bar);
      }
      if (t > 0) {
        mbar_wait(&mma_bar, phase);
        phase ^= 1u;
        asm volatile("tcgen05.fence::after_thread_sync;");
      }
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        float4 gq[8], gn[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) gq[i] = g0[i];
        // the next chunk of this cell (or the first chunk of the next cell) is in flight during this one
        if (q < 3) load_chunk(has ? u : -1, q + 1, gn);
        else load_chunk(un, 0, gn);
        float acc[32];
        if (t > 0) {
          tmem_ld32(taddr0 + 32 * q, acc);
        } else {
#pragma unroll
          for (int i = 0; i < 32; ++i) acc[i] = 0.0f;
        }
        float hv[8];
#pragma unroll
        for (int jj = 0; jj < 8; ++jj) {
          const int j = 8 * q + jj;
          const float4 gg = gq[jj];
          const float ig = sig_tc(acc[4 * jj + 0] + gg.x);
          const float fg = sig_tc(acc[4 * jj + 1] + gg.y);
          const float zg = tanh_tc(acc[4 * jj + 2] + gg.z);
          const float og = sig_tc(acc[4 * jj + 3] + gg.w);
          c[j] = has ? fmaf(fg, c[j], ig * zg) : 0.0f;
          hv[jj] = has ? og * tanh_tc(c[j]) : 0.0f;
        }
        // h_t units 8q..8q+7 -> A (row tid, 16-byte chunks 2q and 2q+1), split hi/lo
#pragma unroll
        for (int h2 = 0; h2 < 2; ++h2) {
          const float4 h4 = make_float4(hv[4 * h2], hv[4 * h2 + 1], hv[4 * h2 + 2], hv[4 * h2 + 3]);
          const float4 hi = make_float4(hi_of(h4.x), hi_of(h4.y), hi_of(h4.z), hi_of(h4.w));
          const float4 lo = make_float4(h4.x - hi.x, h4.y - hi.y, h4.z - hi.z, h4.w - hi.w);
          *reinterpret_cast<float4 *>(a_hi + sw128_off(tid, 2 * q + h2)) = hi;
          *reinterpret_cast<float4 *>(a_lo + sw128_off(tid, 2 * q + h2)) = lo;
        }
#pragma unroll
        for (int i = 0; i < 8; ++i) g0[i] = gn[i];
      }
      u = un;
      // A complete and every TMEM read done before the next cell's MMA
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      asm volatile("tcgen05.fence::before_thread_sync;");
      group_sync(grp);
    }
    // SAGE combine: y_v = S_v + W_neigh h_T (h_T = hi + lo from the A tiles, exact)
    if (act) {
      float h[F];
#pragma unroll
      for (int c4 = 0; c4 < 8; ++c4) {
        const float4 hi = *reinterpret_cast<const float4 *>(a_hi + sw128_off(tid, c4));
        const float4 lo = *reinterpret_cast<const float4 *>(a_lo + sw128_off(tid, c4));
        h[4 * c4 + 0] = hi.x + lo.x;
        h[4 * c4 + 1] = hi.y + lo.y;
        h[4 * c4 + 2] = hi.z + lo.z;
        h[4 * c4 + 3] = hi.w + lo.w;
      }
      const float *Sv = p.GS + (int64_t)v * p.ldg + 4 * F;
      float *yv = p.Y + (int64_t)v * p.ldy;
      for (int o = 0; o < p.F_out; ++o) {
        float y = __ldg(Sv + o);
#pragma unroll
        for (int j = 0; j < F; ++j) y = fmaf(Wnt[j * F + o], h[j], y);
        yv[o] = y;
      }
    }
    group_sync(grp);  // the A tiles are rewritten by the next tile
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.fence::after_thread_sync;");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem_all));
  }
}


// ---------------------------------------------------------------------------
// k_sage_lstm_mma: the recurrent product on warp-level tensor-core MMAs
// (mma.sync m16n8k8 TF32, 3xTF32 split) inside a SIMT-style layout.  One warp
// = 16 center nodes (the MMA's M).  Per cell, the warp computes the gate
// pre-activations D[16 x 128] = G[u_t] + h_{t-1} R^T as 16 n-tiles of 8
// columns (gate column 4j+g); the accumulator fragments are initialised with
// the sparse-fetched rows G[u_t] (each lane loads 8 B of two rows per tile,
// so a warp instruction reads 32 B of 8 rows), h_{t-1} comes from a per-warp
// shared buffer as A fragments (hi/lo), R^T fragments from shared memory
// (pre-split, one float4 per lane per (tile, k-step)).  A lane pair
// (tig, tig^1) holds the four gates of one unit for two rows; one xor-shuffle
// each gives every lane its own (row, unit) cell.
// ---------------------------------------------------------------------------
constexpr int kMmaWarps = 4;

__device__ __forceinline__ void mma_tf32_16x8x8(float (&d)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
  asm volatile(
      "mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};"
      : "+f"(d[0]), "+f"(d[1]), "+f"(d[2]), "+f"(d[3])
      : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}

__device__ __forceinline__ float hi19(float x) { return __uint_as_float(__float_as_uint(x) & 0xFFFFE000u); }

__global__ void __launch_bounds__(kMmaWarps * 32) k_sage_lstm_mma(const LstmParams p) {
  constexpr int F = kLstmF;
  // B fragments of R^T per (n-tile, k-step, lane): (b0_hi, b1_hi, b0_lo, b1_lo)
  __shared__ float4 Bf[16][4][32];
  __shared__ float Wnt[F][F + 1];
  __shared__ float hb[kMmaWarps][16][F + 1];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int gid = lane >> 2, tig = lane & 3;
  for (int q = tid; q < 16 * 4 * 32; q += blockDim.x) {
    const int nt = q / 128, ks = (q / 32) % 4, l = q % 32;
    const int n = 8 * nt + (l >> 2);          // gate column (4j + g)
    const int j = n >> 2, g = n & 3;
    const int k0 = 8 * ks + (l & 3), k1 = k0 + 4;
    const float w0 = p.R[(g * F + j) * F + k0], w1 = p.R[(g * F + j) * F + k1];
    const float h0 = hi19(w0), h1 = hi19(w1);
    Bf[nt][ks][l] = make_float4(h0, h1, w0 - h0, w1 - h1);
  }
  for (int i = tid; i < F * F; i += blockDim.x) {
    const int j = i / F, o = i % F;
    Wnt[j][o] = o < p.F_out ? p.Wn[o * F + j] : 0.0f;
  }
  __syncthreads();
  const int T = p.T;
  float (*h)[F + 1] = hb[warp];
  for (int64_t base = ((int64_t)blockIdx.x * kMmaWarps + warp) * 16; base < p.n;
       base += (int64_t)gridDim.x * kMmaWarps * 16) {
    // rows gid and gid + 8 of this warp's 16 nodes
    int32_t v[2];
    bool has[2];
#pragma unroll
    for (int r = 0; r < 2; ++r) {
      const int64_t idx = base + gid + 8 * r;
      v[r] = idx < p.n ? (p.order ? __ldg(p.order + idx) : (int32_t)idx) : -1;
      has[r] = v[r] >= 0 && __ldg(p.table + (int64_t)v[r] * T) >= 0;
    }
    // this lane's cells: row (tig odd ? gid + 8 : gid), units 2nt + tig/2
    const int myr = tig & 1;
    float c[16];
#pragma unroll
    for (int nt = 0; nt < 16; ++nt) c[nt] = 0.0f;
    for (int i = lane; i < 16 * F; i += 32) h[i / F][i % F] = 0.0f;
    __syncwarp();
    for (int t = 0; t < T; ++t) {
      int32_t u[2];
#pragma unroll
      for (int r = 0; r < 2; ++r) u[r] = has[r] ? __ldg(p.table + (int64_t)v[r] * T + t) : -1;
      // A fragments of h_{t-1} (rows gid, gid+8; k = 8ks + tig, + 4), split hi/lo
      uint32_t ah[4][4], al[4][4];
#pragma unroll
      for (int ks = 0; ks < 4; ++ks) {
        const float x[4] = {h[gid][8 * ks + tig], h[gid + 8][8 * ks + tig], h[gid][8 * ks + tig + 4],
                            h[gid + 8][8 * ks + tig + 4]};
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const float hi = hi19(x[i]);
          ah[ks][i] = __float_as_uint(hi);
          al[ks][i] = __float_as_uint(x[i] - hi);
        }
      }
      __syncwarp();  // every lane has its A fragments before h is overwritten
#pragma unroll
      for (int nt = 0; nt < 16; ++nt) {
        // accumulator = the gathered pre-activations G[u] (2 columns x 2 rows)
        float d[4];
#pragma unroll
        for (int r = 0; r < 2; ++r) {
          float2 gg = make_float2(0.f, 0.f);
          if (u[r] >= 0) gg = __ldg(reinterpret_cast<const float2 *>(p.GS + (int64_t)u[r] * p.ldg + 8 * nt + 2 * tig));
          d[2 * r] = gg.x;
          d[2 * r + 1] = gg.y;
        }
        if (t > 0) {
#pragma unroll
          for (int ks = 0; ks < 4; ++ks) {
            const float4 b = Bf[nt][ks][lane];
            mma_tf32_16x8x8(d, al[ks], __float_as_uint(b.x), __float_as_uint(b.y));
            mma_tf32_16x8x8(d, ah[ks], __float_as_uint(b.z), __float_as_uint(b.w));
            mma_tf32_16x8x8(d, ah[ks], __float_as_uint(b.x), __float_as_uint(b.y));
          }
        }
        // lanes tig even hold (i, f), odd hold (z, o) of unit 2nt + tig/2 for rows gid (d0,d1), gid+8 (d2,d3):
        // even keeps row gid and receives (z, o) of row gid; odd keeps row gid+8 and receives (i, f)
        const float s0 = myr ? d[0] : d[2], s1 = myr ? d[1] : d[3];
        const float r0 = __shfl_xor_sync(0xffffffffu, s0, 1), r1 = __shfl_xor_sync(0xffffffffu, s1, 1);
        const float gi = myr ? r0 : d[0], gf = myr ? r1 : d[1];
        const float gz = myr ? d[2] : r0, go = myr ? d[3] : r1;
        const int j = 2 * nt + (tig >> 1);
        const int row = gid + 8 * myr;
        if (has[myr]) {
          c[nt] = fmaf(sigm(gf), c[nt], sigm(gi) * tanh_f(gz));
          h[row][j] = sigm(go) * tanh_f(c[nt]);
        }
      }
      __syncwarp();
    }
    // SAGE combine: lane o computes output o of the 16 nodes
#pragma unroll 1
    for (int r = 0; r < 16; ++r) {
      const int64_t idx = base + r;
      if (idx >= p.n || lane >= p.F_out) continue;
      const int32_t vv = p.order ? __ldg(p.order + idx) : (int32_t)idx;
      float y = __ldg(p.GS + (int64_t)vv * p.ldg + 4 * F + lane);
#pragma unroll 8
      for (int j = 0; j < F; ++j) y = fmaf(Wnt[j][lane], h[r][j], y);
      p.Y[(int64_t)vv * p.ldy + lane] = y;
    }
    __syncwarp();
  }
}

static int g_lstm_impl = 0;  // 0 = SIMT cells (default), 1 = tcgen05 cells, 2 = mma.sync cells
int set_lstm_impl(int impl) {
  const int old = g_lstm_impl;
  g_lstm_impl = impl;
  return old;
}

cudaError_t launch_sage_lstm(const gnn_plan_s *p, const int32_t *table, int32_t T, const float *GS, int64_t ldg,
                             const float *R, const float *Wn, int32_t F_out, float *Y, int64_t ldy, cudaStream_t s) {
  if (p->n == 0) return cudaSuccess;
  if (g_lstm_impl == 2) {
    LstmParams kp{table, T, GS, ldg, R, Wn, F_out, Y, ldy, p->dg.perm, p->n};
    static int occ = 0;
    if (occ == 0) {
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_sage_lstm_mma, kMmaWarps * 32, 0);
      if (occ <= 0) occ = 1;
    }
    const int64_t per_cta = (int64_t)kMmaWarps * 16;
    const int64_t blocks = std::min<int64_t>((p->n + per_cta - 1) / per_cta, (int64_t)num_sms() * occ);
    k_sage_lstm_mma<<<(unsigned)blocks, kMmaWarps * 32, 0, s>>>(kp);
    count_launch();
    return cudaGetLastError();
  }
  if (g_lstm_impl == 1) {
    LstmParams kp{table, T, GS, ldg, R, Wn, F_out, Y, ldy, p->dg.perm, p->n};
    const size_t smem = (2 + 2 * kTcGroups) * kTcTileBytes + sizeof(float) * kLstmF * kLstmF + 1024;
    static bool init = false;
    if (!init) {
      cudaError_t e = cudaFuncSetAttribute(k_sage_lstm_tc, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      if (e != cudaSuccess) return e;
      init = true;
    }
    const int64_t tiles = (p->n + 127) / 128;
    const int64_t blocks = std::min<int64_t>((tiles + kTcGroups - 1) / kTcGroups, (int64_t)num_sms());
    k_sage_lstm_tc<<<(unsigned)blocks, 128 * kTcGroups, smem, s>>>(kp);
    count_launch();
    return cudaGetLastError();
  }
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
