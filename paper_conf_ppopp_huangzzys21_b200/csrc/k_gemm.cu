// k_gemm.cu — a5 dense transform H = X W (Eq 1 "(x) W")
// with fused epilogue (row scale, column bias, ReLU).
//
// Two implementations behind one entry point:
//   - SIMT fp32 FFMA (exact fp32 products, fp32 accumulate) — the fallback for
//     shapes the tensor-core path does not take (tiny, unaligned);
//   - tcgen05 3xTF32 (k_gemm_tc.cu) — hi/lo split so the tensor cores deliver
//     fp32 accuracy (plain TF32 fails 1e-4).
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>

#include "gnn_internal.h"

namespace gnn {

namespace {
constexpr int BM = 128, BN = 64, BK = 8;
constexpr int TM = 8, TN = 4;  // per-thread micro tile (256 threads = 16 x 16)
}  // namespace

__global__ void __launch_bounds__(256) k_gemm_simt(const float *__restrict__ X, int64_t ldx,
                                                   const float *__restrict__ W, int64_t ldw,
                                                   float *__restrict__ H, int64_t ldh, int64_t m,
                                                   int32_t k, int32_t n,
                                                   const float *__restrict__ row_scale,
                                                   const float *__restrict__ col_bias, int32_t relu) {
  __shared__ float As[2][BK][BM + 4];
  __shared__ float Bs[2][BK][BN];
  const int tid = threadIdx.x;
  const int tx = tid % 16, ty = tid / 16;
  const int64_t row0 = (int64_t)blockIdx.y * BM;
  const int32_t col0 = blockIdx.x * BN;
  float acc[TM][TN];
#pragma unroll
  for (int i = 0; i < TM; ++i)
#pragma unroll
    for (int j = 0; j < TN; ++j) acc[i][j] = 0.0f;

  // loaders: A 128x8 (4 per thread), B 8x64 (2 per thread)
  float ra[4], rb[2];
  auto load_tile = [&](int32_t k0) {
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int e = tid + q * 256;  // 0..1023
      const int r = e / BK, c = e % BK;
      const int64_t gr = row0 + r;
      const int32_t gc = k0 + c;
      ra[q] = (gr < m && gc < k) ? __ldg(X + gr * ldx + gc) : 0.0f;
    }
#pragma unroll
    for (int q = 0; q < 2; ++q) {
      const int e = tid + q * 256;  // 0..511
      const int r = e / BN, c = e % BN;
      const int32_t gr = k0 + r, gc = col0 + c;
      rb[q] = (gr < k && gc < n) ? __ldg(W + (int64_t)gr * ldw + gc) : 0.0f;
    }
  };
  auto store_tile = [&](int buf) {
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int e = tid + q * 256;
      As[buf][e % BK][e / BK] = ra[q];
    }
#pragma unroll
    for (int q = 0; q < 2; ++q) {
      const int e = tid + q * 256;
      Bs[buf][e / BN][e % BN] = rb[q];
    }
  };
  load_tile(0);
  store_tile(0);
  __syncthreads();
  int buf = 0;
  for (int32_t k0 = 0; k0 < k; k0 += BK) {
    const bool more = k0 + BK < k;
    if (more) load_tile(k0 + BK);
#pragma unroll
    for (int kk = 0; kk < BK; ++kk) {
      float a[TM], b[TN];
#pragma unroll
      for (int i = 0; i < TM; ++i) a[i] = As[buf][kk][ty * TM + i];
#pragma unroll
      for (int j = 0; j < TN; ++j) b[j] = Bs[buf][kk][tx * TN + j];
#pragma unroll
      for (int i = 0; i < TM; ++i)
#pragma unroll
        for (int j = 0; j < TN; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
    }
    if (more) {
      store_tile(buf ^ 1);
      __syncthreads();
      buf ^= 1;
    }
  }
#pragma unroll
  for (int i = 0; i < TM; ++i) {
    const int64_t gr = row0 + ty * TM + i;
    if (gr >= m) continue;
    const float sc = row_scale ? row_scale[gr] : 1.0f;
#pragma unroll
    for (int j = 0; j < TN; ++j) {
      const int32_t gc = col0 + tx * TN + j;
      if (gc >= n) continue;
      float y = acc[i][j];
      if (row_scale) y = y * sc;
      if (col_bias) y = y + col_bias[gc];
      if (relu) y = y > 0.0f ? y : 0.0f;
      H[gr * ldh + gc] = y;
    }
  }
}

static int g_gemm_impl = 0;  // 0 auto, 1 simt, 2 tcgen05, 3 tcgen05 with register-fed X tiles

void gemm_tc_set_tma(int on);  // k_gemm_tc.cu

int set_gemm_impl(int impl) {
  int old = g_gemm_impl;
  g_gemm_impl = impl;
  gemm_tc_set_tma(impl != 3);
  return old;
}

// implemented in k_gemm_tc.cu; returns cudaErrorNotSupported when the shape
// is outside what the tcgen05 kernel takes
cudaError_t launch_gemm_tc(const float *X, int64_t ldx, const float *W, int64_t ldw, float *H,
                           int64_t ldh, int64_t m, int32_t k, int32_t n, const float *row_scale,
                           const float *col_bias, int32_t relu, void *ws, size_t ws_bytes, cudaStream_t s,
                           const GemmMirrors *mir);

gnn_status launch_gemm(const float *X, int64_t ldx, const float *W, int64_t ldw, float *H,
                       int64_t ldh, int64_t m, int32_t k, int32_t n, const float *row_scale,
                       const float *col_bias, int32_t relu, void *ws, size_t ws_bytes, cudaStream_t s,
                       const GemmMirrors *mir) {
  if (m == 0 || n == 0) return GNN_OK;
  if (mir && mir->count > 0 && (g_gemm_impl == 1 || !ws || k < 1)) {
    set_error("mirrored GEMM: only the tcgen05 TMA-store epilogue writes mirrors (pass a workspace)");
    return GNN_ERR_UNSUPPORTED;
  }
  if (g_gemm_impl != 1 && ws != nullptr && k > 0) {
    // a caller that passes a workspace gets the tensor cores or an error,
    // never a silent fallback (every n is taken, wide ones as column slices)
    cudaError_t e = launch_gemm_tc(X, ldx, W, ldw, H, ldh, m, k, n, row_scale, col_bias, relu, ws, ws_bytes, s, mir);
    if (e == cudaSuccess) return GNN_OK;
    if (e == cudaErrorInvalidValue) {
      set_error("gemm workspace too small: need gnn_gemm_workspace_size(m, k, n) = " +
                std::to_string(gemm_tc_workspace(m, k, n)) + " bytes");
      return GNN_ERR_WORKSPACE;
    }
    if (e != cudaErrorNotSupported) return cuda_status(e, "gemm tcgen05 launch");
    if (mir && mir->count > 0) {
      set_error("mirrored GEMM: needs the TMA-store epilogue (16-byte aligned X, H, mirrors and leading dimensions)");
      return GNN_ERR_UNSUPPORTED;
    }
    set_error("tcgen05 GEMM: workspace must be 16-byte aligned");
    return GNN_ERR_INVALID_ARG;
  } else if (g_gemm_impl >= 2 && k > 0) {
    set_error("tcgen05 GEMM needs a workspace (gnn_gemm_workspace_size)");
    return GNN_ERR_UNSUPPORTED;
  }
  dim3 grid((n + BN - 1) / BN, (unsigned)((m + BM - 1) / BM));
  if (grid.y > 65535u) {
    // fold very tall problems into several launches
    const int64_t rows_per = (int64_t)65535 * BM;
    for (int64_t r0 = 0; r0 < m; r0 += rows_per) {
      const int64_t mm = std::min<int64_t>(rows_per, m - r0);
      dim3 g2(grid.x, (unsigned)((mm + BM - 1) / BM));
      k_gemm_simt<<<g2, 256, 0, s>>>(X + r0 * ldx, ldx, W, ldw, H + r0 * ldh, ldh, mm, k, n,
                                      row_scale ? row_scale + r0 : nullptr, col_bias, relu);
      count_launch();
    }
  } else {
    k_gemm_simt<<<grid, 256, 0, s>>>(X, ldx, W, ldw, H, ldh, m, k, n, row_scale, col_bias, relu);
    count_launch();
  }
  return cuda_status(cudaGetLastError(), "gemm launch");
}

}  // namespace gnn
