// stream_bench_k.cu — dev experiment kernels (not part of libgnn.so): how
// fast can the C5 gather stream go on this GPU, independent of the
// aggregation kernel's structure?
//   sb_stream: warps take contiguous chunks of the task-ordered index stream
//              and sum the gathered rows (no row logic) -> memory-system bound
//              for this exact access pattern (its L2 reuse included)
//   sb_rows:   same, but rows are respected: a warp processes whole rows
//              (dynamic: atomicAdd on a row counter, rows in task order) and
//              writes each row's sum (the minimal structured kernel)
#include <cuda_runtime.h>
#include <stdint.h>

__device__ __forceinline__ void ld8(const float *p, float (&v)[8]) {
  asm volatile("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]), "=f"(v[6]), "=f"(v[7])
               : "l"(p));
}

template <int U>
__global__ void __launch_bounds__(256) sb_stream(const float *X, const int32_t *idx, int64_t nnz, int64_t chunk,
                                                 float *out) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t b0 = warp * chunk, b1 = min(b0 + chunk, nnz);
  float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  for (int64_t k = b0; k < b1; k += 32) {
    const int cnt = (int)min((int64_t)32, b1 - k);
    const int32_t my = lane < cnt ? idx[k + lane] : 0;
    float v[U][8];
#pragma unroll
    for (int q = 0; q < U; ++q)
      if (q < cnt) ld8(X + (int64_t)__shfl_sync(0xffffffff, my, q) * 256 + lane * 8, v[q]);
    for (int j = 0; j < cnt; j += U) {
#pragma unroll
      for (int q = 0; q < U; ++q) {
        if (j + q < cnt) {
#pragma unroll
          for (int i = 0; i < 8; ++i) acc[i] += v[q][i];
          if (j + q + U < cnt) ld8(X + (int64_t)__shfl_sync(0xffffffff, my, j + q + U) * 256 + lane * 8, v[q]);
        }
      }
    }
  }
  float s = 0;
  for (int i = 0; i < 8; ++i) s += acc[i];
  if (s == 12345.f) out[0] = s;
}

template <int U>
__global__ void __launch_bounds__(256) sb_rows(const float *X, const int32_t *idx, const int64_t *tptr,
                                               const int32_t *trow, int64_t nrows, int32_t *ctr, float *Y) {
  const int lane = threadIdx.x & 31;
  for (;;) {
    int64_t r = 0;
    if (lane == 0) r = atomicAdd(ctr, 1);
    r = __shfl_sync(0xffffffff, r, 0);
    if (r >= nrows) break;
    const int64_t b0 = tptr[r], b1 = tptr[r + 1];
    float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    for (int64_t k = b0; k < b1; k += 32) {
      const int cnt = (int)min((int64_t)32, b1 - k);
      const int32_t my = lane < cnt ? idx[k + lane] : 0;
      float v[U][8];
#pragma unroll
      for (int q = 0; q < U; ++q)
        if (q < cnt) ld8(X + (int64_t)__shfl_sync(0xffffffff, my, q) * 256 + lane * 8, v[q]);
      for (int j = 0; j < cnt; j += U) {
#pragma unroll
        for (int q = 0; q < U; ++q) {
          if (j + q < cnt) {
#pragma unroll
            for (int i = 0; i < 8; ++i) acc[i] += v[q][i];
            if (j + q + U < cnt) ld8(X + (int64_t)__shfl_sync(0xffffffff, my, j + q + U) * 256 + lane * 8, v[q]);
          }
        }
      }
    }
    float *y = Y + (int64_t)trow[r] * 256 + lane * 8;
    *reinterpret_cast<float4 *>(y) = make_float4(acc[0], acc[1], acc[2], acc[3]);
    *reinterpret_cast<float4 *>(y + 4) = make_float4(acc[4], acc[5], acc[6], acc[7]);
  }
}

extern "C" int sb_run_stream(const float *X, const int32_t *idx, int64_t nnz, int64_t chunk, int U, int blocks,
                             float *out) {
  if (U == 2) sb_stream<2><<<blocks, 256>>>(X, idx, nnz, chunk, out);
  if (U == 4) sb_stream<4><<<blocks, 256>>>(X, idx, nnz, chunk, out);
  if (U == 8) sb_stream<8><<<blocks, 256>>>(X, idx, nnz, chunk, out);
  return (int)cudaGetLastError();
}

extern "C" int sb_run_rows(const float *X, const int32_t *idx, const int64_t *tptr, const int32_t *trow,
                           int64_t nrows, int32_t *ctr, int U, int blocks, float *Y) {
  cudaMemset(ctr, 0, 4);
  if (U == 2) sb_rows<2><<<blocks, 256>>>(X, idx, tptr, trow, nrows, ctr, Y);
  if (U == 4) sb_rows<4><<<blocks, 256>>>(X, idx, tptr, trow, nrows, ctr, Y);
  if (U == 8) sb_rows<8><<<blocks, 256>>>(X, idx, tptr, trow, nrows, ctr, Y);
  return (int)cudaGetLastError();
}
