// gather_bench.cu — dev micro-benchmark: achievable bandwidth of random row
// gathers on this GPU (the roofline the aggregation kernel can approach).
// Each warp sums R random rows of F fp32 (one 256-bit load per lane per row
// for F = 256), U rows in flight per warp.  Indices come from a precomputed
// array (like colidx) or from an inline hash (no index traffic).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 gather_bench.cu -o gather_bench
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ void ld8(const float *p, float (&v)[8]) {
  asm volatile("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]), "=f"(v[4]), "=f"(v[5]), "=f"(v[6]), "=f"(v[7])
               : "l"(p));
}

template <int U>
__global__ void __launch_bounds__(256) gather(const float *X, int64_t nrows, const int32_t *idx, int64_t nidx,
                                              int per_warp, float *out) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t base = warp * per_warp;
  float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
  float v[U][8];
  int32_t my = 0;
  for (int j0 = 0; j0 < per_warp; j0 += 32) {
    my = idx[(base + j0 + lane) % nidx];
#pragma unroll
    for (int q = 0; q < U; ++q) ld8(X + (int64_t)__shfl_sync(0xffffffff, my, q) * 256 + lane * 8, v[q]);
    for (int j = 0; j < 32; j += U) {
#pragma unroll
      for (int q = 0; q < U; ++q) {
#pragma unroll
        for (int i = 0; i < 8; ++i) acc[i] += v[q][i];
        if (j + q + U < 32) ld8(X + (int64_t)__shfl_sync(0xffffffff, my, j + q + U) * 256 + lane * 8, v[q]);
      }
    }
  }
  float s = 0;
  for (int i = 0; i < 8; ++i) s += acc[i];
  if (s == 12345.f) out[0] = s;
}

int main() {
  const int64_t nrows = 2449029;  // products-shaped, F = 256 -> 2.5 GB
  float *X;
  int32_t *idx;
  float *out;
  cudaMalloc(&X, nrows * 256 * 4);
  cudaMemset(X, 0, nrows * 256 * 4);
  const int64_t nidx = 1 << 26;
  cudaMalloc(&idx, nidx * 4);
  cudaMalloc(&out, 4);
  int32_t *h = (int32_t *)malloc(nidx * 4);
  uint64_t st = 12345;
  for (int64_t i = 0; i < nidx; ++i) {
    st = st * 6364136223846793005ULL + 1442695040888963407ULL;
    h[i] = (int32_t)((st >> 33) % nrows);
  }
  cudaMemcpy(idx, h, nidx * 4, cudaMemcpyHostToDevice);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const int per_warp = 2048;
  for (int which = 0; which < 2; ++which) {
    // which 0: random over 2.5 GB (DRAM); which 1: random over the first 100 MB (L2-resident)
    if (which == 1) {
      for (int64_t i = 0; i < nidx; ++i) h[i] = h[i] % 97656;
      cudaMemcpy(idx, h, nidx * 4, cudaMemcpyHostToDevice);
    }
    for (int blocks_per_sm : {1, 2, 4, 8}) {
      for (int U : {2, 4, 8}) {
        const int blocks = 148 * blocks_per_sm * 4;  // 4 waves
        const int64_t rows = (int64_t)blocks * 8 * per_warp;
        for (int rep = 0; rep < 2; ++rep) {
          cudaEventRecord(a);
          if (U == 2) gather<2><<<blocks, 256>>>(X, nrows, idx, nidx, per_warp, out);
          if (U == 4) gather<4><<<blocks, 256>>>(X, nrows, idx, nidx, per_warp, out);
          if (U == 8) gather<8><<<blocks, 256>>>(X, nrows, idx, nidx, per_warp, out);
          cudaEventRecord(b);
          cudaEventSynchronize(b);
        }
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        int occ = 0;
        if (U == 2) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, gather<2>, 256, 0);
        if (U == 4) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, gather<4>, 256, 0);
        if (U == 8) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, gather<8>, 256, 0);
        printf("%s blocks/SM(req)=%d occ=%d U=%d: %.3f ms  %.0f GB/s (row bytes)\n", which ? "L2 " : "HBM",
               blocks_per_sm, occ, U, ms, rows * 1024.0 / (ms * 1e-3) / 1e9);
      }
    }
  }
  printf("err=%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
