// gather_roofline.cu — dev micro-benchmark: the measured roofline of random
// row gathers on this B200 (one measured gather ceiling).
//
// Each warp sums rows X[idx[j]] (row = ROWB bytes: 1024 = F 256, 400 = F 100,
// 1056 = GAT 8x32 + 8 scores) for a long run of random indices, two ways:
//   reg : 128-bit / 256-bit ld.global.nc into registers, U rows in flight per
//         warp (the round-1 aggregation kernel's scheme)
//   bulk: cp.async.bulk (TMA 1-D bulk copy, UBLKCP) of each row into a per-warp
//         shared-memory ring of S slots, completion on an mbarrier per slot,
//         then LDS.128 into the accumulators (in-flight bytes bounded by
//         shared memory instead of registers)
// over three working sets: rows spread over 2.5 GB (HBM-bound), over 100 MB
// and over 24 MB (L2-resident, 126 MB L2).  Prints GB/s of gathered row bytes.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 gather_roofline.cu -o gather_roofline
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>

__device__ __forceinline__ uint32_t smem_u32(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int ROWB>
__device__ __forceinline__ void acc_row_gmem(const char *row, int lane, float4 (&a)[3]) {
#pragma unroll
  for (int k = 0; k < 3; ++k) {
    const int c = lane + 32 * k;
    if (c < ROWB / 16) {
      float4 v;
      asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                   : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
                   : "l"(row + 16 * c));
      a[k].x += v.x; a[k].y += v.y; a[k].z += v.z; a[k].w += v.w;
    }
  }
}

// register gather: U rows in flight per warp (loads issued U rows ahead)
template <int ROWB, int U>
__global__ void __launch_bounds__(256) k_reg(const char *X, const int32_t *idx, int64_t nidx, int per_warp,
                                             float *out) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t base = warp * per_warp;
  float4 a[3] = {};
  float4 v[U][3];
  for (int j0 = 0; j0 < per_warp; j0 += 32) {
    const int32_t my = idx[(base + j0 + lane) % nidx];
#pragma unroll
    for (int q = 0; q < U; ++q) {
      const char *r = X + (int64_t)__shfl_sync(~0u, my, q) * ROWB;
#pragma unroll
      for (int k = 0; k < 3; ++k)
        if (lane + 32 * k < ROWB / 16)
          asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                       : "=f"(v[q][k].x), "=f"(v[q][k].y), "=f"(v[q][k].z), "=f"(v[q][k].w)
                       : "l"(r + 16 * (lane + 32 * k)));
    }
    for (int j = 0; j < 32; j += U) {
#pragma unroll
      for (int q = 0; q < U; ++q) {
#pragma unroll
        for (int k = 0; k < 3; ++k) {
          a[k].x += v[q][k].x; a[k].y += v[q][k].y; a[k].z += v[q][k].z; a[k].w += v[q][k].w;
        }
        if (j + q + U < 32) {
          const char *r = X + (int64_t)__shfl_sync(~0u, my, j + q + U) * ROWB;
#pragma unroll
          for (int k = 0; k < 3; ++k)
            if (lane + 32 * k < ROWB / 16)
              asm volatile("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
                           : "=f"(v[q][k].x), "=f"(v[q][k].y), "=f"(v[q][k].z), "=f"(v[q][k].w)
                           : "l"(r + 16 * (lane + 32 * k)));
        }
      }
    }
  }
  float s = 0;
  for (int k = 0; k < 3; ++k) s += a[k].x + a[k].y + a[k].z + a[k].w;
  if (s == 12345.f) out[0] = s;
}

// bulk-copy gather: per-warp ring of S row slots in shared memory
template <int ROWB, int S, int WARPS>
__global__ void __launch_bounds__(WARPS * 32) k_bulk(const char *X, const int32_t *idx, int64_t nidx, int per_warp,
                                                     float *out) {
  constexpr int SLOT = (ROWB + 127) / 128 * 128;
  extern __shared__ __align__(128) char smem[];
  __shared__ uint64_t bar[WARPS][S];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  char *ring = smem + (size_t)w * S * SLOT;
  if (lane == 0)
    for (int s = 0; s < S; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar[w][s])));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t base = warp * per_warp;
  auto issue = [&](int32_t u, int s) {
    const uint32_t b = smem_u32(&bar[w][s]);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(ROWB) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(ring + s * SLOT)),
                 "l"(X + (int64_t)u * ROWB), "r"(ROWB), "r"(b)
                 : "memory");
  };
  int32_t cur = idx[(base + lane) % nidx];          // indices j0 .. j0+31
  int32_t nxt = idx[(base + 32 + lane) % nidx];     // j0+32 .. j0+63
  // prologue: rows 0 .. S-1 (S <= 32)
  {
    const int32_t u = __shfl_sync(~0u, cur, lane < S ? lane : 0);
    if (lane < S) issue(u, lane);
  }
  float4 a[3] = {};
  for (int j = 0; j < per_warp; ++j) {
    const int s = j % S;
    const uint32_t b = smem_u32(&bar[w][s]);
    const uint32_t par = (j / S) & 1;
    asm volatile(
        "{\n\t.reg .pred P1;\n\tW_%=:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
        "@!P1 bra W_%=;\n\t}\n" ::"r"(b),
        "r"(par)
        : "memory");
    const float4 *r = reinterpret_cast<const float4 *>(ring + s * SLOT);
#pragma unroll
    for (int k = 0; k < 3; ++k) {
      const int c = lane + 32 * k;
      if (c < ROWB / 16) {
        const float4 v = r[c];
        a[k].x += v.x; a[k].y += v.y; a[k].z += v.z; a[k].w += v.w;
      }
    }
    __syncwarp();
    // refill slot s with row j + S
    const int jn = j + S;
    if ((jn & 31) == 0) {  // rotate the index window when row jn starts a new batch of 32
      cur = nxt;
      nxt = idx[(base + jn + 32 + lane) % nidx];
    }
    const int32_t u = __shfl_sync(~0u, cur, jn & 31);
    if (lane == 0 && jn < per_warp) {
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      issue(u, s);
    }
  }
  float sum = 0;
  for (int k = 0; k < 3; ++k) sum += a[k].x + a[k].y + a[k].z + a[k].w;
  if (sum == 12345.f) out[0] = sum;
}

// cp.async (LDGSTS) gather: each lane copies its own 16-byte chunks of a row
// into a per-warp shared-memory ring of S row slots and later reads back only
// those chunks (no cross-lane sharing, so no barrier): in-flight data lives in
// shared memory, not in registers
template <int ROWB, int S, int WARPS>
__global__ void __launch_bounds__(WARPS * 32) k_cpa(const char *X, const int32_t *idx, int64_t nidx, int per_warp,
                                                    float *out) {
  constexpr int SLOT = (ROWB + 127) / 128 * 128;
  constexpr int NCH = ROWB / 16;               // 16-byte chunks per row
  constexpr int PER = (NCH + 31) / 32;          // chunks per lane
  extern __shared__ __align__(128) char smem[];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  char *ring = smem + (size_t)w * S * SLOT;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t base = warp * per_warp;
  auto issue = [&](int32_t u, int s) {
    const char *src = X + (int64_t)u * ROWB;
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      const int c = lane + 32 * k;
      if (c < NCH)
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(ring + s * SLOT + 16 * c)),
                     "l"(src + 16 * c)
                     : "memory");
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  int32_t cur = idx[(base + lane) % nidx];
  int32_t nxt = idx[(base + 32 + lane) % nidx];
#pragma unroll
  for (int q = 0; q < S; ++q) issue(__shfl_sync(~0u, cur, q), q);
  float4 a[PER] = {};
  for (int j = 0; j < per_warp; ++j) {
    const int s = j % S;
    asm volatile("cp.async.wait_group %0;" ::"n"(S - 1) : "memory");
#pragma unroll
    for (int k = 0; k < PER; ++k) {
      const int c = lane + 32 * k;
      if (c < NCH) {
        const float4 v = *reinterpret_cast<const float4 *>(ring + s * SLOT + 16 * c);
        a[k].x += v.x; a[k].y += v.y; a[k].z += v.z; a[k].w += v.w;
      }
    }
    const int jn = j + S;
    if ((jn & 31) == 0) {
      cur = nxt;
      nxt = idx[(base + jn + 32 + lane) % nidx];
    }
    const int32_t u = __shfl_sync(~0u, cur, jn & 31);
    if (jn < per_warp) issue(u, s);
    else asm volatile("cp.async.commit_group;" ::: "memory");  // keep the group count uniform
  }
  float sum = 0;
  for (int k = 0; k < PER; ++k) sum += a[k].x + a[k].y + a[k].z + a[k].w;
  if (sum == 12345.f) out[0] = sum;
}

// TMA tile::gather4 gather: one lane issues cp.async.bulk.tensor.2d...gather4
// for 4 rows at a time (one request = 4 rows) into a per-warp ring of S
// slots, completion on an mbarrier per slot
template <int ROWB, int S>
__global__ void __launch_bounds__(256) k_g4(const __grid_constant__ CUtensorMap map, const int32_t *idx, int64_t nidx,
                                            int per_warp, float *out) {
  constexpr int SLOTB = (4 * ROWB + 127) / 128 * 128;  // TMA destinations are 128-byte aligned
  constexpr int NCH = ROWB / 16;
  constexpr int PER = (NCH + 31) / 32;
  extern __shared__ __align__(128) char smem[];
  __shared__ uint64_t bar[8][S];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  char *ring = smem + (size_t)w * S * SLOTB;
  if (lane == 0)
    for (int s = 0; s < S; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&bar[w][s])));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t base = warp * per_warp;
  int32_t cur = idx[(base + lane) % nidx];
  int32_t nxt = idx[(base + 32 + lane) % nidx];
  auto issue = [&](int q, int s) {  // rows 4q .. 4q+3 of the current batch window
    const int j = (4 * q) & 31;
    const int32_t r0 = __shfl_sync(~0u, cur, j), r1 = __shfl_sync(~0u, cur, j + 1),
                  r2 = __shfl_sync(~0u, cur, j + 2), r3 = __shfl_sync(~0u, cur, j + 3);
    if (lane == 0) {
      const uint32_t b = smem_u32(&bar[w][s]);
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(b), "r"(SLOTB) : "memory");
      asm volatile(
          "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, "
          "%3, %4, %5, %6}], [%7];" ::"r"(smem_u32(ring + s * SLOTB)),
          "l"(&map), "r"(0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(b)
          : "memory");
    }
  };
  const int nq = per_warp / 4;
  for (int q = 0; q < S; ++q) issue(q, q);
  float4 a[PER] = {};
  for (int q = 0; q < nq; ++q) {
    const int s = q % S;
    const uint32_t b = smem_u32(&bar[w][s]);
    const uint32_t par = (q / S) & 1;
    {  // bounded wait: trap instead of hanging if a request never completes
      uint32_t ok = 0;
      for (int spin = 0; !ok; ++spin) {
        asm volatile(
            "{\n\t.reg .pred P1;\n\tmbarrier.try_wait.parity.shared::cta.b64 P1, [%1], %2;\n\tselp.u32 %0, 1, 0, P1;\n\t}\n"
            : "=r"(ok)
            : "r"(b), "r"(par)
            : "memory");
        if (spin > (1 << 22)) __trap();
      }
    }
#pragma unroll
    for (int r = 0; r < 4; ++r) {
      const float4 *row = reinterpret_cast<const float4 *>(ring + s * SLOTB + r * ROWB);
#pragma unroll
      for (int k = 0; k < PER; ++k) {
        const int c = lane + 32 * k;
        if (c < NCH) {
          const float4 v = row[c];
          a[k].x += v.x; a[k].y += v.y; a[k].z += v.z; a[k].w += v.w;
        }
      }
    }
    __syncwarp();
    const int qn = q + S;
    if (((4 * qn) & 31) == 0) {
      cur = nxt;
      nxt = idx[(base + 4 * qn + 32 + lane) % nidx];
    }
    if (qn < nq) issue(qn, s);
  }
  float sum = 0;
  for (int k = 0; k < PER; ++k) sum += a[k].x + a[k].y + a[k].z + a[k].w;
  if (sum == 12345.f) out[0] = sum;
}

typedef CUresult (*EncodeTiledFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                  const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
static bool encode_rows(CUtensorMap *m, const void *X, int64_t nrows, int rowb) {
  static EncodeTiledFn fn = nullptr;
  if (!fn) {
    void *f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) != cudaSuccess) return false;
    fn = (EncodeTiledFn)f;
  }
  const cuuint64_t dims[2] = {(cuuint64_t)(rowb / 4), (cuuint64_t)nrows};
  const cuuint64_t strides[1] = {(cuuint64_t)rowb};
  const cuuint32_t box[2] = {(cuuint32_t)(rowb / 4), 1};
  const cuuint32_t es[2] = {1, 1};
  CUresult r = fn(m, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void *)X, dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                  CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) printf("encode failed %d\n", (int)r);
  return r == CUDA_SUCCESS;
}

template <typename K>
static float time_kernel(K launch) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  launch();
  cudaEventRecord(a);
  launch();
  launch();
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms;
  cudaEventElapsedTime(&ms, a, b);
  return ms / 2;
}

template <int ROWB>
static void run_rowb(const char *X, int64_t nrows_total, int32_t *idx_d, std::vector<int32_t> &h, int64_t nidx,
                     float *out) {
  const int64_t sets[3] = {nrows_total, (int64_t)100e6 / ROWB, (int64_t)24e6 / ROWB};
  const char *names[3] = {"2.5GB(HBM)", "100MB(L2) ", "24MB(L2)  "};
  const int per_warp = 4096;
  for (int si = 0; si < 3; ++si) {
    uint64_t st = 12345;
    for (int64_t i = 0; i < nidx; ++i) {
      st = st * 6364136223846793005ULL + 1442695040888963407ULL;
      h[i] = (int32_t)((st >> 33) % (uint64_t)sets[si]);
    }
    cudaMemcpy(idx_d, h.data(), nidx * 4, cudaMemcpyHostToDevice);
    // register gather, 256-thread CTAs, occupancy-limited grid (4 waves of resident CTAs)
    auto reg = [&](auto kern, int U) {
      int occ = 0;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, 256, 0);
      const int blocks = 148 * occ * 2;
      const double rows = (double)blocks * 8 * per_warp;
      const float ms = time_kernel([&] { kern<<<blocks, 256>>>(X, idx_d, nidx, per_warp, out); });
      printf("ROWB %4d %s reg  U=%d occ=%2d CTA/SM: %8.3f ms %7.0f GB/s\n", ROWB, names[si], U, occ, ms,
             rows * ROWB / (ms * 1e-3) / 1e9);
    };
    reg(k_reg<ROWB, 2>, 2);
    reg(k_reg<ROWB, 4>, 4);
    reg(k_reg<ROWB, 8>, 8);
    auto bulk = [&](auto kern, int S, int warps) {
      constexpr int SLOT = (ROWB + 127) / 128 * 128;
      const size_t sm = (size_t)warps * S * SLOT;
      cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
      int occ = 0;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, warps * 32, sm);
      if (occ < 1) return;
      const int blocks = 148 * occ * 2;
      const double rows = (double)blocks * warps * per_warp;
      const float ms = time_kernel([&] { kern<<<blocks, warps * 32, sm>>>(X, idx_d, nidx, per_warp, out); });
      printf("ROWB %4d %s bulk S=%2d warps=%d occ=%2d CTA/SM (%3zu KB smem/SM): %8.3f ms %7.0f GB/s\n", ROWB, names[si],
             S, warps, occ, sm * occ / 1024, ms, rows * ROWB / (ms * 1e-3) / 1e9);
    };
    auto cpa = [&](auto kern, int S, int warps) {
      constexpr int SLOT = (ROWB + 127) / 128 * 128;
      const size_t sm = (size_t)warps * S * SLOT;
      cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
      int occ = 0;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, warps * 32, sm);
      if (occ < 1) return;
      const int blocks = 148 * occ * 2;
      const double rows = (double)blocks * warps * per_warp;
      const float ms = time_kernel([&] { kern<<<blocks, warps * 32, sm>>>(X, idx_d, nidx, per_warp, out); });
      printf("ROWB %4d %s cpa  S=%2d warps=%d occ=%2d CTA/SM (%3zu KB smem/SM, %2d warps/SM): %8.3f ms %7.0f GB/s\n",
             ROWB, names[si], S, warps, occ, sm * occ / 1024, occ * warps, ms, rows * ROWB / (ms * 1e-3) / 1e9);
    };
    cpa(k_cpa<ROWB, 4, 8>, 4, 8);
    cpa(k_cpa<ROWB, 6, 8>, 6, 8);
    cpa(k_cpa<ROWB, 8, 8>, 8, 8);
    cpa(k_cpa<ROWB, 12, 8>, 12, 8);
    cpa(k_cpa<ROWB, 4, 16>, 4, 16);
    cpa(k_cpa<ROWB, 6, 16>, 6, 16);
    cpa(k_cpa<ROWB, 3, 16>, 3, 16);
    if constexpr (ROWB <= 1024 && ROWB % 16 == 0) {
      CUtensorMap map;
      if (encode_rows(&map, X, sets[0], ROWB)) {
        auto g4 = [&](auto kern, int S) {
          const size_t sm = (size_t)8 * S * ((4 * ROWB + 127) / 128 * 128);
          cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
          int occ = 0;
          cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, 256, sm);
          if (occ < 1) return;
          const int blocks = 148 * occ * 2;
          const double rows = (double)blocks * 8 * per_warp;
          const float ms = time_kernel([&] { kern<<<blocks, 256, sm>>>(map, idx_d, nidx, per_warp, out); });
          printf("ROWB %4d %s g4   S=%2d (4 rows/slot) occ=%2d CTA/SM (%3zu KB smem/SM): %8.3f ms %7.0f GB/s  %s\n", ROWB,
                 names[si], S, occ, sm * occ / 1024, ms, rows * ROWB / (ms * 1e-3) / 1e9,
                 cudaGetErrorString(cudaGetLastError()));
        };
        g4(k_g4<ROWB, 1>, 1);
        g4(k_g4<ROWB, 2>, 2);
        g4(k_g4<ROWB, 3>, 3);
      }
    }
  }
}

int main() {
  const size_t bytes = (size_t)2449029 * 1056;  // C5 rows at the widest row size
  char *X;
  cudaMalloc(&X, bytes);
  cudaMemset(X, 0, bytes);
  const int64_t nidx = 1 << 24;
  int32_t *idx;
  float *out;
  cudaMalloc(&idx, nidx * 4);
  cudaMalloc(&out, 4);
  std::vector<int32_t> h(nidx);
  run_rowb<1024>(X, bytes / 1024, idx, h, nidx, out);
  run_rowb<400>(X, bytes / 400, idx, h, nidx, out);
  run_rowb<1056>(X, bytes / 1056, idx, h, nidx, out);
  printf("err=%s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}
