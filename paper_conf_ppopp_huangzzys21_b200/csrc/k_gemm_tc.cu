// k_gemm_tc.cu — a5: H = X W on the 5th-generation tensor cores (tcgen05,
// kind::tf32, accumulator in TMEM) with a 3xTF32 split so the result has fp32
// accuracy (plain TF32 fails the 1e-4 bar):
//     X = Xhi + Xlo, W = Whi + Wlo  (hi = fp32 with the low 13 mantissa bits
//     cleared — exactly representable in TF32; lo = x - hi, exact in fp32)
//     H = Xhi Whi + Xhi Wlo + Xlo Whi      (Xlo Wlo ~ 2^-22 relative, dropped)
// Epilogue fused: row scale (GCN nsrc[u]), column bias, ReLU.
//
// CTA = 128 rows x N (N <= 512; one MMA per 256 columns).  Warps 0-3 load
// X/W tiles from global memory, split them into hi/lo and write them to
// shared memory in the UMMA K-major SWIZZLE_128B layout (32 fp32 of K per
// 128-byte row), then signal an mbarrier; warp 4 (one elected lane) issues
// tcgen05.mma and releases stages with tcgen05.commit; warps 0-3 finally
// read the accumulator with tcgen05.ld (32x32b: one TMEM lane = one row per
// thread) and store it.
#include <cuda_runtime.h>
#include <stdint.h>

#include "gnn_internal.h"

namespace gnn {
namespace tc {

constexpr int BM = 128;
constexpr int BK = 32;           // fp32 elements per 128-byte swizzle row
constexpr int NUM_LOAD_WARPS = 4;
constexpr int THREADS = 32 * (NUM_LOAD_WARPS + 1);
constexpr int TILE_A_BYTES = BM * BK * 4;  // 16 KB

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}

__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_arrive(uint64_t *bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
  const uint32_t addr = smem_u32(bar);
  asm volatile(
      "{\n\t"
      ".reg .pred P1;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@!P1 bra WAIT_%=;\n\t"
      "}\n" ::"r"(addr),
      "r"(parity)
      : "memory");
}

// UMMA shared-memory descriptor: K-major, SWIZZLE_128B, 8-row atoms of 1024 B
__device__ __forceinline__ uint64_t sw128_desc(uint32_t saddr) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr & 0x3FFFF) >> 4);  // start address (>>4), bits 0-13
  d |= (uint64_t)1 << 16;                   // leading byte offset (unused for swizzled K-major)
  d |= (uint64_t)(1024 >> 4) << 32;         // stride byte offset: 8 rows x 128 B
  d |= (uint64_t)1 << 46;                   // descriptor version (sm_100)
  d |= (uint64_t)2 << 61;                   // layout: SWIZZLE_128B
  return d;
}

// instruction descriptor: D f32, A/B tf32, K-major both, M = 128, N
__host__ __device__ constexpr uint32_t idesc_tf32(int n) {
  return (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(BM >> 4) << 24);
}

__device__ __forceinline__ void mma_tf32(uint32_t tmem_d, uint64_t da, uint64_t db, uint32_t idesc,
                                         uint32_t accumulate) {
  asm volatile(
      "{\n\t"
      ".reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t"
      "}\n" ::"r"(tmem_d),
      "l"(da), "l"(db), "r"(idesc), "r"(accumulate));
}

__device__ __forceinline__ void mma_commit(uint64_t *bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                   smem_u32(bar))
               : "memory");
}

// split x into (hi, lo): hi = x with 13 low mantissa bits cleared (TF32-exact), lo = x - hi (exact)
__device__ __forceinline__ void split4(const float4 &x, float4 &hi, float4 &lo) {
  hi.x = __uint_as_float(__float_as_uint(x.x) & 0xFFFFE000u);
  hi.y = __uint_as_float(__float_as_uint(x.y) & 0xFFFFE000u);
  hi.z = __uint_as_float(__float_as_uint(x.z) & 0xFFFFE000u);
  hi.w = __uint_as_float(__float_as_uint(x.w) & 0xFFFFE000u);
  lo.x = x.x - hi.x;
  lo.y = x.y - hi.y;
  lo.z = x.z - hi.z;
  lo.w = x.w - hi.w;
}

// byte offset of 16-byte chunk c (0..7) of row r inside a SW128 K-major tile
__device__ __forceinline__ uint32_t sw128_off(int r, int c) {
  return (uint32_t)((r >> 3) * 1024 + (r & 7) * 128 + ((c ^ (r & 7)) << 4));
}

struct TcParams {
  const float *X;
  int64_t ldx;
  const float *W;
  int64_t ldw;
  float *H;
  int64_t ldh;
  int64_t m;
  int32_t k, n, np;  // np = n rounded up to 16
  const float *row_scale;
  const float *col_bias;
  int32_t relu;
  int32_t stages;
  int32_t tmem_cols;
};

template <bool VEC_X, bool VEC_H>
__global__ void __launch_bounds__(THREADS, 1) k_gemm_tc(const TcParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // carve: [stage][A_hi | A_lo | B_hi | B_lo], 1024-aligned
  uint8_t *smem = (uint8_t *)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  const int NP = p.np;
  const int B_BYTES = NP * 128;
  const int STAGE_BYTES = 2 * TILE_A_BYTES + 2 * B_BYTES;
  __shared__ uint64_t full_bar[4], empty_bar[4], accum_bar;
  __shared__ uint32_t tmem_base_sh;

  const int tid = threadIdx.x;
  const int warp = tid >> 5;
  const int lane = tid & 31;
  const int64_t m0 = (int64_t)blockIdx.x * BM;
  const int num_kb = (p.k + BK - 1) / BK;
  const int S = p.stages;

  if (tid == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full_bar[s], NUM_LOAD_WARPS * 32);
      mbar_init(&empty_bar[s], 1);
    }
    mbar_init(&accum_bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(
                     smem_u32(&tmem_base_sh)),
                 "r"(p.tmem_cols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = tmem_base_sh;

  if (warp < NUM_LOAD_WARPS) {
    // ---------------- producers: global -> split -> swizzled smem ----------------
    for (int kb = 0; kb < num_kb; ++kb) {
      const int s = kb % S, use = kb / S;
      if (use > 0) mbar_wait(&empty_bar[s], (use - 1) & 1);
      uint8_t *st = smem + (size_t)s * STAGE_BYTES;
      uint8_t *a_hi = st, *a_lo = st + TILE_A_BYTES, *b_hi = st + 2 * TILE_A_BYTES, *b_lo = b_hi + B_BYTES;
      const int k0 = kb * BK;
      // A: 128 rows x 8 chunks of 4 fp32
#pragma unroll 2
      for (int q = tid; q < BM * 8; q += NUM_LOAD_WARPS * 32) {
        const int r = q >> 3, c = q & 7;
        const int64_t gm = m0 + r;
        const int gk = k0 + 4 * c;
        float4 x = make_float4(0.f, 0.f, 0.f, 0.f);
        if (gm < p.m) {
          const float *src = p.X + gm * p.ldx + gk;
          if (VEC_X && gk + 3 < p.k) {
            x = __ldg(reinterpret_cast<const float4 *>(src));
          } else {
            if (gk + 0 < p.k) x.x = __ldg(src + 0);
            if (gk + 1 < p.k) x.y = __ldg(src + 1);
            if (gk + 2 < p.k) x.z = __ldg(src + 2);
            if (gk + 3 < p.k) x.w = __ldg(src + 3);
          }
        }
        float4 hi, lo;
        split4(x, hi, lo);
        const uint32_t off = sw128_off(r, c);
        *reinterpret_cast<float4 *>(a_hi + off) = hi;
        *reinterpret_cast<float4 *>(a_lo + off) = lo;
      }
      // B (K-major W^T tile): NP rows (n) x 8 chunks of 4 k; W is [k, n] row-major
      for (int q = tid; q < NP * 8; q += NUM_LOAD_WARPS * 32) {
        const int c = q / NP, nn = q % NP;  // consecutive threads -> consecutive n (coalesced)
        const int gk = k0 + 4 * c;
        float4 w = make_float4(0.f, 0.f, 0.f, 0.f);
        if (nn < p.n) {
          const float *src = p.W + (int64_t)gk * p.ldw + nn;
          if (gk + 0 < p.k) w.x = __ldg(src);
          if (gk + 1 < p.k) w.y = __ldg(src + p.ldw);
          if (gk + 2 < p.k) w.z = __ldg(src + 2 * p.ldw);
          if (gk + 3 < p.k) w.w = __ldg(src + 3 * p.ldw);
        }
        float4 hi, lo;
        split4(w, hi, lo);
        const uint32_t off = sw128_off(nn, c);
        *reinterpret_cast<float4 *>(b_hi + off) = hi;
        *reinterpret_cast<float4 *>(b_lo + off) = lo;
      }
      // make generic-proxy smem writes visible to the tensor core (async proxy)
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      mbar_arrive(&full_bar[s]);
    }
    // ---------------- epilogue: TMEM -> registers -> global ----------------
    mbar_wait(&accum_bar, 0);
    asm volatile("tcgen05.fence::after_thread_sync;");
    const int r = warp * 32 + lane;
    const int64_t gm = m0 + r;
    const float sc = (p.row_scale && gm < p.m) ? __ldg(p.row_scale + gm) : 1.0f;
    for (int c0 = 0; c0 < NP; c0 += 32) {
      uint32_t v[32];
      const uint32_t taddr = tmem + ((uint32_t)(warp * 32) << 16) + (uint32_t)c0;
      asm volatile(
          "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
          "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
          : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]),
            "=r"(v[7]), "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]),
            "=r"(v[14]), "=r"(v[15]), "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]),
            "=r"(v[21]), "=r"(v[22]), "=r"(v[23]), "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]),
            "=r"(v[28]), "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
          : "r"(taddr));
      asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
      if (gm >= p.m) continue;
      float y[32];
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        const int col = c0 + i;
        float t = __uint_as_float(v[i]);
        if (p.row_scale) t = t * sc;
        if (p.col_bias && col < p.n) t = t + __ldg(p.col_bias + col);
        if (p.relu) t = t > 0.0f ? t : 0.0f;
        y[i] = t;
      }
      float *dst = p.H + gm * p.ldh + c0;
      if (VEC_H && c0 + 32 <= p.n) {
#pragma unroll
        for (int i = 0; i < 32; i += 4)
          *reinterpret_cast<float4 *>(dst + i) = make_float4(y[i], y[i + 1], y[i + 2], y[i + 3]);
      } else {
#pragma unroll
        for (int i = 0; i < 32; ++i)
          if (c0 + i < p.n) dst[i] = y[i];
      }
    }
  } else {
    // ---------------- MMA issuer: warp 4, one elected lane ----------------
    for (int kb = 0; kb < num_kb; ++kb) {
      const int s = kb % S, use = kb / S;
      mbar_wait(&full_bar[s], use & 1);
      asm volatile("tcgen05.fence::after_thread_sync;");
      if (lane == 0) {
        const uint32_t st = smem_u32(smem + (size_t)s * STAGE_BYTES);
        const uint32_t a_hi = st, a_lo = st + TILE_A_BYTES, b_hi = st + 2 * TILE_A_BYTES, b_lo = b_hi + B_BYTES;
#pragma unroll
        for (int j = 0; j < BK / 8; ++j) {  // 8 tf32 (32 B) per MMA K step
          const uint32_t ko = j * 32;
          for (int n0 = 0; n0 < NP; n0 += 256) {
            const int nn = NP - n0 < 256 ? NP - n0 : 256;
            const uint32_t id = idesc_tf32(nn);
            const uint32_t bo = (uint32_t)n0 * 128;  // row n0 of the B tile
            const uint32_t d = tmem + (uint32_t)n0;
            const uint32_t acc0 = (kb > 0 || j > 0) ? 1u : 0u;
            mma_tf32(d, sw128_desc(a_lo + ko), sw128_desc(b_hi + bo + ko), id, acc0);
            mma_tf32(d, sw128_desc(a_hi + ko), sw128_desc(b_lo + bo + ko), id, 1u);
            mma_tf32(d, sw128_desc(a_hi + ko), sw128_desc(b_hi + bo + ko), id, 1u);
          }
        }
        mma_commit(&empty_bar[s]);
        if (kb == num_kb - 1) mma_commit(&accum_bar);
      }
      __syncwarp();
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) {
    asm volatile("tcgen05.fence::after_thread_sync;");
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(p.tmem_cols));
  }
}

}  // namespace tc

cudaError_t launch_gemm_tc(const float *X, int64_t ldx, const float *W, int64_t ldw, float *H, int64_t ldh,
                           int64_t m, int32_t k, int32_t n, const float *row_scale, const float *col_bias,
                           int32_t relu, cudaStream_t s) {
  using namespace tc;
  if (n < 1 || n > 512 || k < 1 || m < 1) return cudaErrorNotSupported;
  const int np = (n + 15) / 16 * 16;
  const int stage_bytes = 2 * TILE_A_BYTES + 2 * np * 128;
  int stages = 4;
  while (stages > 2 && stages * stage_bytes > 160 * 1024) --stages;
  const size_t smem = (size_t)stages * stage_bytes + 1024;
  if (smem > 227 * 1024) return cudaErrorNotSupported;
  int cols = 32;
  while (cols < np) cols *= 2;
  TcParams p{X, ldx, W, ldw, H, ldh, m, k, n, np, row_scale, col_bias, relu, stages, cols};
  const bool vx = (ldx % 4 == 0) && ((uintptr_t)X % 16 == 0);
  const bool vh = (ldh % 4 == 0) && ((uintptr_t)H % 16 == 0);
  auto fn = vx ? (vh ? k_gemm_tc<true, true> : k_gemm_tc<true, false>)
               : (vh ? k_gemm_tc<false, true> : k_gemm_tc<false, false>);
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  const int64_t grid = (m + BM - 1) / BM;
  if (grid > 0x7fffffff) return cudaErrorNotSupported;
  fn<<<(unsigned)grid, THREADS, smem, s>>>(p);
  count_launch();
  return cudaGetLastError();
}

}  // namespace gnn
