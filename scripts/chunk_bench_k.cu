// chunk_bench_k.cu — dev experiment (not the product): how fast can the C5
// gather stream be consumed when H is swept in feature chunks of CW floats
// (smaller working set per sweep -> more L2 reuse), and which load path keeps
// enough bytes in flight: registers (LDG), LDGSTS (cp.async) or bulk copies
// (cp.async.bulk, the TMA engine) into a per-warp shared-memory ring.
//
// Every kernel: one warp per destination row (rows in task order, claimed
// from an atomic counter), sequential fp32 sum over the row's sources in CSR
// order per feature (the R9 chain), chunk loop outermost.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -shared -Xcompiler -fPIC chunk_bench_k.cu -o libchunkbench.so
#include <cuda_runtime.h>
#include <stdint.h>

namespace {

template <int NF>
struct Vec {
  float v[NF];
};

template <int NF>
__device__ __forceinline__ void ldg(const float *p, Vec<NF> &r) {
  if constexpr (NF == 8) {
    asm volatile("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=f"(r.v[0]), "=f"(r.v[1]), "=f"(r.v[2]), "=f"(r.v[3]), "=f"(r.v[4]), "=f"(r.v[5]),
                   "=f"(r.v[6]), "=f"(r.v[7])
                 : "l"(p));
  } else if constexpr (NF == 4) {
    float4 x = __ldg(reinterpret_cast<const float4 *>(p));
    r.v[0] = x.x; r.v[1] = x.y; r.v[2] = x.z; r.v[3] = x.w;
  } else if constexpr (NF == 2) {
    float2 x = __ldg(reinterpret_cast<const float2 *>(p));
    r.v[0] = x.x; r.v[1] = x.y;
  } else {
    r.v[0] = __ldg(p);
  }
}

template <int NF>
__device__ __forceinline__ void lds(const float *p, Vec<NF> &r) {
  if constexpr (NF == 4) {
    float4 x = *reinterpret_cast<const float4 *>(p);
    r.v[0] = x.x; r.v[1] = x.y; r.v[2] = x.z; r.v[3] = x.w;
  } else if constexpr (NF == 2) {
    float2 x = *reinterpret_cast<const float2 *>(p);
    r.v[0] = x.x; r.v[1] = x.y;
  } else if constexpr (NF == 8) {
    float4 x = *reinterpret_cast<const float4 *>(p);
    float4 y = *reinterpret_cast<const float4 *>(p + 4);
    r.v[0] = x.x; r.v[1] = x.y; r.v[2] = x.z; r.v[3] = x.w;
    r.v[4] = y.x; r.v[5] = y.y; r.v[6] = y.z; r.v[7] = y.w;
  } else {
    r.v[0] = *p;
  }
}

struct Args {
  const float *X;
  int64_t ldx;
  const int32_t *idx;   // task-ordered sources
  const int64_t *tptr;  // [n+1] offsets in idx (task order)
  const int32_t *trow;  // [n] row id of task i
  int64_t n;
  int F;
  int *ctr;             // [nchunks] zeroed
  float *Y;
};

// ---------------- K_reg: registers, U rows in flight ----------------
template <int CW, int U>
__global__ void __launch_bounds__(256) k_reg(Args a) {
  constexpr int NF = CW / 32;
  const int lane = threadIdx.x & 31;
  int ci = 0;
  for (int c0 = 0; c0 < a.F; c0 += CW, ++ci) {
    int t = 0;
    if (lane == 0) t = atomicAdd(a.ctr + ci, 1);
    t = __shfl_sync(~0u, t, 0);
    while (t < a.n) {
      int tn = 0;
      if (lane == 0) tn = atomicAdd(a.ctr + ci, 1);
      const int64_t b = a.tptr[t], e = a.tptr[t + 1];
      const int row = a.trow[t];
      float acc[NF];
#pragma unroll
      for (int i = 0; i < NF; ++i) acc[i] = 0.f;
      const float *xl = a.X + c0 + lane * NF;
      int32_t nxt = (b + lane < e) ? a.idx[b + lane] : 0;
      for (int64_t k = b; k < e; k += 32) {
        const int cnt = (int)(e - k < 32 ? e - k : 32);
        const int32_t my = nxt;
        if (k + 32 < e) nxt = (k + 32 + lane < e) ? a.idx[k + 32 + lane] : 0;
        Vec<NF> v[U];
#pragma unroll
        for (int q = 0; q < U; ++q)
          if (q < cnt) ldg<NF>(xl + (int64_t)__shfl_sync(~0u, my, q) * a.ldx, v[q]);
        for (int j = 0; j < cnt; j += U) {
#pragma unroll
          for (int q = 0; q < U; ++q) {
            if (j + q < cnt) {
#pragma unroll
              for (int i = 0; i < NF; ++i) acc[i] += v[q].v[i];
              const int nx = j + q + U;
              const int32_t u = __shfl_sync(~0u, my, nx & 31);
              if (nx < cnt) ldg<NF>(xl + (int64_t)u * a.ldx, v[q]);
            }
          }
        }
      }
      float *y = a.Y + (int64_t)row * a.F + c0 + lane * NF;
#pragma unroll
      for (int i = 0; i < NF; ++i) y[i] = acc[i];
      t = __shfl_sync(~0u, tn, 0);
    }
  }
}

// ---------------- K_async: LDGSTS into a per-warp ring of R slots ----------------
// CW floats per row chunk = CW*4 bytes = CW/4 lanes x 16 B; P = 128/CW rows per
// warp instruction (CW <= 128).  Lane l consumes floats [l*NF, l*NF+NF).
__device__ __forceinline__ void cp16(uint32_t sdst, const void *g) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(sdst), "l"(g));
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;"); }
template <int N>
__device__ __forceinline__ void cp_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N)); }

template <int CW, int R, int WARPS>
__global__ void __launch_bounds__(WARPS * 32) k_async(Args a) {
  constexpr int NF = CW / 32;
  constexpr int LPR = CW / 4;          // lanes per row (16 B each)
  constexpr int P = 32 / LPR;          // rows per copy instruction
  extern __shared__ __align__(128) float smem[];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  float *ring = smem + (size_t)wid * R * P * CW;  // R stages x P rows x CW
  const uint32_t ring_s = (uint32_t)__cvta_generic_to_shared(ring);
  int ci = 0;
  for (int c0 = 0; c0 < a.F; c0 += CW, ++ci) {
    int t = 0;
    if (lane == 0) t = atomicAdd(a.ctr + ci, 1);
    t = __shfl_sync(~0u, t, 0);
    while (t < a.n) {
      int tn = 0;
      if (lane == 0) tn = atomicAdd(a.ctr + ci, 1);
      const int64_t b = a.tptr[t], e = a.tptr[t + 1];
      const int row = a.trow[t];
      const int len = (int)(e - b);
      float acc[NF];
#pragma unroll
      for (int i = 0; i < NF; ++i) acc[i] = 0.f;
      const int nst = (len + P - 1) / P;  // stages (P rows each)
      const int sub = lane / LPR, part = lane % LPR;
      // issue stage s: rows b + s*P + sub
      auto issue = [&](int s) {
        const int k = s * P + sub;
        if (k < len) {
          const int32_t u = __ldg(a.idx + b + k);
          cp16(ring_s + (uint32_t)((((s % R) * P + sub) * CW + part * 4) * 4),
               a.X + (int64_t)u * a.ldx + c0 + part * 4);
        }
        cp_commit();
      };
#pragma unroll 1
      for (int s = 0; s < R - 1; ++s) issue(s);
#pragma unroll 1
      for (int s = 0; s < nst; ++s) {
        issue(s + R - 1);
        cp_wait<R - 1>();
        __syncwarp();
        const float *st = ring + (size_t)(s % R) * P * CW;
        const int rows = min(P, len - s * P);
        for (int r = 0; r < rows; ++r) {
          Vec<NF> v;
          lds<NF>(st + r * CW + lane * NF, v);
#pragma unroll
          for (int i = 0; i < NF; ++i) acc[i] += v.v[i];
        }
        __syncwarp();
      }
      cp_wait<0>();
      float *y = a.Y + (int64_t)row * a.F + c0 + lane * NF;
#pragma unroll
      for (int i = 0; i < NF; ++i) y[i] = acc[i];
      t = __shfl_sync(~0u, tn, 0);
    }
  }
}

// ---------------- K_bulk: cp.async.bulk (TMA engine) per row chunk ----------------
__device__ __forceinline__ void mbar_init(uint32_t bar, int cnt) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(cnt));
}
__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void *src, uint32_t bytes, uint32_t bar) {
  asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(dst), "l"(src), "r"(bytes), "r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t phase) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra W;\n"
      "}\n" ::"r"(bar), "r"(phase) : "memory");
}

template <int CW, int R, int WARPS>
__global__ void __launch_bounds__(WARPS * 32) k_bulk(Args a) {
  constexpr int NF = CW / 32;
  extern __shared__ __align__(128) float smem[];
  __shared__ __align__(8) uint64_t bars[WARPS][R];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  float *ring = smem + (size_t)wid * R * CW;
  const uint32_t ring_s = (uint32_t)__cvta_generic_to_shared(ring);
  const uint32_t bar0 = (uint32_t)__cvta_generic_to_shared(&bars[wid][0]);
  if (lane < R) mbar_init(bar0 + 8 * lane, 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  uint32_t phase_bits = 0;  // parity per slot (R <= 32)
  uint32_t use = 0;         // running slot counter
  int ci = 0;
  for (int c0 = 0; c0 < a.F; c0 += CW, ++ci) {
    int t = 0;
    if (lane == 0) t = atomicAdd(a.ctr + ci, 1);
    t = __shfl_sync(~0u, t, 0);
    while (t < a.n) {
      int tn = 0;
      if (lane == 0) tn = atomicAdd(a.ctr + ci, 1);
      const int64_t b = a.tptr[t], e = a.tptr[t + 1];
      const int row = a.trow[t];
      const int len = (int)(e - b);
      float acc[NF];
#pragma unroll
      for (int i = 0; i < NF; ++i) acc[i] = 0.f;
      // lanes 0..R-1 issue the first R rows (one each)
      const uint32_t base = use;
      if (lane < R && lane < len) {
        const uint32_t slot = (base + lane) % R;
        const int32_t u = __ldg(a.idx + b + lane);
        mbar_expect_tx(bar0 + 8 * slot, CW * 4);
        bulk_g2s(ring_s + slot * CW * 4, a.X + (int64_t)u * a.ldx + c0, CW * 4, bar0 + 8 * slot);
      }
      int32_t nidx = (R + lane < len) ? __ldg(a.idx + b + R + lane) : 0;  // next 32 indices after the first R
      int nbase = R;
      for (int k = 0; k < len; ++k) {
        const uint32_t slot = (base + k) % R;
        mbar_wait(bar0 + 8 * slot, (phase_bits >> slot) & 1);
        phase_bits ^= 1u << slot;
        Vec<NF> v;
        lds<NF>(ring + slot * CW + lane * NF, v);
#pragma unroll
        for (int i = 0; i < NF; ++i) acc[i] += v.v[i];
        __syncwarp();
        const int kn = k + R;
        if (kn - nbase >= 32) {
          nbase += 32;
          nidx = (nbase + lane < len) ? __ldg(a.idx + b + nbase + lane) : 0;
        }
        const int32_t u = __shfl_sync(~0u, nidx, (kn - nbase) & 31);
        if (lane == 0 && kn < len) {
          mbar_expect_tx(bar0 + 8 * slot, CW * 4);
          bulk_g2s(ring_s + slot * CW * 4, a.X + (int64_t)u * a.ldx + c0, CW * 4, bar0 + 8 * slot);
        }
      }
      use = base + len;
      float *y = a.Y + (int64_t)row * a.F + c0 + lane * NF;
#pragma unroll
      for (int i = 0; i < NF; ++i) y[i] = acc[i];
      t = __shfl_sync(~0u, tn, 0);
    }
  }
}

template <typename K>
int launch(K k, int blocks, int threads, size_t smem, const Args &a) {
  if (smem > 48 * 1024) cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  k<<<blocks, threads, smem>>>(a);
  return (int)cudaGetLastError();
}

}  // namespace

// kind 0 = reg (p1 = U), 1 = async (p1 = R stages), 2 = bulk (p1 = R slots); blocks per SM p2
extern "C" int cb_run(int kind, int CW, int p1, int p2, const float *X, int64_t ldx, const int32_t *idx,
                      const int64_t *tptr, const int32_t *trow, int64_t n, int F, int *ctr, float *Y) {
  Args a{X, ldx, idx, tptr, trow, n, F, ctr, Y};
  cudaMemsetAsync(ctr, 0, 64 * sizeof(int));
  const int blocks = 148 * p2;
  if (kind == 0) {
#define REG(cw, u) \
  if (CW == cw && p1 == u) return launch(k_reg<cw, u>, blocks, 256, 0, a);
    REG(64, 4) REG(64, 8) REG(64, 16) REG(128, 4) REG(128, 8) REG(256, 4) REG(256, 2)
  } else if (kind == 1) {
#define ASY(cw, r) \
  if (CW == cw && p1 == r) return launch(k_async<cw, r, 8>, blocks, 256, (size_t)8 * r * (128 / cw) * cw * 4, a);
    ASY(64, 4) ASY(64, 8) ASY(64, 12) ASY(128, 4) ASY(128, 8) ASY(128, 12) ASY(128, 16)
  } else {
#define BLK(cw, r) \
  if (CW == cw && p1 == r) return launch(k_bulk<cw, r, 8>, blocks, 256, (size_t)8 * r * cw * 4, a);
    BLK(64, 8) BLK(64, 16) BLK(64, 24) BLK(128, 8) BLK(128, 16) BLK(256, 8) BLK(256, 6)
  }
  return -1;
}
