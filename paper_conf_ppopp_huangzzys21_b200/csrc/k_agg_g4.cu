// k_agg_g4.cu — the streaming TMA-gather aggregation kernel (a6 / a7 for
// rows of up to 256 features per sweep).
//
// One warp streams the source rows of the work units it claims (runs of
// consecutive neighbour groups in task order) through a ring of S
// shared-memory slots.  A slot holds four consecutive edges of the stream: one
// elected lane fetches their four source rows with ONE
// cp.async.bulk.tensor.2d...tile::gather4 (UTMALDG.2D.GATHER4) -- four rows per
// request, completion on the slot's mbarrier -- so the bytes in flight live in
// shared memory (not registers) and the instruction cost per edge is a
// fraction of a load per lane.  Measured on this B200 (scripts/gather_roofline.cu):
// random 1 KB rows from a 100 MB working set 18.0 TB/s with gather4 vs
// 10.6 TB/s with 256-bit register loads; HBM-bound sets 7.3 TB/s either way.
// The stream does not drain at unit or group boundaries: the next unit's rows
// are in flight while the current unit's last rows are consumed.
//
// Arithmetic: the consumer lanes use the (4, 32, 2) lane mapping of the
// register kernel and the same fp32 chain per neighbour group in CSR order
// (R9), so every result is bit-identical to the other mappings; the finished
// group goes through the same epilogue / partial / fixed-order merge
// (finish_unit).  Per-row extras (GAT t_v[h], the destination normaliser of a
// pre-scaled GCN aggregation) arrive by cp.async.bulk on the same mbarrier as
// the unit's first rows; GAT's per-edge scores s_u[h] by a second gather4 of
// the H score columns.
#include <cuda.h>
#include <stdlib.h>
#include <string.h>

#include "k_agg.cuh"

namespace gnn {
namespace g4 {
constexpr int S = 3;        // quads (4 edges) in flight per warp
constexpr int WARPS = 8;    // warps per CTA
constexpr int RUN = 2;      // units claimed per atomic (a narrow window of the task order in flight)
constexpr int QN = 16;      // unit queue entries per warp (power of 2, > the 4 S + 1 units the window can hold)
constexpr int BWMAX = 256;  // features per sweep (TMA box width limit)

__device__ __forceinline__ uint32_t sa(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *bar) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(bar)));
}
__device__ __forceinline__ void mbar_expect(uint64_t *bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(bar)), "r"(bytes) : "memory");
}
// wait for a phase; a request that has not completed after 20 s of wall
// time traps (an error the caller sees) instead of hanging the GPU
__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
  unsigned long long t0 = 0;
  for (uint32_t spin = 0;; ++spin) {
    uint32_t ok;
    asm volatile(
        "{\n\t.reg .pred P1;\n\tmbarrier.try_wait.parity.shared::cta.b64 P1, [%1], %2;\n\tselp.u32 %0, 1, 0, P1;\n\t}\n"
        : "=r"(ok)
        : "r"(sa(bar)), "r"(parity)
        : "memory");
    if (ok) return;
    if ((spin & 1023) == 1023) {
      const unsigned long long t = gtimer();
      if (t0 == 0) t0 = t;
      else if (t - t0 > 20000000000ull) __trap();
    }
  }
}
__device__ __forceinline__ void gather4(void *dst, const CUtensorMap *map, int32_t col, int32_t r0, int32_t r1,
                                        int32_t r2, int32_t r3, uint64_t *bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, "
      "%4, %5, %6}], [%7];" ::"r"(sa(dst)),
      "l"(map), "r"(col), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(sa(bar))
      : "memory");
}
__device__ __forceinline__ void bulk_copy(void *dst, const void *src, uint32_t bytes, uint64_t *bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(sa(dst)),
               "l"(src), "r"(bytes), "r"(sa(bar))
               : "memory");
}

// VEC consecutive floats from shared memory (VEC 8: two 16-byte loads)
template <int VEC>
__device__ __forceinline__ void lds_vec(const float *p, float (&v)[VEC]) {
#pragma unroll
  for (int i = 0; i < VEC; i += 4) {
    const float4 x = *reinterpret_cast<const float4 *>(p + i);
    v[i] = x.x; v[i + 1] = x.y; v[i + 2] = x.z; v[i + 3] = x.w;
  }
}

// shared-memory layout in floats (runtime: box width bw, score width hs = H for GAT); every TMA
// destination slot starts on a 128-byte boundary
struct Layout {
  // row floats per edge (GAT merged: the F features + the H scores of the row,
  // one gather4 of 8-byte elements), score floats per edge in the separate
  // score slots (0: none / merged), extras floats per queue entry, log2 of the
  // row map's element size in floats (0: fp32 elements, 1: 8-byte elements)
  int bw, hs, xe, esh;
  __host__ __device__ static int r32(int x) { return (x + 31) / 32 * 32; }
  __host__ __device__ int rslot() const { return r32(4 * bw); }  // floats per quad of rows
  __host__ __device__ int sslot() const { return r32(4 * hs); }  // floats per quad of scores
  __host__ __device__ int rows_per_warp() const { return S * rslot(); }
  __host__ __device__ int scores_per_warp() const { return S * sslot(); }
  __host__ __device__ int qe() const { return 8 + xe; }  // 8 ints + extras (16-byte multiple)
  __host__ __device__ int queue_per_warp() const { return QN * qe(); }
  __host__ __device__ size_t bytes() const {  // + 128 for aligning the dynamic base
    return sizeof(float) * (size_t)WARPS * (rows_per_warp() + scores_per_warp() + queue_per_warp()) + 128;
  }
};
}  // namespace g4

template <int MODE, int VEC, int NV>
__global__ void __launch_bounds__(g4::WARPS * 32, 2)
    k_stream_g4(const KParams p, const __grid_constant__ CUtensorMap rmap, const __grid_constant__ CUtensorMap smap,
                const g4::Layout L) {
  using namespace g4;
  constexpr bool ATT = MODE == M_GAT;
  // lane mapping (VEC, 32, NV): (4, 32, 2) / (8, 32, 1) for 256 features per sweep, (4, 32, 1) for <= 128
  extern __shared__ __align__(128) float smem_raw[];
  __shared__ uint64_t bars[WARPS][S];
  // 128-byte aligned base as an offset from the shared array, so every slot
  // pointer stays in the shared window (LDS, 32-bit addresses) instead of
  // decaying to a generic pointer (LD.E with 64-bit address arithmetic)
  float *smem = smem_raw + (((128u - (sa(smem_raw) & 127u)) & 127u) >> 2);
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  const DevGraph &g = p.g;
  if ((int32_t)blockIdx.x >= p.n_persist) {  // zero-fill rows without in-edges (R3-i)
    if (p.accum) return;
    const int64_t r0 = (int64_t)(blockIdx.x - p.n_persist) * 32;
    for (int64_t r = r0; r < r0 + 32 && r < g.n_empty; ++r) {
      float *y = p.Y + (int64_t)g.empty_rows[r] * p.ldy;
      for (int f = tid; f < p.F; f += blockDim.x) y[f] = 0.0f;
    }
    return;
  }
  float *rows = smem + (size_t)w * L.rows_per_warp();
  float *scs = smem + (size_t)WARPS * L.rows_per_warp() + (size_t)w * L.scores_per_warp();
  float *queue = smem + (size_t)WARPS * (L.rows_per_warp() + L.scores_per_warp()) + (size_t)w * L.queue_per_warp();
  if (lane == 0)
    for (int s = 0; s < S; ++s) mbar_init(&bars[w][s]);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncwarp();
  const int QE = L.qe(), RS = L.rslot(), SS = L.sslot(), BW = L.bw;
  const bool dst_scale = !ATT && scales_dst(p.weight);
  const uint32_t row_bytes = 4u * 4u * (uint32_t)BW;
  const uint32_t sc_bytes = (ATT && L.hs) ? 4u * 4u * (uint32_t)p.H : 0u;  // separate score gather
  const uint32_t xb = ATT ? 4u * (uint32_t)p.H : 16u;
  const int32_t nunits = g.n_units;
  unsigned long long t_start = 0, busy = 0, n_done = 0, t_unit = 0;
  if (p.trace) t_start = gtimer();
  int pslot = 0;       // producer: slot of the next quad to arm
  uint32_t ppar = 0;   // its phase parity
  int32_t ci = 0;
  for (int32_t c0 = 0; c0 < p.F; c0 += BWMAX, ++ci) {
    int32_t *ctr = p.ws_unit + ci;
    bool valid[NV];
    int32_t head[NV];
#pragma unroll
    for (int n = 0; n < NV; ++n) {
      const int32_t f = c0 + (n * 32 + lane) * VEC;
      valid[n] = f < p.F && (n * 32 + lane) * VEC < BW;
      head[n] = (ATT && valid[n]) ? f / p.Fh : 0;
    }
    const int hsh = ATT ? (lane & (p.H - 1)) : 0;
    // GAT scores of edge r of a quad: in the gathered row after the features
    // (merged map) or in the separate score slot
    const bool merged = ATT && L.hs == 0;
    const int sstr = merged ? BW : p.H;
    const float smxs = ATT ? fkey_decode(__ldg(p.smax + hsh)) : 0.0f;
    // ---- run-claim pipeline: C (atomic issued) -> B (descriptors loading) -> A (ready, first indices loading) -> P
    int32_t uC = 0;
    if (lane == 0) uC = atomicAdd(ctr, RUN);
    int4 dB = make_int4(0, 0, 0, -1), dA = dB, dP = dB;
    int32_t eB = 0, eA = 0, eP = 0, nB = 0, nA = 0, nP = 0;
    int32_t T0A = 0, T1A = 0, firstA = 0, T1P = 0;
    int32_t pp = 0, juP = 0, uendP = 0, ib0 = 0, icur = 0, inxt = 0;
    bool live = false;  // the producer has edges
    auto advance_run = [&]() {
      dP = dA;
      eP = eA;
      nP = nA;
      T1P = T1A;
      live = nP > 0;
      pp = T0A;
      juP = -1;
      uendP = T0A;
      ib0 = T0A;
      icur = firstA;
      inxt = (live && T0A + 32 + lane < T1P) ? ld_stream_i32(g.colidx_t + T0A + 32 + lane) : 0;
      dA = dB;
      eA = eB;
      nA = nB;
      T0A = __shfl_sync(0xffffffffu, dB.x, 0);
      T1A = __shfl_sync(0xffffffffu, eB, nB > 0 ? nB - 1 : 0);
      firstA = (nA > 0 && T0A + lane < T1A) ? ld_stream_i32(g.colidx_t + T0A + lane) : 0;
      const int32_t base = __shfl_sync(0xffffffffu, uC, 0);
      nB = base < nunits ? min(RUN, nunits - base) : 0;
      if (lane < nB) {
        dB = __ldg(g.unit_desc + base + lane);
        eB = __ldg(&g.unit_desc[base + lane + 1].x);
      }
      if (lane == 0) uC = atomicAdd(ctr, RUN);
    };
    advance_run();
    advance_run();
    advance_run();
    int32_t qt = 0, qh = 0;  // unit queue: tail (producer) / head (consumer)
    // ---- producer: the next four edges of the stream into slot pslot ----
    auto produce_quad = [&]() {
      int32_t r4[4] = {0, 0, 0, 0};
      int32_t xrow0 = 0, xrow1 = 0, xrow2 = 0, xrow3 = 0, xent0 = 0, xent1 = 0, xent2 = 0, xent3 = 0;
      int nx = 0, nvalid = 0;
      if (live && pp + 4 <= uendP && pp - ib0 <= 28) {  // fast path: four edges of the current unit and batch
#pragma unroll
        for (int r = 0; r < 4; ++r) r4[r] = __shfl_sync(0xffffffffu, icur, pp - ib0 + r);
        pp += 4;
        nvalid = 4;
      } else {
#pragma unroll
        for (int r = 0; r < 4; ++r) {
          if (live && pp == uendP) {  // next unit (possibly of the next run)
            if (++juP == nP) {
              advance_run();
              juP = 0;
            }
            if (live) {
              uendP = __shfl_sync(0xffffffffu, eP, juP);
              const int32_t urow = __shfl_sync(0xffffffffu, dP.z, juP);
              const int32_t ubeg = __shfl_sync(0xffffffffu, dP.y, juP);
              const int32_t um = __shfl_sync(0xffffffffu, dP.w, juP);
              const int32_t e = qt & (QN - 1);
              if (lane == 0) {
                int *qi = reinterpret_cast<int *>(queue + e * QE);
                qi[0] = urow;
                qi[1] = uendP - pp;  // length
                qi[2] = ubeg;
                qi[3] = um;
                qi[4] = pp;          // task position
              }
              if (ATT || dst_scale) {
                if (nx == 0) { xrow0 = urow; xent0 = e; }
                else if (nx == 1) { xrow1 = urow; xent1 = e; }
                else if (nx == 2) { xrow2 = urow; xent2 = e; }
                else { xrow3 = urow; xent3 = e; }
                ++nx;
              }
              ++qt;
            }
          }
          if (live) {
            if (pp - ib0 == 32) {
              icur = inxt;
              ib0 += 32;
              inxt = ib0 + 32 + lane < T1P ? ld_stream_i32(g.colidx_t + ib0 + 32 + lane) : 0;
            }
            r4[r] = __shfl_sync(0xffffffffu, icur, pp - ib0);
            ++pp;
            ++nvalid;
          }
        }
      }
      if (live && pp - ib0 == 32) {  // keep the batch window ahead of the fast path
        icur = inxt;
        ib0 += 32;
        inxt = ib0 + 32 + lane < T1P ? ld_stream_i32(g.colidx_t + ib0 + 32 + lane) : 0;
      }
      if (lane == 0) {
        uint64_t *bar = &bars[w][pslot];
        uint32_t bytes = (nvalid > 0 ? row_bytes + sc_bytes : 0u) + xb * (uint32_t)nx;
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // generic reads of the slot -> async writes
        mbar_expect(bar, bytes);
        if (nvalid > 0) {
          gather4(rows + (size_t)pslot * RS, &rmap, c0 >> L.esh, r4[0], r4[1], r4[2], r4[3], bar);
          if (ATT && !merged) gather4(scs + (size_t)pslot * SS, &smap, 0, r4[0], r4[1], r4[2], r4[3], bar);
        }
        for (int j = 0; j < nx; ++j) {
          const int32_t xr = j == 0 ? xrow0 : j == 1 ? xrow1 : j == 2 ? xrow2 : xrow3;
          const int32_t xe = j == 0 ? xent0 : j == 1 ? xent1 : j == 2 ? xent2 : xent3;
          float *dst = queue + xe * QE + 8;
          if (ATT) bulk_copy(dst, p.t + (int64_t)xr * p.ldt, xb, bar);
          else bulk_copy(dst, g.ndst + (xr & ~3), 16u, bar);
        }
      }
      if (++pslot == S) {
        pslot = 0;
        ppar ^= 1u;
      }
    };
    int cslot = pslot;       // consumer: slot / parity of the next quad to wait for
    uint32_t cpar = ppar;
    for (int k = 0; k < S; ++k) produce_quad();
    // ---- consumer ----
    Part<MODE, VEC, NV> G;
    float tvs = 0.0f, mbs = 0.0f, nmbs = 0.0f, seens = 0.0f, ls = 0.0f;  // GAT: head hsh's softmax state
    float ndstC = 1.0f;
    int32_t rowC = 0, lenC = 0, begC = 0, mC = -1, tposC = 0, posC = 0;
    bool more = true;
    while (more) {
      if (posC == 0 && qh == qt) break;  // every queued unit done and the producer is exhausted
      mbar_wait(&bars[w][cslot], cpar);
      const float *rq = rows + (size_t)cslot * RS;
      const float *sq = merged ? rq + (p.F - c0) : scs + (size_t)cslot * SS;
      int r = 0;
      while (r < 4) {
        if (posC == 0) {  // first edge of the next queued unit: its entry and extras have landed
          if (qh == qt) {
            more = false;
            break;
          }
          const float *qe = queue + (qh & (QN - 1)) * QE;
          const int *qi = reinterpret_cast<const int *>(qe);
          rowC = qi[0];
          lenC = qi[1];
          begC = qi[2];
          mC = qi[3];
          tposC = qi[4];
          part_init(G);
          if constexpr (ATT) {
            // shared softmax state: lane computes head hsh = lane % H (H a power of two)
            tvs = qe[8 + hsh];
            const float mb = leaky_f(smxs + tvs, p.slope);
            mbs = mb;
            nmbs = -mb * kLog2e;
            seens = -INFINITY;
            ls = 0.0f;
          } else {
            ndstC = dst_scale ? qe[8 + (rowC & 3)] : 1.0f;
          }
          if (p.trace) t_unit = gtimer();
        }
        const int kk = min(4 - r, lenC - posC);  // edges of this unit in the rest of the quad
        const bool one = lenC == 1;
        if (kk == 4) {
          // a whole quad of one unit (the common case): the four edges' terms
          // are independent, so they are issued back to back; the chain still
          // adds them in CSR order (bit-identical to the per-edge loop below)
          if constexpr (ATT) {
            float ex4[4];
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              const float sco = leaky_f(sq[j * sstr + hsh] + tvs, p.slope);
              seens = fmaxf(seens, sco);
              ex4[j] = ex2_f(fmaf(sco, kLog2e, nmbs));
            }
#pragma unroll
            for (int j = 0; j < 4; ++j) ls += ex4[j];
            // no per-lane guards in the fast path: a lane past F reads bytes
            // inside this warp's shared region (the slot's tail / the next
            // slot / the score and queue regions) and its sums are never stored
#pragma unroll
            for (int j = 0; j < 4; ++j) {
#pragma unroll
              for (int n = 0; n < NV; ++n) {
                const float exn = __shfl_sync(0xffffffffu, ex4[j], head[n]);
                float v[VEC];
                lds_vec<VEC>(rq + j * BW + (n * 32 + lane) * VEC, v);
                fma_vec<VEC>(G.a[n], v, exn);
              }
            }
          } else {
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              const float wt = 1.0f;  // weight 1 (pre-scaled GCN: ndst in the epilogue)
#pragma unroll
              for (int n = 0; n < NV; ++n) {  // unguarded, as above
                float v[VEC];
                lds_vec<VEC>(rq + j * BW + (n * 32 + lane) * VEC, v);
                if constexpr (MODE == M_MAX) {
#pragma unroll
                  for (int i = 0; i < VEC; ++i) G.a[n][i] = fmaxf(G.a[n][i], wt * v[i]);
                } else {
                  fma_vec<VEC>(G.a[n], v, wt);
                }
              }
            }
          }
          r = 4;
        } else
        for (int j = 0; j < kk; ++j, ++r) {
          const float *rb = rq + r * BW;
          if constexpr (ATT) {
            // e_uv and exp(e_uv - m) once per head (lane hsh), then to the lanes holding that head
            const float sco = leaky_f(sq[r * sstr + hsh] + tvs, p.slope);
            seens = fmaxf(seens, sco);
            const float ex = one ? 1.0f : ex2_f(fmaf(sco, kLog2e, nmbs));
            ls += ex;
#pragma unroll
            for (int n = 0; n < NV; ++n) {
              const float exn = __shfl_sync(0xffffffffu, ex, head[n]);
              if (!valid[n]) continue;
              float v[VEC];
              lds_vec<VEC>(rb + (n * 32 + lane) * VEC, v);
              fma_vec<VEC>(G.a[n], v, exn);
            }
          } else {
            const float wt = 1.0f;  // weight 1 (pre-scaled GCN: ndst in the epilogue)
#pragma unroll
            for (int n = 0; n < NV; ++n) {
              if (!valid[n]) continue;
              float v[VEC];
              lds_vec<VEC>(rb + (n * 32 + lane) * VEC, v);
              if constexpr (MODE == M_MAX) {
#pragma unroll
                for (int i = 0; i < VEC; ++i) G.a[n][i] = fmaxf(G.a[n][i], wt * v[i]);
              } else {
                fma_vec<VEC>(G.a[n], v, wt);
              }
            }
          }
        }
        posC += kk;
        if (posC == lenC) {
          if constexpr (ATT) {
            float tv[NV], seen[NV];
#pragma unroll
            for (int n = 0; n < NV; ++n) {  // the per-head state to the lanes of each vector
              G.m[n] = __shfl_sync(0xffffffffu, mbs, head[n]);
              G.l[n] = __shfl_sync(0xffffffffu, ls, head[n]);
              seen[n] = __shfl_sync(0xffffffffu, seens, head[n]);
              tv[n] = __shfl_sync(0xffffffffu, tvs, head[n]);
            }
            if (lenC == 1) {
#pragma unroll
              for (int n = 0; n < NV; ++n) G.m[n] = seen[n];
            } else {
              bool loose = false;
#pragma unroll
              for (int n = 0; n < NV; ++n) loose |= valid[n] && !(G.m[n] - seen[n] <= kGatSlack);
              if (__any_sync(0xffffffffu, loose)) gat_recompute_v<VEC, NV>(p, tposC, lenC, c0, lane, valid, head, tv, G, seen);
            }
          }
          finish_unit<MODE, VEC, NV, 32>(p, G, rowC, begC, mC, lenC, c0, ci, lane, 0xffffffffu, &ndstC);
          if (p.trace) {
            busy += gtimer() - t_unit;
            ++n_done;
          }
          ++qh;
          posC = 0;
        }
      }
      __syncwarp();  // every lane is done with this slot before it is refilled
      if (++cslot == S) {
        cslot = 0;
        cpar ^= 1u;
      }
      produce_quad();
    }
    // the quads armed after the last consumed one carry no edges (their phases completed on arrival)
    __syncwarp();
  }
  if (p.trace && lane == 0) {
    atomicAdd(p.trace + 0, busy);
    atomicAdd(p.trace + 1, 1ull);
    atomicMin(p.trace + 2, t_start);
    atomicMax(p.trace + 3, gtimer());
    atomicAdd(p.trace + 4, n_done);
    atomicMax(p.trace + 5, busy);
  }
}

namespace {
typedef CUresult (*EncodeTiledFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                  const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
EncodeTiledFn encode_fn() {
  static EncodeTiledFn fn = nullptr;
  static bool tried = false;
  if (!tried) {
    tried = true;
    void *f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = (EncodeTiledFn)f;
  }
  return fn;
}
// L2 promotion of the gathered rows' misses: a miss is fetched as the whole
// aligned 256-byte block when every row starts on one (C5 agg2: 1 KB rows);
// otherwise the largest block size the row starts stay aligned to, so at most
// the tail block of a row reaches outside it (GAT [z | s] rows of 1056 B at a
// 1088-byte stride: 256-byte promotion fetched 1280 B per row, 64-byte 1088).  env GNN_G4_PROMO = 0 / 64 / 128 / 256 forces one (A/B).
CUtensorMapL2promotion promotion(const float *base, int64_t ld) {
  static int forced = -2;
  if (forced == -2) {
    const char *e = getenv("GNN_G4_PROMO");
    forced = e ? atoi(e) : -1;
  }
  int blk = 256;
  if (forced >= 0) {
    blk = forced;
  } else {
    const uint64_t a = (uint64_t)(uintptr_t)base | (uint64_t)(ld * 4);
    while (blk > 32 && (a & (uint64_t)(blk - 1))) blk >>= 1;
  }
  return blk >= 256 ? CU_TENSOR_MAP_L2_PROMOTION_L2_256B
         : blk >= 128 ? CU_TENSOR_MAP_L2_PROMOTION_L2_128B
         : blk >= 64  ? CU_TENSOR_MAP_L2_PROMOTION_L2_64B
                      : CU_TENSOR_MAP_L2_PROMOTION_NONE;
}
// rows of `width` fp32 features, row stride ld (floats), boxes of box_w x 1
// (gather4 takes 4 box rows); esh = 1: the same bytes as 8-byte elements
// (width and box_w still in floats, even), so a box may span 512 floats
bool encode_rows(CUtensorMap *m, const float *base, int64_t nrows, int32_t width, int64_t ld, int32_t box_w,
                 int esh = 0) {
  if (!encode_fn() || ((uintptr_t)base & 15) || ((ld * 4) & 15) || nrows < 1 || nrows > 0x7fffffffLL) return false;
  if (esh && ((width | box_w) & 1)) return false;
  if ((box_w >> esh) > 256 || ((box_w * 4) & 15)) return false;
  const cuuint64_t dims[2] = {(cuuint64_t)(width >> esh), (cuuint64_t)nrows};
  const cuuint64_t strides[1] = {(cuuint64_t)ld * 4};
  const cuuint32_t box[2] = {(cuuint32_t)(box_w >> esh), 1};
  const cuuint32_t es[2] = {1, 1};
  return encode_fn()(m, esh ? CU_TENSOR_MAP_DATA_TYPE_FLOAT64 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void *)base,
                     dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                     promotion(base, ld),
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}
}  // namespace

// Does the gather4 kernel take this call?  Sum / mean / max with weight 1 or
// the pre-scaled GCN form, or GAT with H a power of two in 4..32;
// 16-byte aligned rows, F % 4 == 0 (DESIGN.md §5.2 rule).
bool g4_admissible(const KParams &kp, int32_t n_src) {
  if (!encode_fn() || n_src < 1) return false;
  if (kp.F % 4 || kp.ldx % 4 || ((uintptr_t)kp.X & 15)) return false;
  if (kp.add_row) return false;
  if (kp.mode == M_GAT) {  // heads: a power of two, 4..32 (16-byte score rows, one lane per head)
    if (kp.H < 4 || kp.H > 32 || (kp.H & (kp.H - 1)) || kp.Fh % 4 || kp.ldt % 4 || ((uintptr_t)kp.t & 15)) return false;
    if (((uintptr_t)(kp.X + kp.F) & 15)) return false;
    return true;
  }
  if (kp.mode > M_MAX) return false;
  // weight 1 or the pre-scaled GCN form (ndst per row); per-edge weights take
  // the cp.async chain (GCN nsrc[u] by 4-byte cp.async per edge tracked with
  // commit groups measured slower there: C3 13.6 vs 11.9 ms; agg1 12.9 vs 7.9)
  return kp.weight == GNN_W_ONE || kp.weight == W_DST_ONLY;
}

template <int MODE, int VEC, int NV>
static cudaError_t launch_g4_mode(const KParams &kp_in, int32_t n_src, cudaStream_t s) {
  using namespace g4;
  g4::Layout L;
  L.bw = kp_in.F < BWMAX ? kp_in.F : BWMAX;
  L.hs = MODE == M_GAT ? kp_in.H : 0;  // GAT score columns
  L.xe = MODE == M_GAT ? (kp_in.H < 4 ? 4 : kp_in.H) : 4;
  L.esh = 0;
  // GAT with one sweep (F <= 256): the H score columns that follow the
  // features ride in the same gather4 as the row (F + H floats as 8-byte
  // elements), one TMA request per quad instead of two (env GNN_G4_MERGED=0: two)
  static int merged_ok = -1;
  if (merged_ok < 0) {
    const char *e = getenv("GNN_G4_MERGED");
    merged_ok = (e && e[0] == '0') ? 0 : 1;
  }
  const bool merged = MODE == M_GAT && merged_ok && kp_in.F <= BWMAX && (kp_in.F + kp_in.H) % 4 == 0 &&
                      kp_in.F + kp_in.H <= 512 && kp_in.F + kp_in.H <= kp_in.ldx;
  CUtensorMap rmap, smap;
  memset(&rmap, 0, sizeof(rmap));
  memset(&smap, 0, sizeof(smap));
  if (merged) {
    L.bw = kp_in.F + kp_in.H;
    L.hs = 0;
    L.esh = 1;
    if (!encode_rows(&rmap, kp_in.X, n_src, L.bw, kp_in.ldx, L.bw, 1)) return cudaErrorNotSupported;
  } else {
    if (!encode_rows(&rmap, kp_in.X, n_src, kp_in.F, kp_in.ldx, L.bw)) return cudaErrorNotSupported;
    if (MODE == M_GAT && !encode_rows(&smap, kp_in.X + kp_in.F, n_src, kp_in.H, kp_in.ldx, kp_in.H))
      return cudaErrorNotSupported;
  }
  const size_t smem = L.bytes();
  static int occ = 0;
  auto fn = k_stream_g4<MODE, VEC, NV>;
  if (occ == 0) {
    cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, fn, WARPS * 32, smem);
    if (occ <= 0) occ = 1;
  }
  cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  KParams kp = kp_in;
  kp.nch = (kp.F + BWMAX - 1) / BWMAX;
  if (kp.nch > kp.n_unit_ctr) return cudaErrorInvalidValue;
  kp.n_persist = (int32_t)std::min<int64_t>((int64_t)num_sms() * occ, std::max<int64_t>(1, kp.g.n_units / RUN + 1));
  cudaError_t e = cudaMemsetAsync(kp.ws_unit, 0, sizeof(int32_t) * (size_t)kp.n_unit_ctr, s);
  if (e == cudaSuccess && kp.g.n_multi > 0)
    e = cudaMemsetAsync(kp.ws_cnt, 0, sizeof(int32_t) * (size_t)kp.g.n_multi * kp.nch, s);
  if (e == cudaSuccess && kp.g.n_multi > 0 && !kp.deterministic)  // sums and max keys start at 0
    e = cudaMemsetAsync(kp.ws_acc, 0, sizeof(float) * (size_t)kp.g.n_multi * kp.FW, s);
  if (e == cudaSuccess && kp.trace) {
    e = cudaMemsetAsync(kp.trace, 0, 8 * sizeof(unsigned long long), s);
    if (e == cudaSuccess) e = cudaMemsetAsync(kp.trace + 2, 0xff, sizeof(unsigned long long), s);
  }
  if (e != cudaSuccess) return e;
  const int64_t blocks = (int64_t)kp.n_persist + (kp.g.n_empty + 31) / 32;
  fn<<<(unsigned)blocks, WARPS * 32, smem, s>>>(kp, rmap, smap, L);
  count_launch();
  return cudaGetLastError();
}

// lane mapping of the consumer: VEC 4 (lane = features 4l and 128 + 4l), or
// env GNN_G4_VEC=8 (8 consecutive features; 2-way shared-memory bank conflicts)
static int g4_vec() {
  static int v = 0;
  if (v == 0) {
    const char *e = getenv("GNN_G4_VEC");
    v = (e && e[0] == '8') ? 8 : 4;  // measured: VEC 4 (conflict-free shared reads) 15.1 vs 17.9 ms on C5
  }
  return v;
}
cudaError_t launch_g4(const KParams &kp, int32_t n_src, cudaStream_t s) {
  const bool narrow = kp.F <= 128;  // one 128-feature vector per lane set
  const bool v8 = !narrow && g4_vec() == 8 && kp.F % 8 == 0;
  switch (kp.mode) {
    case M_SUM:
    case M_MEAN:
      return narrow ? launch_g4_mode<M_SUM, 4, 1>(kp, n_src, s)
                    : v8 ? launch_g4_mode<M_SUM, 8, 1>(kp, n_src, s) : launch_g4_mode<M_SUM, 4, 2>(kp, n_src, s);
    case M_MAX:
      return narrow ? launch_g4_mode<M_MAX, 4, 1>(kp, n_src, s)
                    : v8 ? launch_g4_mode<M_MAX, 8, 1>(kp, n_src, s) : launch_g4_mode<M_MAX, 4, 2>(kp, n_src, s);
    case M_GAT: return narrow ? cudaErrorNotSupported : launch_g4_mode<M_GAT, 4, 2>(kp, n_src, s);
    default: return cudaErrorNotSupported;
  }
}

}  // namespace gnn
