// k_gemm_tc.cu — a5: H = X W on the 5th-generation tensor cores (tcgen05,
// kind::tf32, accumulators in TMEM) with a 3xTF32 split so the result keeps
// fp32 accuracy (plain TF32 fails the 1e-4 bar):
//     X = Xhi + Xlo, W = Whi + Wlo  (hi = fp32 with the 13 low mantissa bits
//     cleared, exactly representable in TF32; lo = x - hi, exact in fp32)
//     H = Xlo Whi + Xhi Wlo + Xhi Whi      (Xlo Wlo ~ 2^-22 relative: dropped)
// Epilogue fused: row scale (GCN nsrc[u]), column bias, ReLU.
//
// Structure (persistent, one CTA per SM, 352 threads):
//   warps 0-3  producers: per 32-wide K block, the 128 x 32 X tile is split
//              into hi/lo in the UMMA K-major SWIZZLE_128B layout.  TMA path
//              (default when X/H rows are 16-byte aligned): warp 9 streams
//              the raw tile into the hi slot with one cp.async.bulk.tensor
//              (the tensor map's SWIZZLE_128B is the UMMA layout; out-of-range
//              K and M are zero-filled), and the producers split it in shared
//              memory (elementwise: hi in place, lo alongside); warp 10 bulk-
//              copies the pre-split, pre-swizzled W image of the K block
//              (built once per call by k_gemm_wimage into the caller's
//              workspace) into its own ring.  Register path (unaligned X, or
//              gnn_set_gemm_impl(3)): the producers load the tile from global
//              memory and one of them issues the W copy; one unified ring.
//   warp 4     MMA issuer: one elected lane issues 3 tcgen05.mma per 8-wide K
//              step per 256-column slice, commits stage release / tile done.
//   warps 5-8  epilogue: tcgen05.ld (32x32b: one TMEM lane = one row per
//              thread), fp32 sum of the partial accumulators, scale/bias/ReLU,
//              then (TMA path) a swizzled 32x32 staging buffer per warp and a
//              TMA bulk tensor store, or (register path) row-per-thread
//              stores.  Runs concurrently with the next tile's MMAs when TMEM
//              holds two tile buffers.
// Column blocks (TMA path, n > 256, <= 8 K blocks): each row tile is two
// work items over column slices of the W image, so both accumulators fit
// TMEM twice and the epilogue overlaps the next item's MMAs.
// CTA pairs (TMA path, default; env GNN_GEMM_CTA2=0 disables): clusters of 2
// CTAs, 256-row work items (128 rows per CTA), each CTA stages its X rows
// and half of the item's W columns; the leader's MMA warp issues
// tcgen05.mma.cta_group::2 (M = 256) once the peer's gate warp has arrived
// (remotely) on its per-stage barrier, and commits with .multicast::cluster
// to both CTAs' stage / tile barriers.  Halving the W stage halves the
// shared-memory operand reads per SM and leaves room for a third W stage.
// Accumulation drift: the tensor core's internal accumulation is not IEEE
// round-to-nearest, so long K chains drift; K blocks are spread round-robin
// over n_acc partial accumulators (summed in fp32 in the epilogue) so that no
// accumulator sees more than ~8 K blocks (<= 96 MMA accumulations).
#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#include "gnn_internal.h"
#include "tc_common.cuh"

namespace gnn {
namespace tc {

constexpr int NUM_PRODUCER_WARPS = 4;
constexpr int MMA_WARP = 4;
constexpr int EPI_WARP0 = 5;
constexpr int TMA_WARP = 9;   // TMA path: X tiles
constexpr int WIMG_WARP = 10; // TMA path: W image blocks
constexpr int THREADS = 32 * 11;      // register path
constexpr int EPI_WARP1 = 11;         // TMA path: second epilogue half (warps 11-14)
constexpr int THREADS_TMA = 32 * 15;
__host__ __device__ constexpr int threads_of(bool tma) { return tma ? THREADS_TMA : THREADS; }
constexpr int TILE_A_BYTES = BM * BK * 4;  // 16 KB per hi or lo
constexpr int MAX_STAGES = 8;

// W image: for each K block kb: [hi tile | lo tile], each NP rows (n) x 128 B,
// K-major, swizzled exactly as in shared memory.
__global__ void k_gemm_wimage(const float *__restrict__ W, int64_t ldw, int32_t k, int32_t n, int32_t np,
                              int32_t num_kb, uint8_t *img) {
  const int64_t total = (int64_t)num_kb * np * 8;
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < total; q += (int64_t)gridDim.x * blockDim.x) {
    const int32_t kb = (int32_t)(q / (np * 8));
    const int32_t rem = (int32_t)(q % (np * 8));
    const int32_t nn = rem >> 3, c = rem & 7;
    const int32_t gk = kb * BK + 4 * c;
    float w[4];
#pragma unroll
    for (int i = 0; i < 4; ++i) w[i] = (nn < n && gk + i < k) ? W[(int64_t)(gk + i) * ldw + nn] : 0.0f;
    float4 hi = make_float4(hi_of(w[0]), hi_of(w[1]), hi_of(w[2]), hi_of(w[3]));
    float4 lo = make_float4(w[0] - hi.x, w[1] - hi.y, w[2] - hi.z, w[3] - hi.w);
    uint8_t *base = img + (size_t)kb * 2 * np * 128;
    const uint32_t off = sw128_off(nn, c);
    *reinterpret_cast<float4 *>(base + off) = hi;
    *reinterpret_cast<float4 *>(base + (size_t)np * 128 + off) = lo;
  }
}

// mirror destinations (NEXT-2) as kernel parameters: one TMA map per mirror
// (same box as hmap) and its base pointer for the scalar score stores
struct MirrorMaps {
  CUtensorMap map[kMaxMirrors];
  float *base[kMaxMirrors];
  int32_t count;
};

struct TcParams {
  const float *X;
  int64_t ldx;
  float *H;
  int64_t ldh;
  const uint8_t *wimg;
  int64_t m;
  int32_t k, n, np, npa;  // np = n rounded to 16; npa = TMEM columns per accumulator
  int32_t num_kb, num_tiles;
  int32_t stages, n_acc, n_buf;
  int32_t sa, sb;  // TMA path: raw X ring (TMA destination, the A_hi operand) and B (W image) ring depths
  int32_t sl;      // TMA path: X_lo ring depth (written by the splitters)
  int32_t eb;      // TMA path with TMA stores: 4 KB staging buffers per epilogue warp (1 or 2)
  int32_t ncb, cbw0;  // TMA path: column blocks per row tile (1 or 2) and block 0's width
  int32_t epi8;    // TMA stores with 8 epilogue warps (two per TMEM lane quadrant, alternate column chunks)
  const float *row_scale;
  const float *col_bias;
  int32_t relu;
  // attention-score epilogue (GAT, Table 2; reading R5): when att
  // is set, the epilogue also writes s_v[h] = <y_v[h*Fh : (h+1)*Fh], a_src_h>
  // and t_v[h] = <y_v[h], a_dst_h> (att_dst) to columns att_col + h and
  // att_col + att_H + h of H.  Fh is a multiple of 32, so every 32-column
  // chunk belongs to one head, and each thread's chunks are contiguous.
  const float *att, *att_dst;
  int32_t att_H, att_Fh, att_col;
};

template <bool VEC_X, bool VEC_H, bool TMA_X, bool CTA2 = false>
__global__ void __launch_bounds__(threads_of(TMA_X), 1) k_gemm_tc(const TcParams p, const __grid_constant__ CUtensorMap xmap,
                                                          const __grid_constant__ CUtensorMap hmap,
                                                          const __grid_constant__ MirrorMaps mir) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t *smem = (uint8_t *)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  const int NP = p.np;
  const int B_BYTES = NP * 128;
  const int STAGE_BYTES = 2 * TILE_A_BYTES + 2 * B_BYTES;
  // register path: full/empty per unified stage [A | B].  TMA path: three
  // rings -- raw X: xfull (TMA bytes) -> aempty (MMA; the raw tile is the
  // A_hi operand: kind::tf32 reads the top 19 bits of each fp32, which is
  // exactly hi_of(x)); X_lo: afull (splitters) -> lempty (MMA); B: full (bulk
  // bytes) -> empty (MMA)
  __shared__ uint64_t full_bar[MAX_STAGES], empty_bar[MAX_STAGES], xfull_bar[MAX_STAGES], afull_bar[MAX_STAGES],
      aempty_bar[MAX_STAGES], lempty_bar[MAX_STAGES], tfull_bar[2], tempty_bar[2];
  // CTA pair: the peer's "stage it complete" gate, arrived remotely on the leader
  __shared__ uint64_t peer_bar[MAX_STAGES];
  __shared__ uint32_t tmem_base_sh;

  const int tid = threadIdx.x;
  const int warp = tid >> 5;
  const int lane = tid & 31;
  const int S = p.stages;
  // CTA pair (TMA path, cluster of 2): a row tile is 256 rows, 128 per CTA;
  // each CTA holds its rows of X and half of the item's W columns; the
  // leader (rank 0) issues the cta_group::2 MMAs for both
  const uint32_t crank = CTA2 ? cluster_ctarank() : 0u;
  const int cta_id = CTA2 ? (int)(blockIdx.x >> 1) : (int)blockIdx.x;
  const int n_cta = CTA2 ? (int)(gridDim.x >> 1) : (int)gridDim.x;
  constexpr int ROWS = CTA2 ? 2 * BM : BM;
  const int n_epi_warps = p.epi8 ? 8 : 4;

  if (tid == 0) {
    if (TMA_X) {
      for (int s = 0; s < p.sa; ++s) {
        mbar_init(&xfull_bar[s], 1);
        mbar_init(&aempty_bar[s], 1);
      }
      for (int s = 0; s < p.sl; ++s) {
        mbar_init(&afull_bar[s], NUM_PRODUCER_WARPS * 32);
        mbar_init(&lempty_bar[s], 1);
      }
      for (int s = 0; s < p.sb; ++s) {
        mbar_init(&full_bar[s], 1);
        mbar_init(&empty_bar[s], 1);
      }
    } else {
      for (int s = 0; s < S; ++s) {
        mbar_init(&full_bar[s], NUM_PRODUCER_WARPS * 32 / 2 + 1);  // 64 A arrivals (one group) + 1 expect_tx
        mbar_init(&empty_bar[s], 1);
      }
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&tfull_bar[b], 1);
      // pair: one arrival per epilogue warp of both CTAs (on the leader's barrier)
      mbar_init(&tempty_bar[b], CTA2 ? 2 * n_epi_warps : 128 * (p.epi8 ? 2 : 1));
    }
    if (CTA2)
      for (int s = 0; s < MAX_STAGES; ++s) mbar_init(&peer_bar[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == MMA_WARP) {
    if (CTA2) {
      asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tmem_base_sh)));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;");
    } else {
      asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tmem_base_sh)));
      asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
    }
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (CTA2) cluster_sync_all();  // both CTAs' barriers initialised before any remote arrive
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = tmem_base_sh;

  const int my_tiles = p.num_tiles > cta_id ? (p.num_tiles - 1 - cta_id) / n_cta + 1 : 0;
  const int total_it = my_tiles * p.num_kb;
  auto tile_of = [&](int it) { return cta_id + (it / p.num_kb) * n_cta; };
  // TMA path: work item vt = (row tile vt / ncb, column block vt % ncb); a
  // column block is a slice of the W image (rows cb_beg .. cb_beg + cb_w)
  auto cb_beg = [&](int vt) { return (p.ncb > 1 && vt % p.ncb) ? p.cbw0 : 0; };
  auto cb_w = [&](int vt) { return p.ncb > 1 ? ((vt % p.ncb) ? NP - p.cbw0 : p.cbw0) : NP; };
  const int B_STAGE = 2 * (p.ncb > 1 ? p.cbw0 : NP) * 128 / (CTA2 ? 2 : 1);  // TMA path B ring stage
  // TMA path smem: [raw X ring sa x 16 KB][X_lo ring sl x 16 KB][W ring sb x B_STAGE][epilogue staging]
  uint8_t *const lo_ring = smem + (size_t)p.sa * TILE_A_BYTES;
  uint8_t *const b_ring = lo_ring + (size_t)p.sl * TILE_A_BYTES;
  if (TMA_X && warp == TMA_WARP) {
    // ----------------------------- TMA issuer (X) -----------------------------
    if (lane == 0) {
      for (int it = 0; it < total_it; ++it) {
        const int s = it % p.sa, use = it / p.sa;
        if (use > 0) mbar_wait(&aempty_bar[s], (use - 1) & 1);
        mbar_arrive_expect_tx(&xfull_bar[s], TILE_A_BYTES);
        tma_load_2d(smem + (size_t)s * TILE_A_BYTES, &xmap, (it % p.num_kb) * BK,
                    (tile_of(it) / p.ncb) * ROWS + (int)crank * BM, &xfull_bar[s]);
      }
    }
  } else if (TMA_X && warp == WIMG_WARP) {
    // ------------------------ bulk-copy issuer (W image) ------------------------
    if (lane == 0) {
      for (int it = 0; it < total_it; ++it) {
        const int s = it % p.sb, use = it / p.sb;
        if (use > 0) mbar_wait(&empty_bar[s], (use - 1) & 1);
        const int vt = tile_of(it), w = cb_w(vt) / (CTA2 ? 2 : 1);  // pair: this CTA's half of the columns
        const int wb = w * 128;  // bytes of one (hi or lo) slice
#ifdef GNN_GEMM_DBG_NOW
        if (use >= p.sb) { mbar_arrive(&full_bar[s]); continue; }  // first fill only: MMAs read stale W
#endif
        mbar_arrive_expect_tx(&full_bar[s], 2 * wb);
        const uint8_t *src = p.wimg + (size_t)(it % p.num_kb) * 2 * B_BYTES + (size_t)(cb_beg(vt) + (int)crank * w) * 128;
        uint8_t *b_img = b_ring + (size_t)s * B_STAGE;
        for (int part = 0; part < 2; ++part)  // hi slice, then lo slice (stage layout [hi w | lo w])
          for (int off = 0; off < wb; off += 16384) {
            const int bytes = wb - off < 16384 ? wb - off : 16384;
            bulk_g2s(b_img + part * wb + off, src + (size_t)part * B_BYTES + off, bytes, &full_bar[s]);
          }
      }
    }
  } else if (TMA_X && warp < NUM_PRODUCER_WARPS) {
    // ---------------------- splitters: raw X tile -> lo ----------------------
    // The split is elementwise and lo shares the raw tile's swizzled layout,
    // so each thread converts fixed 16-byte chunks with no address arithmetic.
    // The raw tile stays in place as the A_hi operand.
    constexpr int NT = NUM_PRODUCER_WARPS * 32;
    constexpr int PER = TILE_A_BYTES / 16 / NT;  // 8 chunks per thread
    for (int it = 0; it < total_it; ++it) {
      const int s = it % p.sa, use = it / p.sa;
      const int l = it % p.sl, luse = it / p.sl;
      mbar_wait(&xfull_bar[s], use & 1);
#ifdef GNN_GEMM_DBG_NOSPLIT
      if (luse > 0) mbar_wait(&lempty_bar[l], (luse - 1) & 1);
      mbar_arrive(&afull_bar[l]);
      continue;
#endif
      const float4 *a_raw = reinterpret_cast<const float4 *>(smem + (size_t)s * TILE_A_BYTES);
      float4 x[PER];
#pragma unroll
      for (int i = 0; i < PER; ++i) x[i] = a_raw[tid + i * NT];
      if (luse > 0) mbar_wait(&lempty_bar[l], (luse - 1) & 1);
      float4 *a_lo = reinterpret_cast<float4 *>(lo_ring + (size_t)l * TILE_A_BYTES);
#pragma unroll
      for (int i = 0; i < PER; ++i) {
        const float4 hi = make_float4(hi_of(x[i].x), hi_of(x[i].y), hi_of(x[i].z), hi_of(x[i].w));
        a_lo[tid + i * NT] = make_float4(x[i].x - hi.x, x[i].y - hi.y, x[i].z - hi.z, x[i].w - hi.w);
      }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      mbar_arrive(&afull_bar[l]);
    }
  } else if (!TMA_X && warp < NUM_PRODUCER_WARPS) {
    // ------------------------------ producers ------------------------------
    // Two producer groups of 2 warps take alternate K blocks (group g handles
    // the global K-block counter it = g, g+2, ...); each group loads its next
    // X tile into registers before waiting for its stage, so two K blocks of
    // X are in flight per CTA while the MMAs run.
    constexpr int GROUP_THREADS = NUM_PRODUCER_WARPS * 32 / 2;           // 64
    constexpr int PER_THREAD = BM * 8 / GROUP_THREADS;                     // 16 float4 chunks
    const int grp = warp >> 1;                                             // 0 or 1
    const int gtid = tid - grp * GROUP_THREADS;
    float4 buf[PER_THREAD];
    auto load_a = [&](int64_t m0, int kb) {
      const int k0 = kb * BK;
#pragma unroll
      for (int i = 0; i < PER_THREAD; ++i) {
        const int q = gtid + i * GROUP_THREADS;
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
        buf[i] = x;
      }
    };
    int it = grp;
    if (it < total_it) load_a((int64_t)tile_of(it) * BM, it % p.num_kb);
    while (it < total_it) {
      const int kb = it % p.num_kb;
      const int s = it % S, use = it / S;
      if (use > 0) mbar_wait(&empty_bar[s], (use - 1) & 1);
      uint8_t *st = smem + (size_t)s * STAGE_BYTES;
      uint8_t *a_hi = st, *a_lo = st + TILE_A_BYTES, *b_img = st + 2 * TILE_A_BYTES;
      if (gtid == 0) {
        mbar_arrive_expect_tx(&full_bar[s], 2 * B_BYTES);
        const uint8_t *src = p.wimg + (size_t)kb * 2 * B_BYTES;
        for (int off = 0; off < 2 * B_BYTES; off += 16384) {
          const int bytes = 2 * B_BYTES - off < 16384 ? 2 * B_BYTES - off : 16384;
          bulk_g2s(b_img + off, src + off, bytes, &full_bar[s]);
        }
      }
#pragma unroll
      for (int i = 0; i < PER_THREAD; ++i) {
        const int q = gtid + i * GROUP_THREADS;
        const int r = q >> 3, c = q & 7;
        const float4 x = buf[i];
        const float4 hi = make_float4(hi_of(x.x), hi_of(x.y), hi_of(x.z), hi_of(x.w));
        const float4 lo = make_float4(x.x - hi.x, x.y - hi.y, x.z - hi.z, x.w - hi.w);
        const uint32_t off = sw128_off(r, c);
        *reinterpret_cast<float4 *>(a_hi + off) = hi;
        *reinterpret_cast<float4 *>(a_lo + off) = lo;
      }
      // generic-proxy smem writes -> visible to the tensor core (async proxy)
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      mbar_arrive(&full_bar[s]);
      it += 2;
      if (it < total_it) load_a((int64_t)tile_of(it) * BM, it % p.num_kb);
    }
  } else if (CTA2 && warp == MMA_WARP && crank != 0) {
    // ------------------- pair peer: gate its stages to the leader -------------------
    if (lane == 0)
      for (int it = 0; it < total_it; ++it) {
        mbar_wait(&xfull_bar[it % p.sa], (it / p.sa) & 1);
        mbar_wait(&afull_bar[it % p.sl], (it / p.sl) & 1);
        mbar_wait(&full_bar[it % p.sb], (it / p.sb) & 1);
        mbar_arrive_cluster(&peer_bar[it % MAX_STAGES], 0);
      }
    __syncwarp();
  } else if (warp == MMA_WARP) {
    // ------------------------------ MMA issuer ------------------------------
    int it = 0, tcount = 0;
    for (int tile = cta_id; tile < p.num_tiles; tile += n_cta, ++tcount) {
      const int b = tcount % p.n_buf, buse = tcount / p.n_buf;
      if (buse > 0) {
        if (CTA2) mbar_wait_cluster(&tempty_bar[b], (buse - 1) & 1);
        else mbar_wait(&tempty_bar[b], (buse - 1) & 1);
      }
      asm volatile("tcgen05.fence::after_thread_sync;");
      const uint32_t tbase = tmem + (uint32_t)(b * p.n_acc * p.npa);
      const int NW = TMA_X ? cb_w(tile) : NP;  // MMA width of this work item
      const uint32_t b_lo_off = TMA_X ? (uint32_t)(NW / (CTA2 ? 2 : 1)) * 128 : (uint32_t)B_BYTES;
      for (int kb = 0; kb < p.num_kb; ++kb, ++it) {
        int s, sA, sL = 0;
        uint32_t a_hi, a_lo, b_hi;
        if (TMA_X) {
          sA = it % p.sa;
          sL = it % p.sl;
          s = it % p.sb;
          mbar_wait(&xfull_bar[sA], (it / p.sa) & 1);
          mbar_wait(&afull_bar[sL], (it / p.sl) & 1);
          mbar_wait(&full_bar[s], (it / p.sb) & 1);
          if (CTA2) mbar_wait_cluster(&peer_bar[it % MAX_STAGES], (it / MAX_STAGES) & 1);
          a_hi = smem_u32(smem + (size_t)sA * TILE_A_BYTES);
          a_lo = smem_u32(lo_ring + (size_t)sL * TILE_A_BYTES);
          b_hi = smem_u32(b_ring + (size_t)s * B_STAGE);
        } else {
          s = sA = it % S;
          mbar_wait(&full_bar[s], (it / S) & 1);
          a_hi = smem_u32(smem + (size_t)s * STAGE_BYTES);
          a_lo = a_hi + TILE_A_BYTES;
          b_hi = a_hi + 2 * TILE_A_BYTES;
        }
        asm volatile("tcgen05.fence::after_thread_sync;");
        if (lane == 0) {
          const uint32_t b_lo = b_hi + b_lo_off;
          const int acc = kb % p.n_acc;
          const uint32_t d0 = tbase + (uint32_t)(acc * p.npa);
          const uint32_t first = (kb < p.n_acc) ? 1u : 0u;  // first K block of this accumulator
#ifndef GNN_GEMM_DBG_NOMMA
#pragma unroll
          for (int j = 0; j < BK / 8; ++j) {  // 8 tf32 (32 B) per MMA K step
            const uint32_t ko = j * 32;
            if (CTA2) {  // NW <= 256: one pair MMA per term
              const uint32_t id = idesc_tf32_pair(NW);
              mma_tf32_pair(d0, sw128_desc(a_lo + ko), sw128_desc(b_hi + ko), id, (first && j == 0) ? 0u : 1u);
              mma_tf32_pair(d0, sw128_desc(a_hi + ko), sw128_desc(b_lo + ko), id, 1u);
              mma_tf32_pair(d0, sw128_desc(a_hi + ko), sw128_desc(b_hi + ko), id, 1u);
              continue;
            }
            for (int n0 = 0; n0 < NW; n0 += 256) {
              const int nn = NW - n0 < 256 ? NW - n0 : 256;
              const uint32_t id = idesc_tf32(nn);
              const uint32_t bo = (uint32_t)n0 * 128;
              const uint32_t d = d0 + (uint32_t)n0;
              mma_tf32(d, sw128_desc(a_lo + ko), sw128_desc(b_hi + bo + ko), id, (first && j == 0) ? 0u : 1u);
              mma_tf32(d, sw128_desc(a_hi + ko), sw128_desc(b_lo + bo + ko), id, 1u);
              mma_tf32(d, sw128_desc(a_hi + ko), sw128_desc(b_hi + bo + ko), id, 1u);
            }
          }
#endif
          if (CTA2) {
            mma_commit_pair(&empty_bar[s]);
            mma_commit_pair(&aempty_bar[sA]);
            mma_commit_pair(&lempty_bar[sL]);
            if (kb == p.num_kb - 1) mma_commit_pair(&tfull_bar[b]);
          } else {
            mma_commit(&empty_bar[s]);
            if (TMA_X) {
              mma_commit(&aempty_bar[sA]);
              mma_commit(&lempty_bar[sL]);
            }
            if (kb == p.num_kb - 1) mma_commit(&tfull_bar[b]);
          }
        }
        __syncwarp();
      }
    }
  } else if ((warp >= EPI_WARP0 && warp < EPI_WARP0 + 4) ||
             (TMA_X && VEC_H && p.epi8 && warp >= EPI_WARP1 && warp < EPI_WARP1 + 4)) {
    // ------------------------------ epilogue ------------------------------
    const int ew = warp - EPI_WARP0;  // 0..3 -> TMEM lanes 32*ew (warp % 4 == ew + 1 ... see note)
    // TMEM lane quadrant accessible by a warp is (warp id % 4): warps 5,6,7,8 -> 1,2,3,0
    const int quad = warp & 3;
    (void)ew;
    // TMA path (VEC_H): each warp stages its 32 rows x 32 columns in a
    // SWIZZLE_128B buffer (row = lane, conflict-free float4 writes) and one
    // lane stores it with a TMA bulk tensor store (coalesced; tails clipped)
#ifdef GNN_GEMM_DBG_REGSTORE
    constexpr bool TMA_H = false;
#else
    constexpr bool TMA_H = TMA_X && VEC_H;
#endif
    // with 8 epilogue warps the two warps of a TMEM lane quadrant take
    // contiguous halves of the item's 32-column chunks (a head's chunks stay
    // with one thread for the attention-score epilogue)
    const int half = warp >= EPI_WARP1 ? 1 : 0;
    const int widx = half ? 4 + warp - EPI_WARP1 : warp - EPI_WARP0;
    uint8_t *const epi_buf = b_ring + (size_t)p.sb * B_STAGE + (size_t)widx * p.eb * 4096;
    int chunk = 0;
    int tcount = 0;
    for (int tile = cta_id; tile < p.num_tiles; tile += n_cta, ++tcount) {
      const int b = tcount % p.n_buf, buse = tcount / p.n_buf;
      mbar_wait(&tfull_bar[b], buse & 1);
      asm volatile("tcgen05.fence::after_thread_sync;");
      const int r = quad * 32 + lane;
      const int rt = TMA_H ? tile / p.ncb : tile;    // row tile
      const int cbb = TMA_H ? cb_beg(tile) : 0;      // first global column of this work item
      const int NW = TMA_H ? cb_w(tile) : NP;
      const int64_t row0 = (int64_t)rt * ROWS + (int64_t)crank * BM;  // this CTA's first row of the tile
      const int64_t gm = row0 + r;
      const float sc = (p.row_scale && gm < p.m) ? __ldg(p.row_scale + gm) : 1.0f;
      const uint32_t tbase = tmem + (uint32_t)(b * p.n_acc * p.npa) + ((uint32_t)(quad * 32) << 16);
      const int n_acc_used = p.num_kb < p.n_acc ? p.num_kb : p.n_acc;
      const int nchunk = (NW + 31) / 32;
      const int cmid = p.epi8 ? (nchunk + 1) / 2 : nchunk;
      float att_s = 0.0f, att_t = 0.0f;
      int att_h = -1;
      // attention scores of head att_h (complete): to columns att_col + h, att_col + H + h
      auto att_flush = [&]() {
        if (att_h >= 0 && gm < p.m) {
          p.H[gm * p.ldh + p.att_col + att_h] = att_s;
          p.H[gm * p.ldh + p.att_col + p.att_H + att_h] = att_t;
          for (int q = 0; q < mir.count; ++q) {  // the same scores into the mirrors (NEXT-2)
            mir.base[q][gm * p.ldh + p.att_col + att_h] = att_s;
            mir.base[q][gm * p.ldh + p.att_col + p.att_H + att_h] = att_t;
          }
        }
      };
#ifdef GNN_GEMM_DBG_NOEPI
      (void)att_flush;
      asm volatile("tcgen05.fence::before_thread_sync;");
      if (CTA2) {
        __syncwarp();
        if (lane == 0) mbar_arrive_cluster(&tempty_bar[b], 0);
      } else {
        mbar_arrive(&tempty_bar[b]);
      }
      continue;
#endif
      for (int c0 = (half ? cmid : 0) * 32; c0 < (half ? nchunk : cmid) * 32; c0 += 32) {
        float y[32];
#pragma unroll
        for (int i = 0; i < 32; ++i) y[i] = 0.0f;
        for (int a = 0; a < n_acc_used; ++a) {
          uint32_t v[32];
          const uint32_t taddr = tbase + (uint32_t)(a * p.npa + c0);
          asm volatile(
              "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
              "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
              : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
                "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]),
                "=r"(v[15]), "=r"(v[16]), "=r"(v[17]), "=r"(v[18]), "=r"(v[19]), "=r"(v[20]), "=r"(v[21]),
                "=r"(v[22]), "=r"(v[23]), "=r"(v[24]), "=r"(v[25]), "=r"(v[26]), "=r"(v[27]), "=r"(v[28]),
                "=r"(v[29]), "=r"(v[30]), "=r"(v[31])
              : "r"(taddr));
          asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
          for (int i = 0; i < 32; ++i) y[i] = (a == 0) ? __uint_as_float(v[i]) : y[i] + __uint_as_float(v[i]);
        }
        if (!TMA_H && gm >= p.m) continue;
#pragma unroll
        for (int i = 0; i < 32; ++i) {
          const int col = cbb + c0 + i;
          float t = y[i];
          if (p.row_scale) t = t * sc;
          if (p.col_bias && col < p.n) t = t + __ldg(p.col_bias + col);
          if (p.relu) t = t > 0.0f ? t : 0.0f;
          y[i] = t;
        }
        if (p.att) {
          const int h = (cbb + c0) / p.att_Fh;
          if (h != att_h) {
            att_flush();
            att_h = h;
            att_s = att_t = 0.0f;
          }
          const float *as = p.att + cbb + c0, *at = p.att_dst + cbb + c0;
          if (!(((uintptr_t)p.att | (uintptr_t)p.att_dst) & 15)) {  // 16-byte loads (warp-uniform)
#pragma unroll
            for (int i = 0; i < 32; i += 4) {
              const float4 a4 = __ldg(reinterpret_cast<const float4 *>(as + i));
              const float4 t4 = __ldg(reinterpret_cast<const float4 *>(at + i));
              att_s = fmaf(y[i + 3], a4.w, fmaf(y[i + 2], a4.z, fmaf(y[i + 1], a4.y, fmaf(y[i], a4.x, att_s))));
              att_t = fmaf(y[i + 3], t4.w, fmaf(y[i + 2], t4.z, fmaf(y[i + 1], t4.y, fmaf(y[i], t4.x, att_t))));
            }
          } else {
#pragma unroll
            for (int i = 0; i < 32; ++i) {
              att_s = fmaf(y[i], __ldg(as + i), att_s);
              att_t = fmaf(y[i], __ldg(at + i), att_t);
            }
          }
        }
        if constexpr (TMA_H) {
          uint8_t *buf = epi_buf + (chunk % p.eb) * 4096;
          if (chunk >= p.eb) {
            if (lane == 0) {
              if (p.eb == 2) bulk_wait_read<1>();
              else bulk_wait_read<0>();
            }
            __syncwarp();
          }
#pragma unroll
          for (int c = 0; c < 8; ++c)
            *reinterpret_cast<float4 *>(buf + lane * 128 + ((c ^ (lane & 7)) << 4)) =
                make_float4(y[4 * c], y[4 * c + 1], y[4 * c + 2], y[4 * c + 3]);
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          __syncwarp();
          if (lane == 0) {
            // the chunk to H and to every mirror (peer replicas, NEXT-2), one bulk group
            tma_store_2d_nc(&hmap, cbb + c0, (int32_t)(row0 + quad * 32), buf);
            for (int q = 0; q < mir.count; ++q) tma_store_2d_nc(&mir.map[q], cbb + c0, (int32_t)(row0 + quad * 32), buf);
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
          }
          ++chunk;
          continue;
        }
        float *dst = p.H + gm * p.ldh + c0;
        if (VEC_H && c0 + 32 <= p.n) {
#pragma unroll
          for (int i = 0; i < 32; i += 4) *reinterpret_cast<float4 *>(dst + i) = make_float4(y[i], y[i + 1], y[i + 2], y[i + 3]);
        } else {
#pragma unroll
          for (int i = 0; i < 32; ++i)
            if (c0 + i < p.n) dst[i] = y[i];
        }
      }
      if (p.att) att_flush();
      asm volatile("tcgen05.fence::before_thread_sync;");
      if (CTA2) {
        __syncwarp();
        if (lane == 0) mbar_arrive_cluster(&tempty_bar[b], 0);
      } else {
        mbar_arrive(&tempty_bar[b]);
      }
    }
    if (TMA_H && lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    if (mir.count > 0) __threadfence_system();  // peer stores performed before the kernel ends
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (CTA2) cluster_sync_all();  // the leader's last commits land in the peer; the peer's arrives in the leader
  if (warp == MMA_WARP) {
    asm volatile("tcgen05.fence::after_thread_sync;");
    if (CTA2) asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, 512;" ::"r"(tmem));
    else asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
  }
}

struct Config {
  int np, npa, num_kb, stages, n_acc, n_buf;
  int sa, sb, sl, eb, epi8;
  int ncb, cbw0, npa_t, nbuf_t, nacc_t;  // TMA path: column blocks and their TMEM layout
  int cta2;                              // TMA path: CTA pairs (cta_group::2)
  size_t smem, smem_tma, wimg_bytes;
};

static int g_epi8 = -1;  // 8 epilogue warps on the TMA path (A/B switch: env GNN_GEMM_EPI8=0 disables)
static int g_cb = -1;  // column blocks on the TMA path (A/B switch: env GNN_GEMM_CB=0 disables)
static int g_cta2 = -1;  // CTA pairs on the TMA path (A/B switch: env GNN_GEMM_CTA2=0/1)
static bool configure(int64_t m, int32_t k, int32_t n, Config &c) {
  if (n < 1 || n > 512 || k < 1 || m < 1) return false;
  c.np = (n + 15) / 16 * 16;
  c.npa = 32;
  while (c.npa < c.np) c.npa *= 2;
  c.num_kb = (k + BK - 1) / BK;
  c.wimg_bytes = (size_t)c.num_kb * 2 * c.np * 128;
  const int stage_bytes = 2 * TILE_A_BYTES + 2 * c.np * 128;
  c.stages = 6;
  while (c.stages > 2 && (size_t)c.stages * stage_bytes + 2048 > 200 * 1024) --c.stages;
  c.smem = (size_t)c.stages * stage_bytes + 1024;
  if (c.smem > 227 * 1024) return false;
  // TMA path, outputs wider than 256 columns with <= 8 K blocks: two column
  // blocks per row tile (widths cbw0 = a multiple of 32, and np - cbw0), so
  // each accumulator fits 256 TMEM columns and the epilogue of one block
  // overlaps the MMAs of the next (a 272-column accumulator cannot be
  // double-buffered in 512 columns).  The X tile is read twice (L2 hit).
  if (g_cb < 0) {
    const char *e = getenv("GNN_GEMM_CB");
    g_cb = (e && e[0] == '0') ? 0 : (e && e[0] == '2') ? 2 : 1;
  }
  c.ncb = 1;
  c.cbw0 = c.np;
  if (g_cb && (c.np > 256 || (g_cb == 2 && c.np == 256)) && c.num_kb <= 8) {
    c.ncb = 2;
    c.cbw0 = (c.np / 2 + 31) / 32 * 32;
    if (c.cbw0 > 256 || c.np - c.cbw0 < 16) {
      c.ncb = 1;
      c.cbw0 = c.np;
    }
  }
  // CTA pairs (cta_group::2): every work item <= 256 columns and >= 32 (the
  // pair MMA's N), so each CTA holds half of the item's W columns
  if (g_cta2 < 0) {
    const char *e = getenv("GNN_GEMM_CTA2");
    g_cta2 = (e && e[0] == '0') ? 0 : 1;
  }
  c.cta2 = 0;
  if (g_cta2) {
    const bool ok1 = c.ncb == 1 && c.np >= 32 && c.np <= 256;
    const bool ok2 = c.ncb == 2 && c.cbw0 >= 32 && c.cbw0 <= 256 && c.np - c.cbw0 >= 32 && c.np - c.cbw0 <= 256;
    c.cta2 = (ok1 || ok2) ? 1 : 0;
  }
  // TMA path: raw X ring (sa x 16 KB, the TMA destination and A_hi), X_lo
  // ring (sl = 2 x 16 KB), W ring (sb x 2 x cbw0 x 128 B), epilogue staging
  // (8 warps x eb x 4 KB).  The X loads come from HBM and need the depth
  // (ncu r2: the MMA warp waited on X 33% of the time with 2 stages), so the
  // raw ring gets what is left after W (2 stages) and the staging (eb = 1).
  {
    const size_t budget = 225 * 1024, b_bytes = 2 * (size_t)c.cbw0 * 128 / (c.cta2 ? 2 : 1);
    if (g_epi8 < 0) {
      const char *e = getenv("GNN_GEMM_EPI8");
      g_epi8 = (e && e[0] == '0') ? 0 : 1;
    }
    static int env_sa = -2, env_sb = -2, env_sl = -2;
    if (env_sa == -2) {
      const char *e = getenv("GNN_GEMM_SA");
      env_sa = e ? atoi(e) : -1;
      e = getenv("GNN_GEMM_SB");
      env_sb = e ? atoi(e) : -1;
      e = getenv("GNN_GEMM_SL");
      env_sl = e ? atoi(e) : -1;
    }
    static int env_eb = -2;
    if (env_eb == -2) {
      const char *e = getenv("GNN_GEMM_EB");
      env_eb = e ? atoi(e) : -1;
    }
    c.sl = env_sl >= 2 && env_sl <= MAX_STAGES ? env_sl : 2;
    // W ring: 3 stages when the pair halves them (measured: GEMM1/2/3 0.97 /
    // 1.50 / 1.67 ms vs 1.05 / 1.56 / 1.71 with 2; profiles/r02_gemm_pair.txt)
    c.sb = env_sb >= 2 && env_sb <= MAX_STAGES ? env_sb : (c.cta2 ? 3 : 2);
    c.epi8 = g_epi8 ? 1 : 0;
    c.eb = 1;
    auto need = [&](int sa, int sb, int eb, int e8) {
      return (size_t)(sa + c.sl) * TILE_A_BYTES + (size_t)sb * b_bytes + (size_t)eb * (e8 ? 8 : 4) * 4096 + 1024;
    };
    if (c.epi8 && need(2, 2, 1, 1) > budget) c.epi8 = 0;
    c.sa = 2;
    const int sa_max = env_sa > 1 && env_sa <= MAX_STAGES ? env_sa : MAX_STAGES;
    while (c.sa < sa_max && need(c.sa + 1, c.sb, c.eb, c.epi8) <= budget) ++c.sa;
    if (env_eb == 2) {  // A/B: two staging buffers per epilogue warp before X depth
      while (c.sa > 2 && need(c.sa, c.sb, 2, c.epi8) > budget) --c.sa;
    }
    if (need(c.sa, c.sb, 2, c.epi8) <= budget) c.eb = 2;
    c.smem_tma = need(c.sa, c.sb, c.eb, c.epi8);
    if (c.smem_tma > budget) c.sa = 0;  // TMA path unavailable for this n
  }
  // TMEM: n_buf tile buffers x n_acc accumulators x npa columns <= 512
  const int slots = 512 / c.npa;  // accumulators that fit
  if (slots < 1) return false;
  if (c.num_kb <= 8 && slots >= 2) {
    c.n_buf = 2;  // overlap the epilogue with the next tile
    c.n_acc = slots / 2;
  } else {
    c.n_buf = 1;
    c.n_acc = slots;
  }
  const int need_acc = (c.num_kb + 7) / 8;  // keep <= 8 K blocks per accumulator when possible
  if (c.n_acc > need_acc) c.n_acc = need_acc;
  if (c.n_acc < 1) c.n_acc = 1;
  c.npa_t = c.npa;
  c.nbuf_t = c.n_buf;
  c.nacc_t = c.n_acc;
  if (c.ncb > 1) {  // both blocks <= 256 columns: double buffer, one accumulator (<= 8 K blocks)
    c.npa_t = 256;
    c.nbuf_t = 2;
    c.nacc_t = 1;
  }
  return true;
}

}  // namespace tc

namespace tc {
// cuTensorMapEncodeTiled through the runtime's driver entry point (no -lcuda)
typedef CUresult (*EncodeTiledFn)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *, const cuuint64_t *,
                                  const cuuint64_t *, const cuuint32_t *, const cuuint32_t *, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
static EncodeTiledFn encode_fn() {
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
static int g_tma_mode = 1;  // 1 = TMA-fed X tiles when the layout allows, 0 = register path
static bool tma_enabled() { return g_tma_mode != 0 && encode_fn() != nullptr; }
// X [m, k] row stride ldx (elements): box 32 (K) x 128 (rows), SWIZZLE_128B
// (= the UMMA K-major layout), out-of-range elements zero-filled
static bool encode_x_map(CUtensorMap *map, const float *X, int64_t ldx, int64_t m, int32_t k) {
  if (((uintptr_t)X & 15) || ((ldx * 4) & 15)) return false;
  const cuuint64_t dims[2] = {(cuuint64_t)k, (cuuint64_t)m};
  const cuuint64_t strides[1] = {(cuuint64_t)ldx * 4};
  const cuuint32_t box[2] = {(cuuint32_t)BK, (cuuint32_t)BM};
  const cuuint32_t estr[2] = {1, 1};
  return encode_fn()(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void *)X, dims, strides, box, estr,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}
// H [m, n] row stride ldh: box 32 (columns) x 32 (rows), SWIZZLE_128B (the
// epilogue's staging layout); stores outside [m, n] are clipped
static bool encode_h_map(CUtensorMap *map, float *H, int64_t ldh, int64_t m, int32_t n) {
  if (((uintptr_t)H & 15) || ((ldh * 4) & 15)) return false;
  const cuuint64_t dims[2] = {(cuuint64_t)n, (cuuint64_t)m};
  const cuuint64_t strides[1] = {(cuuint64_t)ldh * 4};
  const cuuint32_t box[2] = {32, 32};
  const cuuint32_t estr[2] = {1, 1};
  return encode_fn()(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, (void *)H, dims, strides, box, estr,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_NONE,
                     CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}
}  // namespace tc

void gemm_tc_set_tma(int on) { tc::g_tma_mode = on ? 1 : 0; }

// Column slices: an output wider than one launch takes (the W image stages of
// 2 x np x 128 B no longer fit shared memory, n > 320 with K > 256 or n > 512)
// is computed as ceil(n / 256) launches over column slices of equal width
// (a multiple of 32, <= 256); each re-reads X (L2 or HBM).  Returns the
// columns per launch (n when one launch takes the whole width).
static int32_t slice_width(int64_t m, int32_t k, int32_t n) {
  tc::Config c;
  if (tc::configure(m > 0 ? m : 1, k, n, c)) return n;
  const int32_t nsl = (n + 255) / 256;
  return ((n + nsl - 1) / nsl + 31) / 32 * 32;
}

size_t gemm_tc_workspace(int64_t m, int32_t k, int32_t n) {
  if (n < 1 || k < 1) return 0;
  tc::Config c;
  if (!tc::configure(m > 0 ? m : 1, k, slice_width(m, k, n), c)) return 0;
  return (c.wimg_bytes + 255) & ~(size_t)255;
}

struct AttEpi {
  const float *a = nullptr, *a_dst = nullptr;  // [H * Fh] each
  int32_t H = 0, Fh = 0, col = 0;
};
static cudaError_t launch_gemm_tc_one(const float *X, int64_t ldx, const float *W, int64_t ldw, float *H, int64_t ldh,
                                      int64_t m, int32_t k, int32_t n, const float *row_scale, const float *col_bias,
                                      int32_t relu, void *ws, size_t ws_bytes, cudaStream_t s,
                                      const AttEpi &att = AttEpi(), const GemmMirrors *mir = nullptr,
                                      int32_t mir_col = 0);

// Returns cudaErrorNotSupported only for shapes no launch takes (k < 1) or a
// missing / misaligned workspace, cudaErrorInvalidValue for a workspace that
// is too small (the caller reports GNN_ERR_WORKSPACE).
cudaError_t launch_gemm_tc(const float *X, int64_t ldx, const float *W, int64_t ldw, float *H, int64_t ldh,
                           int64_t m, int32_t k, int32_t n, const float *row_scale, const float *col_bias,
                           int32_t relu, void *ws, size_t ws_bytes, cudaStream_t s, const GemmMirrors *mir) {
  if (k < 1 || n < 1 || !ws || ((uintptr_t)ws & 15)) return cudaErrorNotSupported;
  if (ws_bytes < gemm_tc_workspace(m, k, n)) return cudaErrorInvalidValue;
  const int32_t sw = slice_width(m, k, n);
  for (int32_t c0 = 0; c0 < n; c0 += sw) {
    const int32_t w = n - c0 < sw ? n - c0 : sw;
    cudaError_t e = launch_gemm_tc_one(X, ldx, W + c0, ldw, H + c0, ldh, m, k, w, row_scale,
                                       col_bias ? col_bias + c0 : nullptr, relu, ws, ws_bytes, s, AttEpi(), mir, c0);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

// GAT transform with the attention scores in the epilogue (reading R5):
// [Z | s | t] with Z = X W (n = H * Fh columns on the tensor cores) and
// s[h] = Z_h . a_src_h, t[h] = Z_h . a_dst_h accumulated in fp32 from the
// epilogue's Z values.  Needs Fh % 32 == 0 and a single launch for the width;
// returns cudaErrorNotSupported otherwise (the caller folds the scores into
// extra GEMM columns instead).
cudaError_t launch_gemm_att(const float *X, int64_t ldx, const float *W, int64_t ldw, float *Z, int64_t ldz, int64_t m,
                            int32_t k, int32_t H, int32_t Fh, const float *a_src, const float *a_dst, void *ws,
                            size_t ws_bytes, cudaStream_t s, const GemmMirrors *mir) {
  const int32_t n = H * Fh;
  if (Fh % 32 != 0 || k < 1 || !ws || ((uintptr_t)ws & 15) || slice_width(m, k, n) != n) return cudaErrorNotSupported;
  AttEpi att;
  att.a = a_src;
  att.a_dst = a_dst;
  att.H = H;
  att.Fh = Fh;
  att.col = n;
  return launch_gemm_tc_one(X, ldx, W, ldw, Z, ldz, m, k, n, nullptr, nullptr, 0, ws, ws_bytes, s, att, mir, 0);
}

static cudaError_t launch_gemm_tc_one(const float *X, int64_t ldx, const float *W, int64_t ldw, float *H, int64_t ldh,
                                      int64_t m, int32_t k, int32_t n, const float *row_scale, const float *col_bias,
                                      int32_t relu, void *ws, size_t ws_bytes, cudaStream_t s, const AttEpi &att,
                                      const GemmMirrors *mir, int32_t mir_col) {
  using namespace tc;
  Config c;
  if (!configure(m, k, n, c)) return cudaErrorNotSupported;
  if (ws_bytes < c.wimg_bytes) return cudaErrorInvalidValue;
  static int num_sms = 0;
  if (num_sms == 0) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&num_sms, cudaDevAttrMultiProcessorCount, dev);
    if (num_sms <= 0) num_sms = 148;
  }
  uint8_t *img = (uint8_t *)ws;
  {
    const int64_t total = (int64_t)c.num_kb * c.np * 8;
    const int blocks = (int)((total + 255) / 256 < 4096 ? (total + 255) / 256 : 4096);
    k_gemm_wimage<<<blocks, 256, 0, s>>>(W, ldw, k, n, c.np, c.num_kb, img);
    count_launch();
  }
  const int64_t rows_per_tile = c.cta2 ? 2 * BM : BM;  // a pair tile is 256 rows
  const int64_t num_tiles0 = (m + BM - 1) / BM;
  if (num_tiles0 > 0x3fffffff) return cudaErrorNotSupported;
  TcParams p{X, ldx, H, ldh, img, m, k, n, c.np, c.npa, c.num_kb, (int32_t)num_tiles0, c.stages, c.n_acc, c.n_buf,
             c.sa, c.sb, c.sl, c.eb, 1, c.np, c.epi8, row_scale, col_bias, relu, att.a, att.a_dst, att.H, att.Fh, att.col};
  const bool vx = (ldx % 4 == 0) && ((uintptr_t)X % 16 == 0);
  const bool vh = (ldh % 4 == 0) && ((uintptr_t)H % 16 == 0);
  CUtensorMap xmap;
  memset(&xmap, 0, sizeof(xmap));
  // TMA needs 16-byte aligned rows (vx) and a 32-bit row coordinate
  CUtensorMap hmap;
  memset(&hmap, 0, sizeof(hmap));
  const bool tma = vx && c.sa > 0 && (vh || c.ncb == 1) && tma_enabled() && m < 0x7fffff00LL && encode_x_map(&xmap, X, ldx, m, k) &&
                   (!vh || encode_h_map(&hmap, H, ldh, m, n));
  // mirrors: one TMA map each over the same rows / columns (needs the TMA-store epilogue)
  MirrorMaps mm;
  memset(&mm, 0, sizeof(mm));
  if (mir && mir->count > 0) {
    if (!(tma && vh) || mir->count > kMaxMirrors) return cudaErrorNotSupported;
    for (int q = 0; q < mir->count; ++q) {
      float *d = mir->dst[q] + mir_col;
      if (!d || ((uintptr_t)d & 15) || !encode_h_map(&mm.map[q], d, ldh, m, n)) return cudaErrorNotSupported;
      mm.base[q] = d;
    }
    mm.count = mir->count;
  }
  const bool pair = tma && c.cta2;
  const int64_t num_tiles = pair ? (m + rows_per_tile - 1) / rows_per_tile : num_tiles0;
  p.num_tiles = (int32_t)num_tiles;
  auto fn = pair ? (vh ? k_gemm_tc<true, true, true, true> : k_gemm_tc<true, false, true, true>)
          : tma ? (vh ? k_gemm_tc<true, true, true> : k_gemm_tc<true, false, true>)
                : vx ? (vh ? k_gemm_tc<true, true, false> : k_gemm_tc<true, false, false>)
                     : (vh ? k_gemm_tc<false, true, false> : k_gemm_tc<false, false, false>);
  const size_t smem = tma ? c.smem_tma : c.smem;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  if (!(tma && vh)) p.epi8 = 0;
  if (tma && c.ncb > 1) {  // column blocks (vh holds here)
    p.ncb = c.ncb;
    p.cbw0 = c.cbw0;
    p.npa = c.npa_t;
    p.n_buf = c.nbuf_t;
    p.n_acc = c.nacc_t;
    p.num_tiles = (int32_t)(num_tiles * c.ncb);
  }
  if (att.a) {
    // every work item must hold whole heads, and with 8 epilogue warps the
    // boundary between the two halves of an item's chunks must fall between heads
    const int ws0 = p.ncb > 1 ? p.cbw0 : c.np, ws1 = p.ncb > 1 ? c.np - p.cbw0 : c.np;
    if (ws0 % att.Fh != 0 || ws1 % att.Fh != 0) return cudaErrorNotSupported;
    for (int w : {ws0, ws1})
      if ((((w + 31) / 32 + 1) / 2 * 32) % att.Fh != 0) p.epi8 = 0;
  }
  if (pair) {
    // one persistent CTA pair per co-resident cluster slot (clusters of 2
    // share a TPC), or one per work item when there are fewer
    cudaLaunchConfig_t cfg = {};
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = 2;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.blockDim = dim3(threads_of(true));
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    static int max_clusters[2] = {0, 0};  // per epilogue variant (vh)
    int &mc = max_clusters[vh ? 1 : 0];
    cfg.gridDim = dim3(2 * (num_sms / 2));
    if (mc == 0) {
      int nc = 0;
      if (cudaOccupancyMaxActiveClusters(&nc, fn, &cfg) != cudaSuccess || nc < 1) {
        (void)cudaGetLastError();
        nc = num_sms / 2;
      }
      mc = nc;
    }
    const int clusters = (int)(p.num_tiles < mc ? p.num_tiles : mc);
    cfg.gridDim = dim3(2 * clusters);
    e = cudaLaunchKernelEx(&cfg, fn, p, xmap, hmap, mm);
    count_launch();
    return e != cudaSuccess ? e : cudaGetLastError();
  }
  // one persistent CTA per SM, or one per work item when there are fewer
  const int grid = (int)(p.num_tiles < num_sms ? p.num_tiles : num_sms);
  fn<<<grid, threads_of(tma), smem, s>>>(p, xmap, hmap, mm);
  count_launch();
  return cudaGetLastError();
}

}  // namespace gnn
