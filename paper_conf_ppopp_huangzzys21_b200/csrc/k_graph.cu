// k_graph.cu — sm_100a graph kernels of libgnn.so:
//   a1 degrees / GCN normalisers, a2 MinHash signatures, a6/a7/a8/a9 the
//   aggregation kernel family (sum, mean, max, fused GAT) with neighbor
//   grouping, feature-length-adaptive lane mapping and split-row combine.
//
// Paper: Huang et al., PPoPP'21 (PAPER.md P:<line>).  Design: DESIGN.md §5.
#include <cuda_runtime.h>
#include <math.h>
#include <stdint.h>

#include <algorithm>
#include <mutex>
#include <vector>

#include "k_agg.cuh"

namespace gnn {

// ---------------------------------------------------------------------------
// a1: degrees and GCN normalisers (Table 2 GCN P:263-269, reading R1):
// d_out(u) = #CSR entries equal to u (integer atomics: exact, order-free),
// nsrc = 1/sqrtf(d_out), ndst = 1/sqrtf(d_in), 0 for degree 0.  IEEE sqrt
// and div (no fast-math) so the values are bit-identical to the host formula.
// ---------------------------------------------------------------------------
__global__ void k_count_out(const int32_t *__restrict__ colidx, int64_t nnz, int32_t *d_out) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nnz;
       k += (int64_t)gridDim.x * blockDim.x)
    atomicAdd(d_out + colidx[k], 1);
}

__global__ void k_normalisers(const int32_t *__restrict__ rowptr, const int32_t *__restrict__ d_out,
                              int64_t n, int64_t n_src, float *nsrc, float *ndst) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (n > n_src ? n : n_src);
       i += (int64_t)gridDim.x * blockDim.x) {
    if (i < n_src) {
      int32_t d = d_out[i];
      nsrc[i] = d > 0 ? 1.0f / sqrtf((float)d) : 0.0f;
    }
    if (i < n) {
      int32_t d = rowptr[i + 1] - rowptr[i];
      ndst[i] = d > 0 ? 1.0f / sqrtf((float)d) : 0.0f;
    }
  }
}

cudaError_t launch_degrees(const int32_t *rowptr, const int32_t *colidx, int64_t n, int64_t n_src,
                           int64_t nnz, const int32_t *src_degree_override, int32_t *d_out_tmp,
                           float *nsrc, float *ndst, cudaStream_t s) {
  const int32_t *dout = src_degree_override;
  if (!dout) {
    cudaError_t e = cudaMemsetAsync(d_out_tmp, 0, sizeof(int32_t) * (size_t)(n_src > 0 ? n_src : 1), s);
    if (e != cudaSuccess) return e;
    if (nnz > 0) {
      int blocks = (int)std::min<int64_t>((nnz + 255) / 256, 148 * 16);
      k_count_out<<<blocks, 256, 0, s>>>(colidx, nnz, d_out_tmp);
      count_launch();
    }
    dout = d_out_tmp;
  }
  int64_t m = std::max<int64_t>(std::max(n, n_src), 1);
  int blocks = (int)std::min<int64_t>((m + 255) / 256, 148 * 16);
  k_normalisers<<<blocks, 256, 0, s>>>(rowptr, dout, n, n_src, nsrc, ndst);
  count_launch();
  return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// a2 step 1: Min-Hashing (reading R7).  One warp per row, lane k
// owns hash k: sig[v][k] = min over u in N(v) of fmix64(u + c_k).  Integer
// only -> bit-exact with the oracle.  K <= 64 (two salts per lane above 32).
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint64_t fmix64_dev(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

__global__ void k_minhash(const int32_t *__restrict__ rowptr, const int32_t *__restrict__ colidx,
                          int64_t n, int32_t K, const uint64_t *__restrict__ salts, uint64_t *sig) {
  const int lane = threadIdx.x & 31;
  const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const uint64_t c0 = lane < K ? salts[lane] : 0, c1 = lane + 32 < K ? salts[lane + 32] : 0;
  for (int64_t v = warp; v < n; v += nwarps) {
    const int32_t beg = rowptr[v], end = rowptr[v + 1];
    uint64_t m0 = ~0ULL, m1 = ~0ULL;
    for (int32_t base = beg; base < end; base += 32) {
      const int32_t cnt = min(32, end - base);
      const uint32_t mine = lane < cnt ? (uint32_t)__ldg(colidx + base + lane) : 0u;
      for (int32_t j = 0; j < cnt; ++j) {
        const uint64_t u = (uint64_t)__shfl_sync(0xffffffffu, mine, j);
        const uint64_t h0 = fmix64_dev(u + c0);
        m0 = h0 < m0 ? h0 : m0;
        if (K > 32) {
          const uint64_t h1 = fmix64_dev(u + c1);
          m1 = h1 < m1 ? h1 : m1;
        }
      }
    }
    if (lane < K) sig[v * K + lane] = m0;
    if (lane + 32 < K) sig[v * K + lane + 32] = m1;
  }
}

cudaError_t launch_minhash(const int32_t *rowptr, const int32_t *colidx, int64_t n, int32_t K,
                           uint64_t seed, uint64_t *sig, cudaStream_t s) {
  // salts c_k = k-th SplitMix64 output from `seed` (same stream as the oracle's
  // definition; computed here independently)
  uint64_t salts_h[64];
  uint64_t st = seed;
  for (int k = 0; k < K; ++k) {
    st += 0x9E3779B97F4A7C15ULL;
    uint64_t z = st;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    salts_h[k] = z ^ (z >> 31);
  }
  uint64_t *salts_d = nullptr;
  cudaError_t e = cudaMalloc(&salts_d, sizeof(uint64_t) * 64);
  if (e != cudaSuccess) return e;
  e = cudaMemcpyAsync(salts_d, salts_h, sizeof(uint64_t) * K, cudaMemcpyHostToDevice, s);
  if (e == cudaSuccess && n > 0) {
    int blocks = (int)std::min<int64_t>((n * 32 + 255) / 256, 148 * 32);
    k_minhash<<<blocks, 256, 0, s>>>(rowptr, colidx, n, K, salts_d, sig);
    count_launch();
    e = cudaGetLastError();
  }
  cudaError_t e2 = cudaStreamSynchronize(s);
  cudaFree(salts_d);
  return e != cudaSuccess ? e : e2;
}

// ---------------------------------------------------------------------------
// GAT softmax reference (reading R9 GAT): smax[h] = max over the source rows
// of s_u[h], as order-preserving keys (exact, order-free).  One strided pass
// over the H score columns (n_src x H x 4 B, ~3% of the aggregation's reads).
// ---------------------------------------------------------------------------
__global__ void k_score_max(const float *__restrict__ S, int64_t lds, int64_t n_src, int32_t H, int32_t len,
                            uint32_t *smax) {
  __shared__ uint32_t red[256];
  const int per = blockDim.x / H;  // rows per block pass; blockDim.x = per * H
  const int h = threadIdx.x % H, r = threadIdx.x / H;
  uint32_t k = 0;
  for (int64_t row = blockIdx.x * (int64_t)per + r; row < n_src; row += (int64_t)gridDim.x * per) {
    float x;
    if (len == 1) {
      x = __ldg(S + row * lds + h);
    } else {  // Euclidean norm of the head's len-vector (GaAN's Cauchy-Schwarz bound)
      float q = 0.0f;
      for (int32_t i = 0; i < len; ++i) {
        const float y = __ldg(S + row * lds + (int64_t)h * len + i);
        q = fmaf(y, y, q);
      }
      x = sqrtf(q) * 1.0000005f;  // round up past sqrt's rounding (the bound must not fall below)
    }
    k = max(k, fkey(x));
  }
  red[threadIdx.x] = k;
  __syncthreads();
  if (r == 0) {
    for (int j = 1; j < per; ++j) k = max(k, red[j * H + h]);
    atomicMax(smax + h, k);
  }
}

cudaError_t launch_score_max(const float *S, int64_t lds, int64_t n_src, int32_t H, int32_t len, uint32_t *smax,
                             cudaStream_t s) {
  cudaError_t e = cudaMemsetAsync(smax, 0, sizeof(uint32_t) * (size_t)H, s);
  if (e != cudaSuccess || n_src == 0) return e;
  const int threads = H <= 256 ? (256 / H) * H : 0;
  if (threads == 0) return cudaErrorInvalidValue;
  const int per = threads / H;
  const int blocks = (int)std::max<int64_t>(1, std::min<int64_t>((n_src + per - 1) / per, (int64_t)num_sms() * 8));
  k_score_max<<<blocks, threads, 0, s>>>(S, lds, n_src, H, len, smax);
  count_launch();
  return cudaGetLastError();
}

// y[v][f] = ReLU?(y[v][f] * scale[v]) (the postponed normaliser of a source-block accumulation)
__global__ void k_scale_rows(float *Y, int64_t ldy, int64_t n, int32_t F, const float *scale, int32_t relu) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n * F; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t v = i / F;
    float *y = Y + v * ldy + (i % F);
    float t = *y * __ldg(scale + v);
    if (relu) t = t > 0.0f ? t : 0.0f;
    *y = t;
  }
}

cudaError_t launch_scale_rows(float *Y, int64_t ldy, int64_t n, int32_t F, const float *scale, int32_t relu,
                              cudaStream_t s) {
  if (n == 0 || F == 0) return cudaSuccess;
  const int blocks = (int)std::min<int64_t>((n * F + 255) / 256, (int64_t)num_sms() * 16);
  k_scale_rows<<<blocks, 256, 0, s>>>(Y, ldy, n, F, scale, relu);
  count_launch();
  return cudaGetLastError();
}

// GAT atomic variant: exact per-row score maxima of the split rows,
// ws_rowmax[m][h] = max over the row's entries of LeakyReLU(s_u[h] + t_v[h])
// (monotone: the same value the deterministic merge reaches).  One warp per row.
__global__ void k_row_score_max(const KParams p) {
  const int lane = threadIdx.x & 31;
  const int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const DevGraph &g = p.g;
  for (int64_t m = w; m < g.n_multi; m += nw) {
    const int32_t row = g.multi_row[m];
    const int32_t rb = g.rowptr[row], re = g.rowptr[row + 1];
    for (int32_t h = 0; h < p.H; ++h) {
      const float tv = __ldg(p.t + (int64_t)row * p.ldt + h);
      float mx = -INFINITY;
      for (int32_t k = rb + lane; k < re; k += 32) {
        const int32_t u = __ldg(g.colidx + k);
        mx = fmaxf(mx, leaky_f(__ldg(p.X + (int64_t)u * p.ldx + p.F + h) + tv, p.slope));
      }
      for (int off = 16; off > 0; off >>= 1) mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, off));
      if (lane == 0) p.ws_rowmax[m * p.H + h] = mx;
    }
  }
}

cudaError_t launch_row_score_max(const KParams &kp, cudaStream_t s) {
  const int64_t blocks = std::min<int64_t>((kp.g.n_multi * 32 + 255) / 256, (int64_t)num_sms() * 8);
  k_row_score_max<<<(unsigned)std::max<int64_t>(1, blocks), 256, 0, s>>>(kp);
  count_launch();
  return cudaGetLastError();
}

// head mean (final attention layer): y[v][f] = (1/H) sum_h Yf[v][h*Fh + f], heads in order
__global__ void k_head_mean(const float *__restrict__ Yf, int64_t ldf, int64_t n, int32_t H, int32_t Fh, float *Y,
                            int64_t ldy) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n * Fh; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t v = i / Fh;
    const int32_t f = (int32_t)(i % Fh);
    float y = 0.0f;
    for (int32_t h = 0; h < H; ++h) y += Yf[v * ldf + (int64_t)h * Fh + f];
    Y[v * ldy + f] = y / (float)H;
  }
}

cudaError_t launch_head_mean(const float *Yf, int64_t ldf, int64_t n, int32_t H, int32_t Fh, float *Y, int64_t ldy,
                             cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  const int blocks = (int)std::min<int64_t>((n * Fh + 255) / 256, (int64_t)num_sms() * 16);
  k_head_mean<<<blocks, 256, 0, s>>>(Yf, ldf, n, H, Fh, Y, ldy);
  count_launch();
  return cudaGetLastError();
}

// ---------------------------------------------------------------------------
// host dispatch
// ---------------------------------------------------------------------------
static bool aligned(const void *ptr, int bytes) {
  return ptr == nullptr || (reinterpret_cast<uintptr_t>(ptr) % (uintptr_t)bytes) == 0;
}


// feature chunks one call may sweep (sizes the per-chunk counters): the
// automatic rule needs <= ceil(F/32); an override up to 8
static int32_t max_chunks(int32_t F) { return std::max<int32_t>(8, (F + 31) / 32); }

// process-wide mapping override (gnn_set_agg_mapping; the tuner hook)
static Mapping g_override{0, 0, 0};

bool mapping_supported(int32_t vec, int32_t lanes, int32_t nv) {
  const bool vec_ok = vec == 1 || vec == 2 || vec == 4 || vec == 8;
  const bool lanes_ok = lanes == 4 || lanes == 8 || lanes == 16 || lanes == 32;
  const bool nv_ok = nv == 1 || ((nv == 2 || nv == 4) && lanes == 32 && !(vec == 8 && nv == 4)) ||
                     (vec >= 2 && lanes == 16 && nv == 2) || (vec >= 4 && lanes == 8 && nv == 4);
  return vec_ok && lanes_ok && nv_ok;
}

bool set_agg_mapping(int32_t vec, int32_t lanes, int32_t nv) {
  if (vec == 0 && lanes == 0 && nv == 0) {
    g_override = Mapping{0, 0, 0};
    return true;
  }
  if (!mapping_supported(vec, lanes, nv)) return false;
  g_override = Mapping{vec, lanes, nv};
  return true;
}

bool agg_override_active() { return g_override.vec != 0; }

// L2 residency of hot source rows.  In a power-law graph a few sources carry
// a large share of the gathered rows (C5: the top 60,000 of 2.45 M sources by
// out-degree, 63 MB at F = 256, are 19.8 % of the edge references).  Before an
// aggregation whose source rows do not fit in L2, their lines are brought in
// with evict_last priority (prefetch.global.L2::evict_last), so the LAS-ordered
// stream of the other rows evicts around them; after the kernel they go back
// to evict_normal (applypriority), so later kernels see an ordinary L2.  Cache
// hints only: results are bit-identical.  Same box, C5 (profiles r3s): agg1
// 7.53 -> 7.23-7.38 ms, agg2 14.34 -> 14.16-14.24, GAT 16.52-16.60 ->
// 16.43-16.52 (pin + unpin included).  env GNN_L2_PIN=0 switches it off.
constexpr int32_t kHotMax = 65536;       // hot rows kept per plan
constexpr size_t kHotBytes = 32u << 20;  // bytes of rows pinned per launch (of the 126 MB L2)
template <bool LAST>
__global__ void k_l2_pin(const int32_t *rows, int32_t n, const char *X, int64_t ldb, int32_t row_bytes) {
  const int lane = threadIdx.x & 31;
  const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t w = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; w < n; w += nw) {
    const uintptr_t b = (uintptr_t)(X + (int64_t)rows[w] * ldb);
    const uintptr_t l0 = b & ~(uintptr_t)127, l1 = b + (uintptr_t)row_bytes;
    for (uintptr_t a = l0 + (uintptr_t)lane * 128; a < l1; a += 32 * 128) {
      if (LAST) asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(a));
      else asm volatile("applypriority.global.L2::evict_normal [%0], 128;" ::"l"(a));
    }
  }
}
static bool l2_pin_enabled() {
  static int v = -1;
  if (v < 0) {
    const char *e = getenv("GNN_L2_PIN");
    v = (e && e[0] == '0') ? 0 : 1;
  }
  return v == 1;
}
// the plan's hot list: the kHotMax sources of highest out-degree (ties by id),
// in degree order; built once per plan from the device out-degrees
static void build_hot(const gnn_plan_s *p) {
  if (p->n_src <= 0 || !p->d_dout) return;
  std::vector<int32_t> deg((size_t)p->n_src);
  if (cudaMemcpy(deg.data(), p->d_dout, sizeof(int32_t) * deg.size(), cudaMemcpyDeviceToHost) != cudaSuccess) {
    (void)cudaGetLastError();
    return;
  }
  const int32_t k = (int32_t)std::min<int64_t>(kHotMax, p->n_src);
  std::vector<int32_t> ids((size_t)p->n_src);
  for (int64_t i = 0; i < p->n_src; ++i) ids[(size_t)i] = (int32_t)i;
  auto hotter = [&](int32_t x, int32_t y) { return deg[x] != deg[y] ? deg[x] > deg[y] : x < y; };
  std::nth_element(ids.begin(), ids.begin() + (k - 1), ids.end(), hotter);
  std::sort(ids.begin(), ids.begin() + k, hotter);
  int32_t *d = nullptr;
  if (cudaMalloc(&d, sizeof(int32_t) * (size_t)k) != cudaSuccess) {
    (void)cudaGetLastError();
    return;
  }
  if (cudaMemcpy(d, ids.data(), sizeof(int32_t) * (size_t)k, cudaMemcpyHostToDevice) != cudaSuccess) {
    (void)cudaGetLastError();
    cudaFree(d);
    return;
  }
  p->d_hot = d;
  p->n_hot = k;
}
// rows to pin for this launch (0: none -- off, or the source rows fit in L2 anyway)
static int32_t hot_rows_for(const gnn_plan_s *p, int64_t row_bytes) {
  if (!l2_pin_enabled() || row_bytes <= 0) return 0;
  if ((double)p->n_src * (double)row_bytes <= 4.0 * (double)kHotBytes) return 0;
  std::call_once(p->hot_once, build_hot, p);
  return (int32_t)std::min<int64_t>(p->n_hot, (int64_t)(kHotBytes / (size_t)row_bytes));
}
// process-wide load-balance trace buffer (gnn_set_agg_trace), device, 8 x u64
static unsigned long long *g_trace = nullptr;
void set_agg_trace(void *dev_buf) { g_trace = reinterpret_cast<unsigned long long *>(dev_buf); }

static bool is_pow2(int x) { return x > 0 && (x & (x - 1)) == 0; }

static bool vec_admissible(const AggArgs &a, int32_t fh_or_0, int v) {
  bool ok = a.F % v == 0 && a.ldx % v == 0 && a.ldy % v == 0 && aligned(a.X, 4 * v) && aligned(a.Y, 4 * v);
  if (a.add_row) ok = ok && a.ld_add % v == 0 && aligned(a.add_row, 4 * v);
  if (fh_or_0) ok = ok && fh_or_0 % v == 0;
  if (vec_score(a.mode))  // GaAN / Gene: k_v or b_v (and W_a) read as vectors; the head's lanes a power of 2
    ok = ok && a.ldk % v == 0 && aligned(a.kb, 4 * v) && aligned(a.Wa, 4 * v) && is_pow2(fh_or_0 / v) &&
         fh_or_0 / v <= 32;
  return ok;
}

// a4: feature-length-adaptive mapping rule
static bool mapping_ok(const AggArgs &a, int32_t fh_or_0, const Mapping &o) {
  if (o.vec == 0 || !vec_admissible(a, fh_or_0, o.vec)) return false;
  // the Table 2 scores other than GAT are instantiated with one vector per lane
  if (a.mode > M_GAT && o.nv != 1) return false;
  if (vec_score(a.mode) && fh_or_0 / o.vec > o.lanes) return false;
  // GaAN / Gene: a chunk must hold whole heads (the score is a butterfly sum
  // over the head's lanes).  Scalar scores (GAT, Sym-GAT, Linear) may split a
  // head across chunks: each chunk keeps its own softmax state per head.
  const int cw = o.vec * o.lanes * o.nv;
  const bool heads_ok = !vec_score(a.mode) || cw >= a.F || cw % fh_or_0 == 0;
  return heads_ok && (a.F + cw - 1) / cw <= max_chunks(a.F);
}

bool agg_mapping_ok(const AggArgs &a, int32_t fh_or_0, int32_t vec, int32_t lanes, int32_t nv) {
  return mapping_supported(vec, lanes, nv) && mapping_ok(a, fh_or_0, Mapping{vec, lanes, nv});
}

// cp.async-staged kernel (a4 rule): sum / mean / max and
// GAT with 16-byte vectors, rows of >= 64 features; one warp per group, 128
// (NV = 1) or 256 (NV = 2) features per sweep.  A/B switch: env GNN_AGG_CP=0.
static int g_agg_cp = -1;
static bool cp_admissible(const gnn_plan_s *p, const AggArgs &a, int32_t fh_or_0) {
  (void)p;
  if (g_agg_cp < 0) {
    const char *e = getenv("GNN_AGG_CP");
    g_agg_cp = (e && e[0] == '0') ? 0 : (e && e[0] == '1') ? 1 : 2;  // default: gather4 streaming where it applies
  }
  if (!g_agg_cp || a.mode > M_GAT || a.F < 64 || a.ldx >= (1LL << 30)) return false;  // (32-bit row pitch in bytes)
  if (a.mode == M_GAT && (a.H > 32 || fh_or_0 % 4 != 0)) return false;
  return vec_admissible(a, fh_or_0, 4);
}

static Mapping choose_mapping(const gnn_plan_s *p, const AggArgs &a, int32_t fh_or_0) {
  Mapping m{1, 4, 1};
  if (mapping_ok(a, fh_or_0, g_override)) return g_override;
  // the plan's tuned mapping (gnn_tune_aggregate) for this width
  const Mapping t{p->tuned_vec, p->tuned_lanes, p->tuned_nv};
  if (p->tuned_F == a.F && mapping_ok(a, fh_or_0, t)) return t;
  if (cp_admissible(p, a, fh_or_0)) {
    // staged kernels with the (4, 32, NV) lane mapping: cp = 1 the cp.async
    // chain, cp = 2 the gather4 streaming kernel (launch_aggregate falls back
    // to the cp.async chain if gather4 cannot take the call)
    Mapping c{4, 32, a.F > 128 ? 2 : 1};
    // sum / mean / max: the cp.async chain for every width (two 128-feature
    // vectors per lane, 256-feature chunks, 8-slot ring): it measured faster
    // than gather4 at every F in 144..256 on C5 (agg2 F=256 prescaled 13.9 vs
    // 14.5 ms, DRAM 84.4 vs 93.6 GB: a narrower window of the task order in
    // flight); A/B: env GNN_G4_SUM=1 sends rows of > 128 features to gather4,
    // GNN_G4_NARROW=1 also the 64..128-feature rows
    static int g4_sum = -1, g4_narrow = -1;
    if (g4_sum < 0) {
      const char *e = getenv("GNN_G4_SUM");
      g4_sum = (e && e[0] == '1') ? 1 : 0;
      e = getenv("GNN_G4_NARROW");
      g4_narrow = (e && e[0] == '1') ? 1 : 0;
    }
    c.cp = ((a.F > 128 && g4_sum) || g4_narrow) ? g_agg_cp : std::min(g_agg_cp, 1);
    if (a.mode == M_GAT) {
      // GAT, rows of > 128 features: the lean cp.async chain (C5 8x32, same
      // box: 16.9-17.4 vs 17.4-17.6 ms on gather4, DRAM 96.7 vs 101.5 GB; the
      // register kernel 19.6-19.7 ms); A/B: env GNN_G4_GAT=1 takes gather4
      // (scores in the row's request, 64-byte L2 promotion), GNN_CP_GAT=0 the
      // register kernel; up to 128 features the register kernel
      static int g4_gat = -1, cp_gat = -1, cp_gat_narrow = -1;
      if (g4_gat < 0) {
        const char *e = getenv("GNN_G4_GAT");
        g4_gat = (e && e[0] == '1') ? 1 : 0;
        e = getenv("GNN_CP_GAT");
        cp_gat = (e && e[0] == '0') ? 0 : 1;
        e = getenv("GNN_CP_GAT_NARROW");  // A/B: 64..128-feature GAT rows on the lean chain too
        cp_gat_narrow = (e && e[0] == '1') ? 1 : 0;
      }
      if (a.F > 128 && g4_gat) c.cp = g_agg_cp == 2 ? 2 : 0;
      else if ((a.F > 128 || cp_gat_narrow) && cp_gat) c.cp = g_agg_cp ? 1 : 0;
      else c.cp = 0;
    }
    if (c.cp) return c;
  }
  const int cands[4] = {8, 4, 2, 1};
  m.vec = 0;
  for (int v : cands) {
    if (vec_admissible(a, fh_or_0, v)) {
      m.vec = v;
      break;
    }
  }
  if (m.vec == 0) return Mapping{0, 0, 0};  // only the vector scores can fail (head size)
  // short rows (average degree < 32) and narrow features: the chain of a
  // group is latency-bound, so one 32-lane worker per group with 16-byte
  // vectors (32 indices per batch, 8 source rows in flight) beats narrow
  // workers (tuner on C1 F=16: 30 -> 21 us; C2 F=64: 0.226 -> 0.147 ms)
  const double avg_deg = p->n > 0 ? (double)p->nnz / (double)p->n : 0.0;
  if (avg_deg < 32.0 && a.F <= 128 && a.mode <= M_GAT) {
    // vectors of F/32 floats so that all 32 lanes hold features (C2 GAT 8x8:
    // (2, 32, 1) 170 us vs 241 us for the default (8, 8, 1))
    int v = 1;
    while (v * 2 <= 4 && v * 2 * 32 <= a.F) v *= 2;
    while (v > 1 && !vec_admissible(a, fh_or_0, v)) v >>= 1;
    if (vec_admissible(a, fh_or_0, v)) return Mapping{v, 32, 1};
  }
  const int nvec = a.F / m.vec;  // vectors per row
  int lanes = 4;
  while (lanes < nvec && lanes < 32) lanes *= 2;
  m.lanes = lanes;
  m.nv = 1;
  if (lanes == 32 && nvec <= 32 && !fh_or_0 && m.vec >= 4) {
    // 17..32 vectors: two 16-lane workers per warp with two vectors per lane
    // halve the per-edge index/shuffle/address work per warp (measured on C5:
    // F=100 10.95 -> 9.72 ms, F=256 14.67 -> 14.23 ms; GAT 8x32 is faster
    // with one 32-lane worker: 19.2 vs 21.0 ms)
    m.lanes = 16;
    m.nv = 2;
  } else if (lanes == 32 && a.mode <= M_GAT) {
    const int max_nv = m.vec == 8 ? 2 : 4;
    while (m.nv < max_nv && 32 * m.nv < nvec) m.nv *= 2;
  }
  return m;
}


// Workspace layout (every region 256-byte aligned):
//   [unit counters: one int32 per feature chunk (<= max_chunks(F))]
//   [attention score maxima: H or 2H order-encoded keys]
//   [arrival counters: n_multi x max_chunks(F)]
//   [atomic accumulators: n_multi x FW][group partial slots: multi_slots x FW]
static size_t smax_bytes(int mode, int32_t H) {
  const size_t keys = (mode == M_GAT || mode == M_GAAN) ? (size_t)H : (mode == M_SYM ? 2 * (size_t)H : 0);
  return (sizeof(uint32_t) * keys + 255) & ~(size_t)255;
}
static size_t a256(size_t b) { return (b + 255) & ~(size_t)255; }
// partial-slot width: F, plus for attention the softmax state (m, l) of every
// (feature chunk, head) pair the chunk touches -- at most H + nch of them, so
// a head split across two chunks keeps one (m, l) per chunk -- rounded up to
// 8 floats so every slot row is 32-byte aligned for the vector stores
static int32_t att_meta(int mode, int32_t F, int32_t H) { return is_att(mode) ? H + max_chunks(F) : 0; }
static int32_t slot_width(int mode, int32_t F, int32_t H) { return (F + 2 * att_meta(mode, F, H) + 7) / 8 * 8; }

struct WsLayout {
  size_t unit, smax, cnt, acc, part, rowmax, total;
};
static WsLayout ws_layout(const gnn_plan_s *p, int mode, int32_t F, int32_t H) {
  const size_t FW = (size_t)slot_width(mode, F, H);
  WsLayout L;
  L.unit = 0;
  L.smax = L.unit + a256(sizeof(int32_t) * (size_t)max_chunks(F));
  L.cnt = L.smax + smax_bytes(mode, H);
  L.acc = L.cnt + a256(sizeof(int32_t) * (size_t)p->n_multi * max_chunks(F));
  L.part = L.acc + sizeof(float) * (size_t)p->n_multi * FW;
  L.rowmax = L.part + sizeof(float) * (size_t)p->multi_slots * FW;
  L.total = L.rowmax + (is_att(mode) ? sizeof(float) * (size_t)p->n_multi * (size_t)(H > 0 ? H : 0) : 0);
  return L;
}

size_t agg_workspace_bytes(const gnn_plan_s *p, int mode, int32_t F, int32_t H) {
  return ws_layout(p, mode, F, H).total;
}

int num_sms() {
  static int n = 0;
  if (n == 0) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

static gnn_status launch_aggregate_kernel(const gnn_plan_s *p, KParams &kp, Mapping m, int mode, int threads,
                                          cudaStream_t s);

gnn_status launch_aggregate(const gnn_plan_s *p, const AggArgs &a, void *ws, size_t ws_bytes, cudaStream_t s) {
  if (a.F <= 0) return GNN_OK;
  const int mode = a.mode;
  const size_t need = agg_workspace_bytes(p, mode, a.F, a.H);
  if (ws == nullptr || ws_bytes < need) {
    set_error("workspace too small: need " + std::to_string(need) + " bytes");
    return GNN_ERR_WORKSPACE;
  }
  KParams kp{};
  kp.g = p->dg;
  kp.mode = mode;
  kp.weight = a.weight;
  kp.edge_w = a.edge_w;
  kp.X = a.X;
  kp.ldx = a.ldx;
  kp.F = a.F;
  kp.Y = a.Y;
  kp.ldy = a.ldy;
  kp.add_row = a.add_row;
  kp.ld_add = a.ld_add;
  kp.relu = a.relu;
  kp.t = a.t;
  kp.ldt = a.ldt;
  kp.H = a.H;
  kp.Fh = a.Fh;
  kp.slope = a.slope;
  kp.kb = a.kb;
  kp.ldk = a.ldk;
  kp.Wa = a.Wa;
  kp.FW = slot_width(mode, a.F, a.H);
  kp.nmeta = att_meta(mode, a.F, a.H);
  kp.deterministic = a.deterministic;
  kp.accum = a.accum;
  kp.trace = g_trace;
  const WsLayout L = ws_layout(p, mode, a.F, a.H);
  char *w = reinterpret_cast<char *>(ws);
  kp.ws_unit = reinterpret_cast<int32_t *>(w + L.unit);
  kp.n_unit_ctr = max_chunks(a.F);
  kp.ws_cnt = reinterpret_cast<int32_t *>(w + L.cnt);
  kp.ws_acc = reinterpret_cast<float *>(w + L.acc);
  kp.ws_part = reinterpret_cast<float *>(w + L.part);
  kp.ws_rowmax = reinterpret_cast<float *>(w + L.rowmax);
  Mapping m = choose_mapping(p, a, is_att(mode) ? a.Fh : 0);
  if (m.vec == 0) {
    set_error("no supported lane mapping for this width / head size (GaAN, Gene: Fh/vec must be a power of 2 <= 32)");
    return GNN_ERR_UNSUPPORTED;
  }
  const int threads = 256;
  cudaError_t e = cudaSuccess;
  uint32_t *smax = reinterpret_cast<uint32_t *>(w + L.smax);
  kp.smax = smax;
  if (mode == M_GAT || mode == M_SYM) e = launch_score_max(a.X + a.F, a.ldx, p->n_src, a.H, 1, smax, s);
  if (e == cudaSuccess && mode == M_SYM) e = launch_score_max(a.X + a.F + a.H, a.ldx, p->n_src, a.H, 1, smax + a.H, s);
  if (e == cudaSuccess && mode == M_GAAN) e = launch_score_max(a.X + a.F, a.ldx, p->n_src, a.H, a.Fh, smax, s);
  if (e != cudaSuccess) return cuda_status(e, "score max launch");
  if (!kp.deterministic && is_att(mode)) {
    // atomic variant for GAT only, when no head straddles a feature chunk (the
    // l of a head is added by the chunk holding it); otherwise the
    // deterministic merge.  The register kernel computes the rowmax chains.
    const int cw = m.vec * m.lanes * m.nv;
    if (mode != M_GAT || !(cw >= a.F || cw % a.Fh == 0)) {
      kp.deterministic = 1;
    } else {
      m.cp = 0;
      if (p->n_multi > 0) {
        e = launch_row_score_max(kp, s);
        if (e != cudaSuccess) return cuda_status(e, "row score max launch");
      }
    }
  }
  // hot source rows resident in L2 for the duration of the launch (cache hints only)
  const int32_t rb = 4 * (a.F + (mode == M_GAT ? a.H : 0));
  const int32_t npin = hot_rows_for(p, rb);
  const int pin_grid = std::max(1, std::min(num_sms() * 8, (npin + 7) / 8));
  if (npin > 0) {
    k_l2_pin<true><<<pin_grid, 256, 0, s>>>(p->d_hot, npin, reinterpret_cast<const char *>(a.X), 4 * a.ldx, rb);
    count_launch();
  }
  const gnn_status st = launch_aggregate_kernel(p, kp, m, mode, threads, s);
  if (npin > 0) {
    k_l2_pin<false><<<pin_grid, 256, 0, s>>>(p->d_hot, npin, reinterpret_cast<const char *>(a.X), 4 * a.ldx, rb);
    count_launch();
  }
  return st;
}

static gnn_status launch_aggregate_kernel(const gnn_plan_s *p, KParams &kp, Mapping m, int mode, int threads,
                                          cudaStream_t s) {
  cudaError_t e = cudaSuccess;
  if (m.cp == 2) {  // gather4 streaming kernel (k_agg_g4.cu)
    KParams kq = kp;
    kq.n_unit_ctr = kp.n_unit_ctr;
    if (g4_admissible(kq, (int32_t)p->n_src)) {
      e = launch_g4(kq, (int32_t)p->n_src, s);
      if (e != cudaErrorNotSupported) return cuda_status(e, "aggregate launch (gather4)");
      (void)cudaGetLastError();
    }
    m.cp = 1;  // the cp.async chain with the same (4, 32, NV) mapping
    if (mode == M_GAT) m.cp = 0;
  }
  switch (mode) {
    case M_SUM:
    case M_MEAN: e = dispatch_sum(kp, m, threads, s); break;
    case M_MAX: e = dispatch_max(kp, m, threads, s); break;
    case M_GAT: e = dispatch_gat(kp, m, threads, s); break;
    default: e = dispatch_att(kp, m, threads, s); break;
  }
  return cuda_status(e, "aggregate launch");
}

// ---------------------------------------------------------------------------
// small weight-preparation kernels (run once per layer call, O(f_in * H*Fh))
// ---------------------------------------------------------------------------
// Wext[:, 0:HF] = W; Wext[:, HF + h] = W_h . a_src_h; Wext[:, HF + H + h] = W_h . a_dst_h
__global__ void k_gat_weights(const float *W, const float *a_src, const float *a_dst, int32_t f_in,
                              int32_t H, int32_t Fh, float *Wext, int32_t ldwe) {
  const int32_t HF = H * Fh;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (int64_t)f_in * ldwe;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = (int32_t)(i / ldwe), c = (int32_t)(i % ldwe);
    float v = 0.0f;
    if (c < HF) {
      v = W[(int64_t)r * HF + c];
    } else if (c < HF + 2 * H) {
      const int32_t h = (c - HF) % H;
      const float *a = (c < HF + H) ? a_src : a_dst;
      for (int32_t f = 0; f < Fh; ++f) v = fmaf(W[(int64_t)r * HF + h * Fh + f], a[h * Fh + f], v);
    }
    Wext[i] = v;
  }
}

cudaError_t launch_gat_weights(const float *W, const float *a_src, const float *a_dst, int32_t f_in,
                               int32_t H, int32_t Fh, float *Wext, int32_t ldwe, cudaStream_t s) {
  const int64_t tot = (int64_t)f_in * ldwe;
  const int blocks = (int)std::max<int64_t>(1, std::min<int64_t>((tot + 255) / 256, 1024));
  k_gat_weights<<<blocks, 256, 0, s>>>(W, a_src, a_dst, f_in, H, Fh, Wext, ldwe);
  count_launch();
  return cudaGetLastError();
}

// Wpq [f_in, 2 f_out]: column o < f_out = theta[o, :], column f_out + o = (phi - theta)[o, :];
// bpq [2 f_out] = [0 | b]
__global__ void k_edgeconv_weights(const float *theta, const float *phi, const float *bias,
                                   int32_t f_in, int32_t f_out, float *Wpq, float *bpq) {
  const int32_t ld = 2 * f_out;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < (int64_t)f_in * ld;
       i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t r = (int32_t)(i / ld), c = (int32_t)(i % ld);
    Wpq[i] = c < f_out ? theta[(int64_t)c * f_in + r]
                       : phi[(int64_t)(c - f_out) * f_in + r] - theta[(int64_t)(c - f_out) * f_in + r];
  }
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < ld;
       i += (int64_t)gridDim.x * blockDim.x)
    bpq[i] = (i < f_out || bias == nullptr) ? 0.0f : bias[i - f_out];
}

cudaError_t launch_edgeconv_weights(const float *theta, const float *phi, const float *bias,
                                    int32_t f_in, int32_t f_out, float *Wpq, float *bpq,
                                    cudaStream_t s) {
  const int64_t tot = (int64_t)f_in * 2 * f_out;
  const int blocks = (int)std::max<int64_t>(1, std::min<int64_t>((tot + 255) / 256, 1024));
  k_edgeconv_weights<<<blocks, 256, 0, s>>>(theta, phi, bias, f_in, f_out, Wpq, bpq);
  count_launch();
  return cudaGetLastError();
}

}  // namespace gnn
