// plan.cpp — host side of the planner (libgnn.so):
//   a2 steps 2-5 of locality-aware task scheduling (LSH banding, candidate
//      pairs, similarity, capped pair merging, cluster schedule);
//   a3 neighbor grouping and CTA work tiles (reading R8).
// MinHash signatures (a2 step 1) come from the GPU kernel in k_graph.cu.
// This is an independent implementation of the same integer specification
// the oracle follows (R7/R8): results must be bit-identical.
#include <algorithm>
#include <cstring>
#include <chrono>
#include <cstring>
#include <queue>
#include <thread>
#include <vector>

#include "gnn_internal.h"

namespace gnn {

namespace {

struct BandKey {
  uint64_t b0, b1;  // band tuple (r <= 2 handled directly; r > 2 hashed into rank order below)
  uint32_t rank;    // position of the node in (full signature, id) order
  uint32_t id;
  bool operator<(const BandKey &o) const {
    if (b0 != o.b0) return b0 < o.b0;
    if (b1 != o.b1) return b1 < o.b1;
    return rank < o.rank;
  }
};

}  // namespace

// LSH banding: for band j, non-empty nodes ordered by (band
// tuple, full signature, id); buckets = runs of equal band tuple; candidate
// pairs (m_i, m_{i+d}), 1 <= d <= W.  Union over bands, dedup, sorted.
int64_t las_lsh_pairs(int64_t n, const int64_t *rowptr, const uint64_t *sig, int32_t K, int32_t r,
                      int32_t W, std::vector<int32_t> &pairs) {
  const int32_t nb = K / r;
  std::vector<uint32_t> nodes;
  nodes.reserve((size_t)n);
  for (int64_t v = 0; v < n; ++v)
    if (rowptr[v + 1] > rowptr[v]) nodes.push_back((uint32_t)v);
  // rank by (full signature, id)
  std::vector<uint32_t> order(nodes);
  std::sort(order.begin(), order.end(), [&](uint32_t a, uint32_t b) {
    const uint64_t *sa = sig + (size_t)a * K, *sb = sig + (size_t)b * K;
    for (int32_t k = 0; k < K; ++k)
      if (sa[k] != sb[k]) return sa[k] < sb[k];
    return a < b;
  });
  std::vector<uint32_t> rank((size_t)n, 0);
  for (size_t i = 0; i < order.size(); ++i) rank[order[i]] = (uint32_t)i;

  const unsigned nthreads = std::max(1u, std::min(8u, std::thread::hardware_concurrency()));
  std::vector<std::vector<uint64_t>> local(nthreads);
  auto work = [&](unsigned tid) {
    std::vector<BandKey> keys(nodes.size());
    std::vector<uint64_t> &out = local[tid];
    for (int32_t j = (int32_t)tid; j < nb; j += (int32_t)nthreads) {
      for (size_t i = 0; i < nodes.size(); ++i) {
        const uint32_t v = nodes[i];
        const uint64_t *s = sig + (size_t)v * K + (size_t)j * r;
        BandKey bk;
        bk.b0 = s[0];
        bk.b1 = r > 1 ? s[1] : 0;
        bk.rank = rank[v];
        bk.id = v;
        keys[i] = bk;
      }
      std::sort(keys.begin(), keys.end());
      auto same_band = [&](const BandKey &x, const BandKey &y) {
        if (x.b0 != y.b0 || x.b1 != y.b1) return false;
        for (int32_t q = 2; q < r; ++q)
          if (sig[(size_t)x.id * K + (size_t)j * r + q] != sig[(size_t)y.id * K + (size_t)j * r + q])
            return false;
        return true;
      };
      size_t s0 = 0;
      while (s0 < keys.size()) {
        size_t e = s0 + 1;
        while (e < keys.size() && same_band(keys[s0], keys[e])) ++e;
        for (size_t i = s0; i < e; ++i)
          for (int32_t d = 1; d <= W && i + (size_t)d < e; ++d) {
            uint32_t a = keys[i].id, b = keys[i + d].id;
            if (a > b) std::swap(a, b);
            out.push_back(((uint64_t)a << 32) | b);
          }
        s0 = e;
      }
    }
  };
  if (r > 2) {
    // band tuples longer than 2: fall back to an exact comparator on the tuple
    // (rank order still breaks ties), single-threaded
    for (int32_t j = 0; j < nb; ++j) {
      std::vector<uint32_t> ord(nodes);
      std::sort(ord.begin(), ord.end(), [&](uint32_t a, uint32_t b) {
        const uint64_t *sa = sig + (size_t)a * K + (size_t)j * r, *sb = sig + (size_t)b * K + (size_t)j * r;
        for (int32_t q = 0; q < r; ++q)
          if (sa[q] != sb[q]) return sa[q] < sb[q];
        return rank[a] < rank[b];
      });
      auto eq = [&](uint32_t a, uint32_t b) {
        return std::memcmp(sig + (size_t)a * K + (size_t)j * r, sig + (size_t)b * K + (size_t)j * r,
                           sizeof(uint64_t) * r) == 0;
      };
      size_t s0 = 0;
      while (s0 < ord.size()) {
        size_t e = s0 + 1;
        while (e < ord.size() && eq(ord[s0], ord[e])) ++e;
        for (size_t i = s0; i < e; ++i)
          for (int32_t d = 1; d <= W && i + (size_t)d < e; ++d) {
            uint32_t a = ord[i], b = ord[i + d];
            if (a > b) std::swap(a, b);
            local[0].push_back(((uint64_t)a << 32) | b);
          }
        s0 = e;
      }
    }
  } else {
    std::vector<std::thread> th;
    for (unsigned t = 0; t < nthreads; ++t) th.emplace_back(work, t);
    for (auto &t : th) t.join();
  }
  size_t tot = 0;
  for (auto &l : local) tot += l.size();
  std::vector<uint64_t> all;
  all.reserve(tot);
  for (auto &l : local) {
    all.insert(all.end(), l.begin(), l.end());
    std::vector<uint64_t>().swap(l);
  }
  std::sort(all.begin(), all.end());
  all.erase(std::unique(all.begin(), all.end()), all.end());
  pairs.resize(all.size() * 2);
  for (size_t i = 0; i < all.size(); ++i) {
    pairs[2 * i] = (int32_t)(all[i] >> 32);
    pairs[2 * i + 1] = (int32_t)(all[i] & 0xffffffffu);
  }
  return (int64_t)all.size();
}

namespace {
struct HEnt {
  int32_t sim, a, b;
};
struct HCmp {  // priority_queue pops the "largest": sim desc, a asc, b asc
  bool operator()(const HEnt &x, const HEnt &y) const {
    if (x.sim != y.sim) return x.sim < y.sim;
    if (x.a != y.a) return x.a > y.a;
    return x.b > y.b;
  }
};
inline int32_t sim_of(const uint64_t *sig, int32_t K, int64_t a, int64_t b) {
  const uint64_t *sa = sig + (size_t)a * K, *sb = sig + (size_t)b * K;
  int32_t s = 0;
  for (int32_t k = 0; k < K; ++k) s += sa[k] == sb[k];
  return s;
}
}  // namespace

// Pair merging and task scheduling; spec R7.
int64_t las_merge(int64_t n, const uint64_t *sig, int32_t K, const std::vector<int32_t> &pairs,
                  int32_t cap, int32_t min_sim, int32_t cluster_order, std::vector<int32_t> &perm,
                  std::vector<int32_t> &cluster_of) {
  std::vector<int32_t> parent((size_t)n), size((size_t)n, 1);
  for (int64_t v = 0; v < n; ++v) parent[v] = (int32_t)v;
  auto find = [&](int64_t x) {
    int64_t r = x;
    while (parent[r] != r) r = parent[r];
    while (parent[x] != r) {
      int64_t nx = parent[x];
      parent[x] = (int32_t)r;
      x = nx;
    }
    return r;
  };
  const size_t np = pairs.size() / 2;
  std::vector<HEnt> init(np);
  for (size_t i = 0; i < np; ++i)
    init[i] = HEnt{sim_of(sig, K, pairs[2 * i], pairs[2 * i + 1]), pairs[2 * i], pairs[2 * i + 1]};
  std::priority_queue<HEnt, std::vector<HEnt>, HCmp> pq(HCmp(), std::move(init));
  while (!pq.empty()) {
    const HEnt e = pq.top();
    pq.pop();
    if (parent[e.a] == e.a && parent[e.b] == e.b) {
      if (size[e.a] + size[e.b] <= cap) {
        int32_t keep = (size[e.a] != size[e.b]) ? (size[e.a] > size[e.b] ? e.a : e.b) : std::min(e.a, e.b);
        int32_t gone = keep == e.a ? e.b : e.a;
        parent[gone] = keep;
        size[keep] += size[gone];
      }
    } else {
      const int64_t ra = find(e.a), rb = find(e.b);
      if (ra != rb && size[ra] + size[rb] <= cap) {
        const int32_t s = sim_of(sig, K, ra, rb);
        if (s >= min_sim) pq.push(HEnt{s, (int32_t)std::min(ra, rb), (int32_t)std::max(ra, rb)});
      }
    }
  }
  // schedule (R7): clusters ordered by (representative signature,
  // smallest member) when cluster_order == 1, by smallest member when 0;
  // members ascending
  std::vector<int64_t> cnt((size_t)n, 0), off((size_t)n, -1);
  std::vector<std::pair<int64_t, int64_t>> cl;  // (representative, smallest member)
  for (int64_t v = 0; v < n; ++v) {
    const int64_t r = find(v);
    if (cnt[r]++ == 0) cl.emplace_back(r, v);
  }
  if (cluster_order == 1) {
    std::sort(cl.begin(), cl.end(), [&](const std::pair<int64_t, int64_t> &x, const std::pair<int64_t, int64_t> &y) {
      const uint64_t *sa = sig + (size_t)x.first * K, *sb = sig + (size_t)y.first * K;
      for (int32_t k = 0; k < K; ++k)
        if (sa[k] != sb[k]) return sa[k] < sb[k];
      return x.second < y.second;
    });
  }
  int64_t pos = 0;
  for (const auto &c : cl) {
    off[c.first] = pos;
    pos += cnt[c.first];
  }
  perm.assign((size_t)n, 0);
  cluster_of.assign((size_t)n, 0);
  for (int64_t v = 0; v < n; ++v) {
    const int64_t r = find(v);
    perm[off[r]++] = (int32_t)v;
    cluster_of[v] = (int32_t)r;
  }
  const int64_t nc = (int64_t)cl.size();
  return nc;
}

// a3: neighbor groups in task order (reading R8).  Pure host
// function (also gnn_groups_host).
void schedule_host(int64_t n, const int64_t *rowptr, const int32_t *perm, int64_t ng,
                   std::vector<int32_t> &grp_row, std::vector<int64_t> &grp_beg) {
  grp_row.clear();
  grp_beg.clear();
  for (int64_t i = 0; i < n; ++i) {
    const int64_t v = perm ? perm[i] : i;
    const int64_t beg = rowptr[v], end = rowptr[v + 1];
    for (int64_t b = beg; b < end; b += ng) {
      grp_row.push_back((int32_t)v);
      grp_beg.push_back(b);
      if (end - b <= ng) break;
    }
  }
}

// Work units in task order = neighbour groups: a row with one
// group is one unit; the groups of a longer row are separate units whose
// partials meet in the workspace.  Source indices are re-laid out in task order
// (colidx_t) so every unit reads one contiguous stream.
gnn_status build_schedule(gnn_plan_s *p) {
  const int64_t n = p->n, ng = p->ng;
  schedule_host(n, p->rowptr.data(), p->perm.data(), ng, p->grp_row, p->grp_beg);
  std::vector<int32_t> desc, colidx_t((size_t)p->nnz + 16, 0), multi_slot, multi_units, multi_row, empty;
  desc.reserve((size_t)p->grp_row.size() * 4 + 4);
  int64_t tpos = 0, slots = 0;
  for (int64_t i = 0; i < n; ++i) {
    const int64_t v = p->perm[i];
    const int64_t rb = p->rowptr[v], re = p->rowptr[v + 1];
    if (re == rb) continue;
    std::memcpy(colidx_t.data() + tpos, p->colidx_h + rb, sizeof(int32_t) * (size_t)(re - rb));
    const int64_t ngrp = (re - rb + ng - 1) / ng;
    int32_t m = -1;
    if (ngrp > 1) {
      m = (int32_t)multi_slot.size();
      multi_slot.push_back((int32_t)slots);
      multi_units.push_back((int32_t)ngrp);
      multi_row.push_back((int32_t)v);
      slots += ngrp;
    }
    for (int64_t b = rb; b < re; b += ng) desc.insert(desc.end(), {(int32_t)(tpos + (b - rb)), (int32_t)b, (int32_t)v, m});
    tpos += re - rb;
  }
  const int64_t n_units = (int64_t)desc.size() / 4;
  desc.insert(desc.end(), {(int32_t)tpos, 0, 0, -1});
  for (int64_t v = 0; v < n; ++v)
    if (p->rowptr[v + 1] == p->rowptr[v]) empty.push_back((int32_t)v);
  p->n_multi = (int64_t)multi_slot.size();
  p->multi_slots = slots;
  p->n_empty = (int64_t)empty.size();

  auto upload = [&](const void *src, size_t bytes, void **dst) -> cudaError_t {
    *dst = nullptr;
    cudaError_t e = cudaMalloc(dst, bytes > 0 ? bytes : 16);
    if (e != cudaSuccess) return e;
    p->sched_allocs.push_back(*dst);
    if (bytes > 0) e = cudaMemcpy(*dst, src, bytes, cudaMemcpyHostToDevice);
    return e;
  };
  void *d;
  cudaError_t e;
#define UP(vec, field)                                                                 \
  e = upload((vec).data(), sizeof(int32_t) * (vec).size(), &d);                       \
  if (e != cudaSuccess) return cuda_status(e, "plan upload");                         \
  p->dg.field = reinterpret_cast<decltype(p->dg.field)>(d);
  UP(desc, unit_desc)
  UP(colidx_t, colidx_t)
  UP(multi_slot, multi_slot)
  UP(multi_units, multi_units)
  UP(multi_row, multi_row)
  UP(empty, empty_rows)
  UP(p->perm, perm)
#undef UP
  p->dg.n_units = (int32_t)n_units;
  p->dg.n_multi = (int32_t)p->n_multi;
  p->dg.n_empty = (int32_t)p->n_empty;
  p->dg.ng = (int32_t)ng;
  p->info.n_groups = (int64_t)p->grp_row.size();
  p->info.n_tiles = n_units;  // work units (one per neighbour group)
  p->info.n_split_rows = p->n_multi;
  p->info.n_empty_rows = p->n_empty;
  return GNN_OK;
}

// NG bound (R8): largest multiple of 16 <= 10 * average degree,
// clamped to [16, 4096]
int64_t default_group_size(int64_t n, int64_t nnz) {
  const double avg = n > 0 ? (double)nnz / (double)n : 0.0;
  int64_t ng = (int64_t)(std::min(4096.0, 10.0 * avg) / 16.0) * 16;
  return ng < 16 ? 16 : ng;
}

// Rebuild the NG schedule (work units, task-ordered index stream) of an
// existing plan for another group bound; the LAS schedule (perm) is kept.
// Synchronous; the caller guarantees no call is in flight on the plan.
gnn_status rebuild_schedule(gnn_plan_s *p, int64_t group_size) {
  if (group_size < 0) group_size = default_group_size(p->n, p->nnz);
  int cur = 0;
  cudaGetDevice(&cur);
  cudaSetDevice(p->device);
  std::vector<int32_t> col((size_t)p->nnz);
  cudaError_t e = cudaSuccess;
  if (p->nnz > 0)
    e = cudaMemcpy(col.data(), p->dg.colidx, sizeof(int32_t) * (size_t)p->nnz, cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) {
    cudaSetDevice(cur);
    return cuda_status(e, "rebuild: colidx download");
  }
  for (void *d : p->sched_allocs) cudaFree(d);
  p->sched_allocs.clear();
  p->info.group_size = (int32_t)group_size;
  p->ng = group_size == 0 ? (1 << 30) : (int32_t)group_size;
  const auto t0 = std::chrono::steady_clock::now();
  p->colidx_h = col.data();
  gnn_status st = build_schedule(p);
  p->colidx_h = nullptr;
  p->info.ms_ng = std::chrono::duration<double, std::milli>(std::chrono::steady_clock::now() - t0).count();
  cudaSetDevice(cur);
  return st;
}

}  // namespace gnn
