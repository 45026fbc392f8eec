// plan_io.cpp — plan save / load (libgnn.so).  The paper runs LAS once,
// offline, and reuses the schedule across runs because the graph structure
// does not change ("the graph structure ... is invariant", LAS
// costs ~600 GCN iterations).  A saved plan holds the CSR, the source
// out-degrees behind the GCN normalisers, the LAS task order and (optionally)
// the LAS intermediates; loading it rebuilds the device plan with the saved
// order (gnn_plan_create_perm) and never reruns MinHash / LSH / merging.
//
// File layout (little-endian, 8-byte aligned sections):
//   "GNNPLAN1" | u32 version (1) | u32 flags (bit 0: LAS intermediates)
//   | gnn_plan_opts | i64 n, n_src, nnz, n_clusters, n_pairs
//   | rowptr i64[n+1] | colidx i32[nnz] | d_out i32[n_src] | perm i32[n]
//   | [cluster_of i32[n] | sig u64[n*K] | pairs i32[2*n_pairs]]   (flag bit 0)
//   | u64 FNV-1a of every preceding byte
#include <climits>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "gnn_internal.h"

namespace gnn {
namespace {

constexpr char kMagic[8] = {'G', 'N', 'N', 'P', 'L', 'A', 'N', '1'};
constexpr uint32_t kVersion = 1;

struct Hash {
  uint64_t h = 1469598103934665603ULL;
  void add(const void *p, size_t n) {
    const uint8_t *b = (const uint8_t *)p;
    for (size_t i = 0; i < n; ++i) h = (h ^ b[i]) * 1099511628211ULL;
  }
};

struct Writer {
  FILE *f;
  Hash h;
  bool ok = true;
  void put(const void *p, size_t n) {
    if (!ok || n == 0) return;
    h.add(p, n);
    ok = fwrite(p, 1, n, f) == n;
  }
  template <typename T>
  void val(T v) { put(&v, sizeof(T)); }
};

struct Reader {
  FILE *f;
  Hash h;
  bool ok = true;
  void get(void *p, size_t n) {
    if (!ok || n == 0) return;
    ok = fread(p, 1, n, f) == n;
    if (ok) h.add(p, n);
  }
  template <typename T>
  T val() {
    T v{};
    get(&v, sizeof(T));
    return v;
  }
};

}  // namespace
}  // namespace gnn

using namespace gnn;

extern "C" {

gnn_status gnn_plan_save(gnn_plan_t p, const char *path, int32_t with_las) {
  try {
    if (!p || !path) {
      set_error("plan/path is NULL");
      return GNN_ERR_INVALID_ARG;
    }
    int cur = 0;
    cudaGetDevice(&cur);
    cudaSetDevice(p->device);
    std::vector<int32_t> col((size_t)p->nnz), dout((size_t)p->n_src);
    cudaError_t e = cudaSuccess;
    if (p->nnz > 0) e = cudaMemcpy(col.data(), p->dg.colidx, sizeof(int32_t) * col.size(), cudaMemcpyDeviceToHost);
    if (e == cudaSuccess && p->n_src > 0)
      e = cudaMemcpy(dout.data(), p->d_dout, sizeof(int32_t) * dout.size(), cudaMemcpyDeviceToHost);
    cudaSetDevice(cur);
    if (e != cudaSuccess) return cuda_status(e, "plan save: download");
    const bool las = with_las && p->opts.reorder && !p->sig.empty();
    FILE *f = fopen(path, "wb");
    if (!f) {
      set_error(std::string("plan save: cannot open ") + path);
      return GNN_ERR_INVALID_ARG;
    }
    Writer w{f};
    w.put(kMagic, 8);
    w.val<uint32_t>(kVersion);
    w.val<uint32_t>(las ? 1u : 0u);
    w.put(&p->opts, sizeof(gnn_plan_opts));
    w.val<int64_t>(p->n);
    w.val<int64_t>(p->n_src);
    w.val<int64_t>(p->nnz);
    w.val<int64_t>(p->n_clusters);
    w.val<int64_t>(las ? (int64_t)(p->pairs.size() / 2) : 0);
    w.put(p->rowptr.data(), sizeof(int64_t) * p->rowptr.size());
    w.put(col.data(), sizeof(int32_t) * col.size());
    w.put(dout.data(), sizeof(int32_t) * dout.size());
    w.put(p->perm.data(), sizeof(int32_t) * p->perm.size());
    if (las) {
      w.put(p->cluster_of.data(), sizeof(int32_t) * p->cluster_of.size());
      w.put(p->sig.data(), sizeof(uint64_t) * p->sig.size());
      w.put(p->pairs.data(), sizeof(int32_t) * p->pairs.size());
    }
    const uint64_t digest = w.h.h;
    const bool ok = w.ok && fwrite(&digest, 1, 8, f) == 8;
    if (fclose(f) != 0 || !ok) {
      set_error(std::string("plan save: write failed: ") + path);
      return GNN_ERR_INTERNAL;
    }
    return GNN_OK;
  } catch (const std::bad_alloc &) {
    set_error("host allocation failed");
    return GNN_ERR_NOMEM;
  } catch (...) {
    set_error("internal: plan save");
    return GNN_ERR_INTERNAL;
  }
}

gnn_status gnn_plan_load(const char *path, gnn_plan_t *out) {
  try {
    if (!path || !out) {
      set_error("path/out is NULL");
      return GNN_ERR_INVALID_ARG;
    }
    *out = nullptr;
    FILE *f = fopen(path, "rb");
    if (!f) {
      set_error(std::string("plan load: cannot open ") + path);
      return GNN_ERR_INVALID_ARG;
    }
    Reader r{f};
    auto bad = [&](const char *why) {
      fclose(f);
      set_error(std::string("plan load: ") + why + ": " + path);
      return GNN_ERR_INVALID_ARG;
    };
    char magic[8];
    r.get(magic, 8);
    if (!r.ok || memcmp(magic, kMagic, 8) != 0) return bad("not a gnn plan file");
    const uint32_t ver = r.val<uint32_t>(), flags = r.val<uint32_t>();
    if (ver != kVersion) return bad("unsupported version");
    gnn_plan_opts opts;
    r.get(&opts, sizeof(opts));
    if (opts.struct_size != sizeof(gnn_plan_opts)) return bad("options struct mismatch");
    const int64_t n = r.val<int64_t>(), n_src = r.val<int64_t>(), nnz = r.val<int64_t>();
    const int64_t n_clusters = r.val<int64_t>(), n_pairs = r.val<int64_t>();
    if (!r.ok || n < 0 || n_src < 0 || nnz < 0 || nnz >= INT32_MAX || n >= INT32_MAX || n_src >= INT32_MAX ||
        n_pairs < 0)
      return bad("corrupt header");
    std::vector<int64_t> rowptr((size_t)n + 1);
    std::vector<int32_t> col((size_t)nnz), dout((size_t)n_src), perm((size_t)n), cl;
    std::vector<uint64_t> sig;
    std::vector<int32_t> pairs;
    r.get(rowptr.data(), sizeof(int64_t) * rowptr.size());
    r.get(col.data(), sizeof(int32_t) * col.size());
    r.get(dout.data(), sizeof(int32_t) * dout.size());
    r.get(perm.data(), sizeof(int32_t) * perm.size());
    if (flags & 1u) {
      const int64_t K = opts.minhash_k;
      if (K < 1 || K > 64) return bad("corrupt LAS section");
      cl.resize((size_t)n);
      sig.resize((size_t)n * (size_t)K);
      pairs.resize((size_t)n_pairs * 2);
      r.get(cl.data(), sizeof(int32_t) * cl.size());
      r.get(sig.data(), sizeof(uint64_t) * sig.size());
      r.get(pairs.data(), sizeof(int32_t) * pairs.size());
    }
    const uint64_t want = r.h.h;
    uint64_t digest = 0;
    const bool got = fread(&digest, 1, 8, f) == 8;
    if (!r.ok || !got) return bad("truncated file");
    if (digest != want) return bad("checksum mismatch");
    fclose(f);
    gnn_plan_t p = nullptr;
    gnn_status st = create_plan(n, n_src, nnz, rowptr.data(), col.data(), dout.data(), perm.data(), &opts, &p);
    if (st != GNN_OK) return st;
    p->n_clusters = n_clusters;
    p->info.n_clusters = n_clusters;
    if (flags & 1u) {
      p->sig.swap(sig);
      p->pairs.swap(pairs);
      p->cluster_of.swap(cl);
      p->info.n_pairs = n_pairs;
    } else {
      p->opts.reorder = opts.reorder;
    }
    *out = p;
    return GNN_OK;
  } catch (const std::bad_alloc &) {
    set_error("host allocation failed");
    return GNN_ERR_NOMEM;
  } catch (...) {
    set_error("internal: plan load");
    return GNN_ERR_INTERNAL;
  }
}

}  // extern "C"
