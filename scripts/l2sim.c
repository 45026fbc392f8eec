/* dev tool: LRU simulation of the gather stream of an aggregation in a given
 * task order (rows in perm order, each row's sources in CSR order).  Returns
 * the number of misses for a cache of `cap` rows.  Approximates the L2 at row
 * granularity with the in-flight window folded into sequential order. */
#include <stdint.h>
#include <stdlib.h>
int64_t lru_misses(int64_t n, const int64_t *rowptr, const int32_t *colidx, const int32_t *perm, int64_t cap) {
  int32_t *prev = malloc(sizeof(int32_t) * n), *next = malloc(sizeof(int32_t) * n);
  char *in = calloc(n, 1);
  int32_t head = -1, tail = -1; /* head = most recent */
  int64_t size = 0, misses = 0;
  for (int64_t i = 0; i < n; ++i) {
    int64_t v = perm ? perm[i] : i;
    for (int64_t k = rowptr[v]; k < rowptr[v + 1]; ++k) {
      int32_t u = colidx[k];
      if (in[u]) {
        if (head == u) continue;
        /* unlink */
        if (prev[u] >= 0) next[prev[u]] = next[u];
        if (next[u] >= 0) prev[next[u]] = prev[u];
        if (tail == u) tail = prev[u];
      } else {
        ++misses;
        in[u] = 1;
        ++size;
        if (size > cap) { /* evict tail */
          int32_t t = tail;
          tail = prev[t];
          if (tail >= 0) next[tail] = -1;
          in[t] = 0;
          --size;
          if (head == t) head = -1;
        }
      }
      prev[u] = -1;
      next[u] = head;
      if (head >= 0) prev[head] = u;
      head = u;
      if (tail < 0) tail = u;
    }
  }
  free(prev); free(next); free(in);
  return misses;
}

/* BFS order of clusters over a symmetric CSR adjacency (clusters 0..C-1);
 * starts in `start_order`, neighbours in adjacency order. */
void bfs_order(int64_t C, const int64_t *adj_ptr, const int32_t *adj, const int32_t *start_order, int32_t *out) {
  char *vis = calloc(C, 1);
  int64_t head = 0, tail = 0;
  for (int64_t s = 0; s < C; ++s) {
    int32_t r = start_order[s];
    if (vis[r]) continue;
    vis[r] = 1;
    out[tail++] = r;
    while (head < tail) {
      int32_t c = out[head++];
      for (int64_t k = adj_ptr[c]; k < adj_ptr[c + 1]; ++k) {
        int32_t d = adj[k];
        if (!vis[d]) { vis[d] = 1; out[tail++] = d; }
      }
    }
  }
  free(vis);
}
