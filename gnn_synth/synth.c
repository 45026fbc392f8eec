/*
 * gnn_synth/synth.c — seeded synthetic INPUT generators shared by the oracle
 * tests, the GPU parity tests and bench.py.
 *
 * This file holds none of the method's arithmetic (no aggregation, no
 * normalisation, no hashing of the planner): it only draws graphs.  Both the
 * oracle and the CUDA path consume the CSR bytes it produces.
 *
 * GEN-PL ("neighbor-template" power law), DESIGN.md §3:
 *   1. expected row lengths w_v ~ lognormal(mu, sigma) with
 *      sigma^2 = ln(1 + var/mean^2), mu = ln(mean) - sigma^2/2, clipped to
 *      `cap` and rescaled (Table 3 mean / max / variance);
 *   2. integer row lengths d_v by largest remainder so that sum d_v == nnz
 *      exactly, the heaviest row forced to `cap`;
 *   3. community g(v) = floor(v / comm) (pre-relabel) owns a template T_g of
 *      ceil(2*rho*mean_g) sources drawn proportional to w;
 *   4. row v takes min(round(rho*d_v), |T_g|) sources uniformly from T_g and the
 *      rest proportional to w (alias table), no self loops, no duplicates;
 *   5. a random relabel permutation is applied to row and column ids, rows are
 *      written in CSR order with sources sorted ascending.
 * The graph is directed (row v = in-neighbours of v); because sources are drawn
 * with the same weights that set the row lengths, out-degree follows in-degree
 * in expectation.
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct { uint64_t s; } rng_t;

static inline uint64_t rng_next(rng_t *r) {
  uint64_t z = (r->s += 0x9E3779B97F4A7C15ULL);
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}
static inline double rng_u01(rng_t *r) { return (double)(rng_next(r) >> 11) * 0x1.0p-53; }
static inline uint64_t rng_below(rng_t *r, uint64_t n) {
  /* Lemire-style multiply-shift; bias < n / 2^64, irrelevant here */
  return (uint64_t)(((__uint128_t)rng_next(r) * n) >> 64);
}
static double rng_normal(rng_t *r) {
  double u1 = rng_u01(r), u2 = rng_u01(r);
  if (u1 < 1e-300) u1 = 1e-300;
  return sqrt(-2.0 * log(u1)) * cos(6.283185307179586 * u2);
}

/* ---- alias table (Walker) for drawing ids proportional to w ---- */
typedef struct { int64_t n; double *prob; int64_t *alias; } alias_t;

static int alias_build(alias_t *a, const double *w, int64_t n) {
  a->n = n;
  a->prob = (double *)malloc(sizeof(double) * n);
  a->alias = (int64_t *)malloc(sizeof(int64_t) * n);
  int64_t *small = (int64_t *)malloc(sizeof(int64_t) * n);
  int64_t *large = (int64_t *)malloc(sizeof(int64_t) * n);
  if (!a->prob || !a->alias || !small || !large) return -1;
  double tot = 0;
  for (int64_t i = 0; i < n; ++i) tot += w[i];
  int64_t ns = 0, nl = 0;
  for (int64_t i = 0; i < n; ++i) {
    a->prob[i] = w[i] * (double)n / tot;
    a->alias[i] = i;
    if (a->prob[i] < 1.0) small[ns++] = i; else large[nl++] = i;
  }
  while (ns > 0 && nl > 0) {
    int64_t s = small[--ns], l = large[--nl];
    a->alias[s] = l;
    a->prob[l] = (a->prob[l] + a->prob[s]) - 1.0;
    if (a->prob[l] < 1.0) small[ns++] = l; else large[nl++] = l;
  }
  while (nl > 0) a->prob[large[--nl]] = 1.0;
  while (ns > 0) a->prob[small[--ns]] = 1.0;
  free(small);
  free(large);
  return 0;
}
static inline int64_t alias_draw(const alias_t *a, rng_t *r) {
  int64_t i = (int64_t)rng_below(r, (uint64_t)a->n);
  return rng_u01(r) < a->prob[i] ? i : a->alias[i];
}
static void alias_free(alias_t *a) { free(a->prob); free(a->alias); }

static int cmp_i64(const void *x, const void *y) {
  int64_t a = *(const int64_t *)x, b = *(const int64_t *)y;
  return (a > b) - (a < b);
}
static int cmp_i32(const void *x, const void *y) {
  int32_t a = *(const int32_t *)x, b = *(const int32_t *)y;
  return (a > b) - (a < b);
}

typedef struct { double frac; int64_t id; } frac_t;
static int cmp_frac_desc(const void *x, const void *y) {
  const frac_t *a = (const frac_t *)x, *b = (const frac_t *)y;
  if (a->frac != b->frac) return a->frac < b->frac ? 1 : -1;
  return (a->id > b->id) - (a->id < b->id);
}

/* small-array insertion sort + dedup helpers */
static int64_t sort_unique_i64(int64_t *v, int64_t k) {
  if (k <= 1) return k;
  if (k < 32) {
    for (int64_t i = 1; i < k; ++i) {
      int64_t x = v[i], j = i - 1;
      while (j >= 0 && v[j] > x) { v[j + 1] = v[j]; --j; }
      v[j + 1] = x;
    }
  } else {
    qsort(v, (size_t)k, sizeof(int64_t), cmp_i64);
  }
  int64_t m = 1;
  for (int64_t i = 1; i < k; ++i)
    if (v[i] != v[m - 1]) v[m++] = v[i];
  return m;
}

/*
 * Returns 0 on success.  rowptr[n+1] and colidx[nnz] are caller-allocated.
 * stats (may be NULL) receives {max_deg, mean*1e6, var*1e3, zero_rows}.
 */
int synth_powerlaw_ex(int64_t n, int64_t nnz, double mean, double var, int64_t cap,
                      int64_t comm, double rho, uint64_t seed, int64_t *rowptr,
                      int32_t *colidx, int64_t *stats, int64_t *relabel_out) {
  if (n <= 1 || nnz < 0 || cap < 1) return -1;
  if (cap > n - 1) cap = n - 1;
  if (nnz > n * cap) return -2;
  rng_t rng = {seed * 0x2545F4914F6CDD1DULL + 0x1234567ULL};
  double *w = (double *)malloc(sizeof(double) * n);
  int64_t *deg = (int64_t *)malloc(sizeof(int64_t) * n);
  if (!w || !deg) return -3;
  /* 1. lognormal weights, clipped to cap and rescaled to the target mean */
  double s2 = log(1.0 + var / (mean * mean));
  double sg = sqrt(s2), mu = log(mean) - 0.5 * s2;
  for (int64_t i = 0; i < n; ++i) w[i] = exp(mu + sg * rng_normal(&rng));
  double target_mean = (double)nnz / (double)n;
  int64_t imax = 0;
  for (int it = 0; it < 8; ++it) {
    double tot = 0;
    for (int64_t i = 0; i < n; ++i) tot += w[i];
    double sc = target_mean * n / tot;
    for (int64_t i = 0; i < n; ++i) {
      w[i] *= sc;
      if (w[i] > (double)cap) w[i] = (double)cap;
    }
  }
  for (int64_t i = 1; i < n; ++i) if (w[i] > w[imax]) imax = i;
  /* 2. integer row lengths by largest remainder, sum == nnz exactly */
  {
    double tot = 0;
    for (int64_t i = 0; i < n; ++i) tot += w[i];
    frac_t *fr = (frac_t *)malloc(sizeof(frac_t) * n);
    int64_t sum = 0;
    for (int64_t i = 0; i < n; ++i) {
      double x = w[i] * (double)nnz / tot;
      int64_t d = (int64_t)floor(x);
      if (d > cap) d = cap;
      deg[i] = d;
      sum += d;
      fr[i].frac = x - floor(x);
      fr[i].id = i;
    }
    sum -= deg[imax];
    deg[imax] = cap;
    sum += cap;
    qsort(fr, (size_t)n, sizeof(frac_t), cmp_frac_desc);
    int64_t guard = 0;
    while (sum != nnz && guard < 64) {
      for (int64_t j = 0; j < n && sum != nnz; ++j) {
        int64_t i = fr[j].id;
        if (i == imax) continue;
        if (sum < nnz && deg[i] < cap) { deg[i]++; sum++; }
        else if (sum > nnz && deg[i] > 0) { deg[i]--; sum--; }
      }
      ++guard;
    }
    free(fr);
    if (sum != nnz) { free(w); free(deg); return -4; }
  }
  alias_t al;
  if (alias_build(&al, w, n)) return -3;
  /* 3. community templates */
  int64_t ncomm = comm > 0 ? (n + comm - 1) / comm : 0;
  int64_t *tpl_off = NULL, *tpl = NULL;
  if (rho > 0 && ncomm > 0) {
    tpl_off = (int64_t *)calloc((size_t)ncomm + 1, sizeof(int64_t));
    for (int64_t g = 0; g < ncomm; ++g) {
      int64_t lo = g * comm, hi = lo + comm < n ? lo + comm : n;
      double md = 0;
      for (int64_t v = lo; v < hi; ++v) md += (double)deg[v];
      md /= (double)(hi - lo);
      int64_t ts = (int64_t)ceil(2.0 * rho * md);
      if (ts > n / 2) ts = n / 2;
      tpl_off[g + 1] = tpl_off[g] + ts;
    }
    tpl = (int64_t *)malloc(sizeof(int64_t) * (tpl_off[ncomm] + 1));
    int64_t *buf = NULL;
    int64_t bufcap = 0;
    for (int64_t g = 0; g < ncomm; ++g) {
      int64_t ts = tpl_off[g + 1] - tpl_off[g];
      if (bufcap < 2 * ts + 64) { bufcap = 2 * ts + 64; buf = (int64_t *)realloc(buf, sizeof(int64_t) * bufcap); }
      int64_t k = 0;
      while (k < ts) {
        int64_t need = ts - k;
        for (int64_t j = 0; j < need; ++j) buf[k + j] = alias_draw(&al, &rng);
        k = sort_unique_i64(buf, k + need);
      }
      memcpy(tpl + tpl_off[g], buf, sizeof(int64_t) * ts);
    }
    free(buf);
  }
  /* relabel permutation (Fisher-Yates) */
  int64_t *perm = (int64_t *)malloc(sizeof(int64_t) * n);
  for (int64_t i = 0; i < n; ++i) perm[i] = i;
  for (int64_t i = n - 1; i > 0; --i) {
    int64_t j = (int64_t)rng_below(&rng, (uint64_t)(i + 1));
    int64_t t = perm[i]; perm[i] = perm[j]; perm[j] = t;
  }
  /* rowptr in relabelled order */
  rowptr[0] = 0;
  {
    int64_t *dnew = (int64_t *)malloc(sizeof(int64_t) * n);
    for (int64_t v = 0; v < n; ++v) dnew[perm[v]] = deg[v];
    for (int64_t v = 0; v < n; ++v) rowptr[v + 1] = rowptr[v] + dnew[v];
    free(dnew);
  }
  /* 4. rows */
  int64_t maxd = 0;
  for (int64_t v = 0; v < n; ++v) if (deg[v] > maxd) maxd = deg[v];
  int64_t *row = (int64_t *)malloc(sizeof(int64_t) * (2 * maxd + 64));
  int64_t *tcopy = NULL;
  int64_t tcap = 0;
  for (int64_t v = 0; v < n; ++v) {
    int64_t d = deg[v];
    if (d == 0) continue;
    int64_t k = 0;
    if (tpl) {
      int64_t g = v / comm;
      int64_t ts = tpl_off[g + 1] - tpl_off[g];
      int64_t kt = (int64_t)llround(rho * (double)d);
      if (kt > ts) kt = ts;
      if (kt > 0) {
        if (tcap < ts) { tcap = ts; tcopy = (int64_t *)realloc(tcopy, sizeof(int64_t) * tcap); }
        memcpy(tcopy, tpl + tpl_off[g], sizeof(int64_t) * ts);
        for (int64_t j = 0; j < kt; ++j) { /* partial Fisher-Yates */
          int64_t r = j + (int64_t)rng_below(&rng, (uint64_t)(ts - j));
          int64_t t = tcopy[j]; tcopy[j] = tcopy[r]; tcopy[r] = t;
          if (tcopy[j] != v) row[k++] = tcopy[j];
        }
        k = sort_unique_i64(row, k);
      }
    }
    int64_t tries = 0;
    while (k < d) {
      int64_t need = d - k;
      int64_t m = k;
      for (int64_t j = 0; j < need; ++j) {
        int64_t u = (tries > 16) ? (int64_t)rng_below(&rng, (uint64_t)n) : alias_draw(&al, &rng);
        if (u != v) row[m++] = u;
      }
      k = sort_unique_i64(row, m);
      ++tries;
    }
    /* k == d now (never overshoots: at most `need` appended each round) */
    int64_t base = rowptr[perm[v]];
    for (int64_t j = 0; j < d; ++j) colidx[base + j] = (int32_t)perm[row[j]];
    qsort(colidx + base, (size_t)d, sizeof(int32_t), cmp_i32);
  }
  if (stats) {
    double m1 = (double)nnz / n, m2 = 0;
    int64_t zeros = 0;
    for (int64_t v = 0; v < n; ++v) {
      double dd = (double)deg[v] - m1;
      m2 += dd * dd;
      zeros += deg[v] == 0;
    }
    stats[0] = maxd;
    stats[1] = (int64_t)llround(m1 * 1e6);
    stats[2] = (int64_t)llround(m2 / n * 1e3);
    stats[3] = zeros;
  }
  if (relabel_out) memcpy(relabel_out, perm, sizeof(int64_t) * (size_t)n);
  free(row); free(tcopy); free(perm); free(tpl); free(tpl_off);
  alias_free(&al);
  free(w); free(deg);
  return 0;
}

int synth_powerlaw(int64_t n, int64_t nnz, double mean, double var, int64_t cap,
                   int64_t comm, double rho, uint64_t seed, int64_t *rowptr,
                   int32_t *colidx, int64_t *stats) {
  return synth_powerlaw_ex(n, nnz, mean, var, cap, comm, rho, seed, rowptr, colidx, stats, NULL);
}

/* LSD radix sort of uint64 keys (16-bit digits), tmp of the same size */
static void radix_u64(uint64_t *a, uint64_t *tmp, int64_t m, int bits) {
  int64_t *cnt = (int64_t *)malloc(sizeof(int64_t) * 65536);
  for (int sh = 0; sh < bits; sh += 16) {
    memset(cnt, 0, sizeof(int64_t) * 65536);
    for (int64_t i = 0; i < m; ++i) cnt[(a[i] >> sh) & 0xFFFF]++;
    int64_t s = 0;
    for (int d = 0; d < 65536; ++d) { int64_t c = cnt[d]; cnt[d] = s; s += c; }
    for (int64_t i = 0; i < m; ++i) tmp[cnt[(a[i] >> sh) & 0xFFFF]++] = a[i];
    memcpy(a, tmp, sizeof(uint64_t) * (size_t)m);
  }
  free(cnt);
}
static int64_t unique_u64(uint64_t *a, int64_t m) {
  if (m == 0) return 0;
  int64_t k = 1;
  for (int64_t i = 1; i < m; ++i)
    if (a[i] != a[k - 1]) a[k++] = a[i];
  return k;
}

/*
 * GEN-PL, undirected (SURVEY.md §8(d) steps 1-6 for C1/C3/C5): `nnz` CSR
 * entries = nnz/2 undirected pairs, symmetrised, no self loops, no duplicates.
 *   1. lognormal expected degrees w_v (mean nnz/n, Table 3 variance, clipped
 *      to cap, the heaviest at cap);
 *   2. community g(v) = floor(v / comm) owns a template of ceil(2*rho*mean_g)
 *      nodes drawn proportional to w;
 *   3. node v proposes about w_v / 2 partners: round(rho * that) uniformly
 *      from its template, the rest proportional to w (so its expected degree
 *      is ~w_v: its own proposals plus being proposed);
 *   4. pairs are canonicalised to (min, max) and deduplicated; top-up draws
 *      (v ~ w, partner as in 3) until there are nnz/2 pairs, random ones are
 *      dropped if over;
 *   5. degree floor 1: every isolated node is attached to a partner ~ w, and
 *      as many pairs whose endpoints both have degree >= 3 are removed;
 *   6. symmetrise, random relabel, CSR rows sorted by source id.
 */
int synth_powerlaw_sym(int64_t n, int64_t nnz, double mean, double var, int64_t cap, int64_t comm,
                       double rho, uint64_t seed, int64_t *rowptr, int32_t *colidx, int64_t *stats,
                       int64_t *relabel_out) {
  (void)mean;
  if (n <= 2 || nnz < 2 || (nnz & 1) || cap < 1) return -1;
  if (cap > n - 1) cap = n - 1;
  const int64_t P = nnz / 2;
  if (P > n * (n - 1) / 2) return -2;
  rng_t rng = {seed * 0x2545F4914F6CDD1DULL + 0x7654321ULL};
  double *w = (double *)malloc(sizeof(double) * n);
  if (!w) return -3;
  double s2 = log(1.0 + var / ((double)nnz / n * (double)nnz / n));
  double sg = sqrt(s2), mu = log((double)nnz / n) - 0.5 * s2;
  for (int64_t i = 0; i < n; ++i) w[i] = exp(mu + sg * rng_normal(&rng));
  const double target_mean = (double)nnz / (double)n;
  for (int it = 0; it < 8; ++it) {
    double tot = 0;
    for (int64_t i = 0; i < n; ++i) tot += w[i];
    double sc = target_mean * n / tot;
    for (int64_t i = 0; i < n; ++i) {
      w[i] *= sc;
      if (w[i] > (double)cap) w[i] = (double)cap;
    }
  }
  int64_t imax = 0;
  for (int64_t i = 1; i < n; ++i) if (w[i] > w[imax]) imax = i;
  w[imax] = (double)cap;
  alias_t al;
  if (alias_build(&al, w, n)) return -3;
  /* templates */
  int64_t ncomm = comm > 0 ? (n + comm - 1) / comm : 0;
  int64_t *tpl_off = NULL, *tpl = NULL;
  if (rho > 0 && ncomm > 0) {
    tpl_off = (int64_t *)calloc((size_t)ncomm + 1, sizeof(int64_t));
    for (int64_t g = 0; g < ncomm; ++g) {
      int64_t lo = g * comm, hi = lo + comm < n ? lo + comm : n;
      double md = 0;
      for (int64_t v = lo; v < hi; ++v) md += w[v];
      md /= (double)(hi - lo);
      int64_t ts = (int64_t)ceil(2.0 * rho * md);
      if (ts > n / 2) ts = n / 2;
      if (ts < 1) ts = 1;
      tpl_off[g + 1] = tpl_off[g] + ts;
    }
    tpl = (int64_t *)malloc(sizeof(int64_t) * (tpl_off[ncomm] + 1));
    int64_t *buf = NULL, bufcap = 0;
    for (int64_t g = 0; g < ncomm; ++g) {
      int64_t ts = tpl_off[g + 1] - tpl_off[g];
      if (bufcap < 2 * ts + 64) { bufcap = 2 * ts + 64; buf = (int64_t *)realloc(buf, sizeof(int64_t) * bufcap); }
      int64_t k = 0;
      while (k < ts) {
        int64_t need = ts - k;
        for (int64_t j = 0; j < need; ++j) buf[k + j] = alias_draw(&al, &rng);
        k = sort_unique_i64(buf, k + need);
      }
      memcpy(tpl + tpl_off[g], buf, sizeof(int64_t) * ts);
    }
    free(buf);
  }
  /* partner of v: from v's template with probability rho (when it has one), else ~ w */
  #define PARTNER(v)                                                                         \
    ((tpl && rng_u01(&rng) < rho)                                                            \
         ? tpl[tpl_off[(v) / comm] + (int64_t)rng_below(&rng, (uint64_t)(tpl_off[(v) / comm + 1] - tpl_off[(v) / comm]))] \
         : alias_draw(&al, &rng))
  /* 3. proposals: about w_v / 2 per node, by largest remainder so the total is P */
  int64_t cap_keys = P + P / 4 + 1024, m = 0;
  uint64_t *key = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)cap_keys);
  uint64_t *tmp = (uint64_t *)malloc(sizeof(uint64_t) * (size_t)cap_keys);
  if (!key || !tmp) return -3;
  {
    double tot = 0;
    for (int64_t i = 0; i < n; ++i) tot += w[i];
    double carry = 0;
    for (int64_t v = 0; v < n; ++v) {
      double x = w[v] * (double)P / tot + carry;
      int64_t h = (int64_t)floor(x);
      carry = x - (double)h;
      for (int64_t j = 0; j < h && m < cap_keys; ++j) {
        int64_t u = PARTNER(v);
        if (u == v) continue;
        int64_t a = v < u ? v : u, b = v < u ? u : v;
        key[m++] = (uint64_t)a * (uint64_t)n + (uint64_t)b;
      }
    }
  }
  int bits = 0;
  while (bits < 64 && ((uint64_t)1 << bits) <= (uint64_t)n * (uint64_t)n) bits += 16;
  radix_u64(key, tmp, m, bits);
  m = unique_u64(key, m);
  /* 4. top-up / trim to exactly P pairs */
  int guard = 0;
  double eff = 0.5;  /* fraction of top-up draws that survive dedup (updated per round) */
  while (m < P && guard++ < 64) {
    int64_t need = P - m, add = (int64_t)((double)need / eff * 1.1) + 64, m0 = m;
    if (m + add > cap_keys) {
      cap_keys = m + add + 1024;
      key = (uint64_t *)realloc(key, sizeof(uint64_t) * (size_t)cap_keys);
      tmp = (uint64_t *)realloc(tmp, sizeof(uint64_t) * (size_t)cap_keys);
    }
    for (int64_t j = 0; j < add; ++j) {
      int64_t v = alias_draw(&al, &rng), u = PARTNER(v);
      if (u == v) continue;
      int64_t a = v < u ? v : u, b = v < u ? u : v;
      key[m++] = (uint64_t)a * (uint64_t)n + (uint64_t)b;
    }
    const int64_t drawn = m - m0;
    radix_u64(key, tmp, m, bits);
    m = unique_u64(key, m);
    if (drawn > 0) eff = (double)(m - m0) / (double)drawn;
    if (eff < 0.05) eff = 0.05;
  }
  if (m < P) return -4;
  if (m > P) { /* drop random pairs: partial Fisher-Yates moves the dropped ones to the tail */
    for (int64_t j = 0; j < m - P; ++j) {
      int64_t r = j + (int64_t)rng_below(&rng, (uint64_t)(m - j));
      uint64_t t = key[j]; key[j] = key[r]; key[r] = t;
    }
    memmove(key, key + (m - P), sizeof(uint64_t) * (size_t)P);
    m = P;
    radix_u64(key, tmp, m, bits);
  }
  /* 5. degree floor 1: attach every isolated node to a partner ~ w, then
     remove as many pairs whose endpoints both have degree >= 3 (then >= 2;
     random scan start) so that no endpoint becomes isolated */
  int64_t *deg = (int64_t *)calloc((size_t)n, sizeof(int64_t));
  for (int64_t i = 0; i < m; ++i) { deg[key[i] / n]++; deg[key[i] % n]++; }
  {
    int64_t attached = 0, m0 = m;
    for (int64_t v = 0; v < n; ++v) {
      if (deg[v] != 0) continue;
      int64_t u;
      do { u = alias_draw(&al, &rng); } while (u == v);
      if (m >= cap_keys) {
        cap_keys = m + 1024;
        key = (uint64_t *)realloc(key, sizeof(uint64_t) * (size_t)cap_keys);
        tmp = (uint64_t *)realloc(tmp, sizeof(uint64_t) * (size_t)cap_keys);
      }
      int64_t a2 = v < u ? v : u, b2 = v < u ? u : v;
      key[m++] = (uint64_t)a2 * (uint64_t)n + (uint64_t)b2;  /* new: v had no pair */
      deg[v]++; deg[u]++;
      ++attached;
    }
    if (attached > 0) {
      int64_t removed = 0, start = (int64_t)rng_below(&rng, (uint64_t)m0);
      uint8_t *dead = (uint8_t *)calloc((size_t)m, 1);
      for (int thr = 3; thr >= 2 && removed < attached; --thr)
        for (int64_t t = 0; t < m0 && removed < attached; ++t) {
          int64_t i = (start + t) % m0;
          int64_t a2 = (int64_t)(key[i] / n), b2 = (int64_t)(key[i] % n);
          if (!dead[i] && deg[a2] >= thr && deg[b2] >= thr) { dead[i] = 1; deg[a2]--; deg[b2]--; ++removed; }
        }
      int64_t k = 0;
      for (int64_t i = 0; i < m; ++i) if (!dead[i]) key[k++] = key[i];
      free(dead);
      m = k;
      radix_u64(key, tmp, m, bits);
    }
  }
  /* 6. relabel + symmetric CSR */
  int64_t *perm = (int64_t *)malloc(sizeof(int64_t) * n);
  for (int64_t i = 0; i < n; ++i) perm[i] = i;
  for (int64_t i = n - 1; i > 0; --i) {
    int64_t j = (int64_t)rng_below(&rng, (uint64_t)(i + 1));
    int64_t t = perm[i]; perm[i] = perm[j]; perm[j] = t;
  }
  memset(deg, 0, sizeof(int64_t) * (size_t)n);
  for (int64_t i = 0; i < m; ++i) { deg[perm[key[i] / n]]++; deg[perm[key[i] % n]]++; }
  rowptr[0] = 0;
  for (int64_t v = 0; v < n; ++v) rowptr[v + 1] = rowptr[v] + deg[v];
  if (rowptr[n] != nnz) { /* only the floor step can shift the count (by duplicates it removed) */
    free(deg); free(perm); free(key); free(tmp); free(tpl); free(tpl_off); alias_free(&al); free(w);
    return -5;
  }
  int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * n);
  memcpy(fill, rowptr, sizeof(int64_t) * n);
  for (int64_t i = 0; i < m; ++i) {
    int64_t a = perm[key[i] / n], b = perm[key[i] % n];
    colidx[fill[a]++] = (int32_t)b;
    colidx[fill[b]++] = (int32_t)a;
  }
  int64_t maxd = 0, zeros = 0;
  double m2 = 0, m1 = (double)nnz / n;
  for (int64_t v = 0; v < n; ++v) {
    const int64_t d = rowptr[v + 1] - rowptr[v];
    if (d > 1) qsort(colidx + rowptr[v], (size_t)d, sizeof(int32_t), cmp_i32);
    if (d > maxd) maxd = d;
    zeros += d == 0;
    m2 += ((double)d - m1) * ((double)d - m1);
  }
  if (stats) {
    stats[0] = maxd;
    stats[1] = (int64_t)llround(m1 * 1e6);
    stats[2] = (int64_t)llround(m2 / n * 1e3);
    stats[3] = zeros;
  }
  if (relabel_out) memcpy(relabel_out, perm, sizeof(int64_t) * (size_t)n);
  #undef PARTNER
  free(fill); free(deg); free(perm); free(key); free(tmp); free(tpl); free(tpl_off);
  alias_free(&al);
  free(w);
  return 0;
}

/* uniform fp32 features in [lo, hi) with row stride ld (pad columns = 0) */
void synth_uniform_f32(int64_t rows, int64_t cols, int64_t ld, float lo, float hi,
                       uint64_t seed, float *out) {
  rng_t rng = {seed * 0x9E3779B97F4A7C15ULL + 77ULL};
  for (int64_t i = 0; i < rows; ++i) {
    float *r = out + i * ld;
    for (int64_t j = 0; j < cols; ++j) r[j] = lo + (hi - lo) * (float)rng_u01(&rng);
    for (int64_t j = cols; j < ld; ++j) r[j] = 0.0f;
  }
}
