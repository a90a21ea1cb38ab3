/*
 * gen.c -- seeded synthetic graph / feature generators (see gen.h).
 *
 * Graph recipe ("Chung-Lu with planted communities"):
 *   1. expected off-diagonal degrees w_i = c * (i+1)^(-1/(gamma-1)), capped at
 *      max_deg, c solved so that sum_i w_i = 2 * U (U = undirected pairs wanted);
 *   2. every node gets a community hash(seed, i) % n_comm;
 *   3. sample s = 0,1,2,...: u ~ w (alias table); with prob mu, v ~ w graph-wide,
 *      else v ~ w restricted to comm(u); pair {u,v} (u != v);
 *   4. deduplicate; if fewer than U distinct pairs, sample more (the counter-based
 *      draws of a longer run extend the shorter one); if more, keep the U pairs with
 *      the smallest hash(seed, pair) -- so nnz is exact and thread-count independent;
 *   5. relabel nodes by a random permutation (scatters hubs, as in real graphs);
 *   6. emit both directions + a self-loop per node ("self-looped"),
 *      sorted by (row, col) -> hybrid CSR/COO (Fig. 2d);
 *   7. values: U(0,1], GCN 1/sqrt(deg_r deg_c), or ones.
 * None of this is the method's arithmetic; it only shapes inputs.
 */
#include "gen.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

/* ---------------------------------------------------------------- RNG ---- */
static inline uint64_t mix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ULL;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}
static inline uint64_t rnd(uint64_t seed, uint64_t stream, uint64_t i) {
  return mix64(mix64(mix64(seed) + stream) + i);
}
static inline double unif01(uint64_t r) { return (double)(r >> 11) * 0x1.0p-53; }

/* ---------------------------------------------------------- radix sort ---- */
/* LSD radix sort of uint64 keys whose values are < 2^bits; tmp has n slots.
 * Result ends in `a` (copied back if the pass count is odd). */
static void radix_sort_u64(uint64_t *a, uint64_t *tmp, int64_t n, int bits) {
  const int D = 11, B = 1 << D;
  int passes = (bits + D - 1) / D;
  int64_t *cnt = (int64_t *)malloc(sizeof(int64_t) * B);
  uint64_t *src = a, *dst = tmp;
  for (int p = 0; p < passes; ++p) {
    int sh = p * D;
    memset(cnt, 0, sizeof(int64_t) * B);
    for (int64_t i = 0; i < n; ++i) cnt[(src[i] >> sh) & (B - 1)]++;
    int64_t s = 0;
    for (int b = 0; b < B; ++b) { int64_t c = cnt[b]; cnt[b] = s; s += c; }
    for (int64_t i = 0; i < n; ++i) dst[cnt[(src[i] >> sh) & (B - 1)]++] = src[i];
    uint64_t *t = src; src = dst; dst = t;
  }
  if (src != a) memcpy(a, src, sizeof(uint64_t) * n);
  free(cnt);
}

/* k-th smallest (0-based) of v[0..n) by quickselect (v is permuted). */
static uint64_t select_kth(uint64_t *v, int64_t n, int64_t k) {
  int64_t lo = 0, hi = n - 1;
  uint64_t st = 0x12345ULL;
  while (lo < hi) {
    st = mix64(st);
    uint64_t piv = v[lo + (int64_t)(st % (uint64_t)(hi - lo + 1))];
    int64_t i = lo, j = hi;
    while (i <= j) {
      while (v[i] < piv) ++i;
      while (v[j] > piv) --j;
      if (i <= j) { uint64_t t = v[i]; v[i] = v[j]; v[j] = t; ++i; --j; }
    }
    if (k <= j) hi = j; else if (k >= i) lo = i; else return v[k];
  }
  return v[k];
}

/* --------------------------------------------------------- alias table ---- */
static void alias_build(const double *w, int64_t n, double *prob, int32_t *alias) {
  double sum = 0;
  for (int64_t i = 0; i < n; ++i) sum += w[i];
  int32_t *small = (int32_t *)malloc(sizeof(int32_t) * n);
  int32_t *large = (int32_t *)malloc(sizeof(int32_t) * n);
  int64_t ns = 0, nl = 0;
  for (int64_t i = 0; i < n; ++i) {
    prob[i] = (sum > 0) ? w[i] * (double)n / sum : 1.0;
    alias[i] = (int32_t)i;
    if (prob[i] < 1.0) small[ns++] = (int32_t)i; else large[nl++] = (int32_t)i;
  }
  while (ns > 0 && nl > 0) {
    int32_t s = small[--ns], l = large[--nl];
    alias[s] = l;
    prob[l] = (prob[l] + prob[s]) - 1.0;
    if (prob[l] < 1.0) small[ns++] = l; else large[nl++] = l;
  }
  while (nl > 0) prob[large[--nl]] = 1.0;
  while (ns > 0) prob[small[--ns]] = 1.0;
  free(small);
  free(large);
}
static inline int64_t alias_draw(const double *prob, const int32_t *alias, int64_t n,
                                 uint64_t r) {
  int64_t j = (int64_t)(((r >> 32) * (uint64_t)n) >> 32);
  double coin = (double)(r & 0xffffffffULL) * 0x1.0p-32;
  return coin < prob[j] ? j : alias[j];
}

/* ------------------------------------------------------------- graphs ---- */
int64_t gen_graph_nnz(const gen_graph_params_t *p) {
  if (!p || p->n <= 0) return 0;
  int64_t t = p->target_nnz < p->n ? p->n : p->target_nnz;
  return p->n + 2 * ((t - p->n) / 2);
}

static int cmp_i32(const void *a, const void *b) {
  int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
  return (x > y) - (x < y);
}

int gen_graph(const gen_graph_params_t *p, int32_t *row_ptr, int32_t *row_ind,
              int32_t *col_ind, float *val, int32_t *comm, int64_t cap,
              int64_t *nnz_out) {
  if (!p || !row_ptr || !row_ind || !col_ind || !nnz_out) return -1;
  const int64_t n = p->n;
  if (n <= 0 || n >= (1LL << 30) || p->gamma <= 1.0 || p->n_comm < 1) return -1;
  const int64_t nnz = gen_graph_nnz(p);
  if (nnz > cap || nnz >= (1LL << 31)) return -2;
  const int64_t U = (nnz - n) / 2; /* distinct undirected off-diagonal pairs */
  if ((double)U > 0.5 * (double)n * (double)(n - 1)) return -3;
  const uint64_t seed = p->seed;
  int nb = 1;
  while ((1LL << nb) < n) ++nb;
  const uint64_t mask = (1ULL << nb) - 1;

  /* 1. expected degrees */
  double *w = (double *)malloc(sizeof(double) * n);
  const double beta = 1.0 / (p->gamma - 1.0);
  const double dmax = p->max_deg > 0 ? p->max_deg : (double)(n - 1);
  const double want = 2.0 * (double)U;
  for (int64_t i = 0; i < n; ++i) w[i] = pow((double)(i + 1), -beta);
  double c = 0;
  {
    double s = 0;
    for (int64_t i = 0; i < n; ++i) s += w[i];
    c = s > 0 ? want / s : 0;
    for (int it = 0; it < 100; ++it) {
      double sc = 0;
      for (int64_t i = 0; i < n; ++i) { double x = c * w[i]; sc += x < dmax ? x : dmax; }
      if (sc <= 0 || fabs(sc - want) <= 1e-9 * want) break;
      c *= want / sc;
    }
  }
  for (int64_t i = 0; i < n; ++i) { double x = c * w[i]; w[i] = x < dmax ? x : dmax; }

  /* 2. communities (pre-relabel ids) and per-community alias tables */
  const int64_t nc = p->n_comm;
  int32_t *comm0 = (int32_t *)malloc(sizeof(int32_t) * n);
  int64_t *coff = (int64_t *)calloc(nc + 1, sizeof(int64_t));
  for (int64_t i = 0; i < n; ++i) {
    comm0[i] = (int32_t)(rnd(seed, 1, i) % (uint64_t)nc);
    coff[comm0[i] + 1]++;
  }
  for (int64_t k = 0; k < nc; ++k) coff[k + 1] += coff[k];
  int32_t *cnodes = (int32_t *)malloc(sizeof(int32_t) * n);
  {
    int64_t *fill = (int64_t *)malloc(sizeof(int64_t) * nc);
    memcpy(fill, coff, sizeof(int64_t) * nc);
    for (int64_t i = 0; i < n; ++i) cnodes[fill[comm0[i]]++] = (int32_t)i;
    free(fill);
  }
  double *gprob = (double *)malloc(sizeof(double) * n);
  int32_t *galias = (int32_t *)malloc(sizeof(int32_t) * n);
  alias_build(w, n, gprob, galias);
  double *cprob = (double *)malloc(sizeof(double) * n);
  int32_t *calias = (int32_t *)malloc(sizeof(int32_t) * n);
  {
    double *cw = (double *)malloc(sizeof(double) * n);
    for (int64_t i = 0; i < n; ++i) cw[i] = w[cnodes[i]];
    for (int64_t k = 0; k < nc; ++k) {
      int64_t o = coff[k], m = coff[k + 1] - o;
      if (m > 0) alias_build(cw + o, m, cprob + o, calias + o);
    }
    free(cw);
  }

  /* 3-4. sample pairs until >= U distinct, then keep exactly U */
  uint64_t *keys = NULL, *tmp = NULL;
  int64_t nkeys = 0;
  int64_t S = U + U / 8 + 1024;
  int ok = 0;
  for (int round = 0; round < 40 && U > 0; ++round) {
    free(keys);
    free(tmp);
    keys = (uint64_t *)malloc(sizeof(uint64_t) * S);
    tmp = (uint64_t *)malloc(sizeof(uint64_t) * S);
#pragma omp parallel for schedule(static)
    for (int64_t s = 0; s < S; ++s) {
      int64_t u = alias_draw(gprob, galias, n, rnd(seed, 10, s));
      int64_t v;
      if (unif01(rnd(seed, 11, s)) < p->mu || nc == 1) {
        v = alias_draw(gprob, galias, n, rnd(seed, 12, s));
      } else {
        int32_t k = comm0[u];
        int64_t o = coff[k], m = coff[k + 1] - o;
        v = cnodes[o + alias_draw(cprob + o, calias + o, m, rnd(seed, 12, s))];
      }
      uint64_t lo = (uint64_t)(u < v ? u : v), hi = (uint64_t)(u < v ? v : u);
      keys[s] = (u == v) ? UINT64_MAX : ((lo << nb) | hi);
    }
    int64_t m = 0;
    for (int64_t s = 0; s < S; ++s)
      if (keys[s] != UINT64_MAX) keys[m++] = keys[s];
    radix_sort_u64(keys, tmp, m, 2 * nb);
    int64_t uq = 0;
    for (int64_t s = 0; s < m; ++s)
      if (uq == 0 || keys[s] != keys[uq - 1]) keys[uq++] = keys[s];
    nkeys = uq;
    if (uq >= U) { ok = 1; break; }
    double f = uq > 0 ? (double)U / (double)uq : 2.0;
    if (f > 4.0) f = 4.0;
    S = (int64_t)((double)S * f * 1.05) + 4096;
  }
  if (U == 0) ok = 1;
  if (!ok) {
    free(keys); free(tmp); free(w); free(comm0); free(coff); free(cnodes);
    free(gprob); free(galias); free(cprob); free(calias);
    return -4;
  }
  if (nkeys > U) {
    /* keep the U pairs with the smallest hash(seed, 14, pair); ties by key order */
    uint64_t *h = tmp; /* reuse (size S >= nkeys) */
    for (int64_t j = 0; j < nkeys; ++j) h[j] = rnd(seed, 14, keys[j]);
    uint64_t *hc = (uint64_t *)malloc(sizeof(uint64_t) * nkeys);
    memcpy(hc, h, sizeof(uint64_t) * nkeys);
    uint64_t thr = select_kth(hc, nkeys, U - 1);
    free(hc);
    int64_t below = 0;
    for (int64_t j = 0; j < nkeys; ++j) below += (h[j] < thr);
    int64_t eq_quota = U - below, m = 0;
    for (int64_t j = 0; j < nkeys; ++j) {
      if (h[j] < thr || (h[j] == thr && eq_quota-- > 0)) keys[m++] = keys[j];
    }
    nkeys = m;
  }

  /* 5. relabel: pi[i] = rank of i when nodes are sorted by hash(seed, 15, i) */
  int32_t *pi = (int32_t *)malloc(sizeof(int32_t) * n);
  if (p->relabel) {
    uint64_t *rk = (uint64_t *)malloc(sizeof(uint64_t) * n);
    uint64_t *rt = (uint64_t *)malloc(sizeof(uint64_t) * n);
    for (int64_t i = 0; i < n; ++i) rk[i] = (rnd(seed, 15, i) & ~mask) | (uint64_t)i;
    radix_sort_u64(rk, rt, n, 64);
    for (int64_t r = 0; r < n; ++r) pi[rk[r] & mask] = (int32_t)r;
    free(rk);
    free(rt);
  } else {
    for (int64_t i = 0; i < n; ++i) pi[i] = (int32_t)i;
  }
  if (comm)
    for (int64_t i = 0; i < n; ++i) comm[pi[i]] = comm0[i];

  /* 6. CSR: counting sort by row, then sort columns within each row */
  int64_t *deg = (int64_t *)calloc(n + 1, sizeof(int64_t));
  for (int64_t i = 0; i < n; ++i) deg[i] = 1; /* self-loop */
  for (int64_t j = 0; j < nkeys; ++j) {
    deg[pi[keys[j] >> nb]]++;
    deg[pi[keys[j] & mask]]++;
  }
  row_ptr[0] = 0;
  for (int64_t i = 0; i < n; ++i) row_ptr[i + 1] = (int32_t)(row_ptr[i] + deg[i]);
  int64_t *fill = deg; /* reuse as cursor */
  for (int64_t i = 0; i < n; ++i) fill[i] = row_ptr[i];
  for (int64_t i = 0; i < n; ++i) col_ind[fill[i]++] = (int32_t)i;
  for (int64_t j = 0; j < nkeys; ++j) {
    int32_t a = pi[keys[j] >> nb], b = pi[keys[j] & mask];
    col_ind[fill[a]++] = b;
    col_ind[fill[b]++] = a;
  }
#pragma omp parallel for schedule(dynamic, 1024)
  for (int64_t i = 0; i < n; ++i) {
    int32_t *c0 = col_ind + row_ptr[i];
    int64_t len = row_ptr[i + 1] - row_ptr[i];
    if (len < 24) {
      for (int64_t x = 1; x < len; ++x) {
        int32_t v = c0[x];
        int64_t y = x - 1;
        while (y >= 0 && c0[y] > v) { c0[y + 1] = c0[y]; --y; }
        c0[y + 1] = v;
      }
    } else {
      qsort(c0, (size_t)len, sizeof(int32_t), cmp_i32);
    }
    for (int64_t x = row_ptr[i]; x < row_ptr[i + 1]; ++x) row_ind[x] = (int32_t)i;
  }

  /* 7. values */
  if (val) {
    if (p->val_mode == 0) {
      gen_values_uniform(seed ^ 0x5A5A5A5AULL, nnz, val);
    } else if (p->val_mode == 1) {
#pragma omp parallel for schedule(static)
      for (int64_t x = 0; x < nnz; ++x) {
        double dr = (double)(row_ptr[row_ind[x] + 1] - row_ptr[row_ind[x]]);
        double dc = (double)(row_ptr[col_ind[x] + 1] - row_ptr[col_ind[x]]);
        val[x] = (float)(1.0 / sqrt(dr * dc));
      }
    } else {
      for (int64_t x = 0; x < nnz; ++x) val[x] = 1.0f;
    }
  }
  *nnz_out = nnz;

  free(keys); free(tmp); free(w); free(comm0); free(coff); free(cnodes);
  free(gprob); free(galias); free(cprob); free(calias); free(pi); free(deg);
  return 0;
}

/* ----------------------------------------------------------- features ---- */
void gen_features(uint64_t seed, int64_t row0, int64_t rows, int64_t K, int64_t ld,
                  float *out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < rows; ++i) {
    uint64_t base = (uint64_t)(row0 + i) * (uint64_t)K;
    float *o = out + i * ld;
    for (int64_t k = 0; k < K; ++k) {
      uint64_t r = rnd(seed, 20, base + (uint64_t)k) >> 40; /* 24 random bits */
      /* odd multiples of 2^-24 in (-1, 1): exact in fp32, never 0 or subnormal */
      o[k] = (float)(((double)(int64_t)(2 * r + 1) - 16777216.0) * 0x1.0p-24);
    }
  }
}

void gen_values_uniform(uint64_t seed, int64_t nnz, float *val) {
#pragma omp parallel for schedule(static)
  for (int64_t x = 0; x < nnz; ++x) {
    uint64_t r = rnd(seed, 21, (uint64_t)x) >> 40;     /* 24 bits */
    val[x] = (float)((double)(r + 1) * 0x1.0p-24);    /* (0, 1] */
  }
}
