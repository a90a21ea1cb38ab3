/*
 * oracle.c -- TEST INFRASTRUCTURE ONLY (see oracle.h).  Plain C, fp64, no
 * blocking / fusion / reordering beyond what the paper's algorithms state.
 * Compiled with -O2 -ffp-contract=off (no FMA contraction, no fast-math) -fopenmp: SpMM
 * runs one contiguous range of whole rows per thread, SDDMM splits the nonzeros; neither
 * changes any sum's order, so results are identical for every thread count.
 */
#include "oracle.h"

#include <math.h>
#include <stddef.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* Thread count of the OpenMP loops below (timing / determinism tests); 0 = unchanged. */
int oracle_threads(int n) {
#ifdef _OPENMP
  if (n > 0) omp_set_num_threads(n);
  return omp_get_max_threads();
#else
  (void)n;
  return 1;
#endif
}

/* ------------------------------------------------------------ SpMM ------ */
/* Algorithm 1 over nonzeros [s, e). */
static int spmm_range(int64_t s, int64_t e, const int32_t *row_ind, const int32_t *col_ind,
                      const float *val, int64_t K, const float *A, int64_t lda, int64_t r0,
                      int64_t nrows, double *O, double *T) {
  for (int64_t i = s; i < e; ++i) {                         /* line 1 */
    int64_t r = row_ind[i], c = col_ind[i];                 /* line 2 */
    double v = val ? (double)val[i] : 1.0;
    if (r < r0 || r >= r0 + nrows || c < 0) return -1;
    double *o = O + (r - r0) * K;
    const float *a = A + c * lda;
    for (int64_t k = 0; k < K; ++k) {                       /* line 3 */
      double term = v * (double)a[k];
      o[k] += term;                                         /* line 4 */
      if (T) T[(r - r0) * K + k] += fabs(term);
    }
  }
  return 0;
}

/* Algorithm 1 over [i0, i1).  With OpenMP the nonzeros are cut into one contiguous range
 * per thread, each cut moved forward to the next row start, so every row is summed by one
 * thread in nonzero order: the result is the serial loop's, bit for bit, for any thread
 * count (row_ind is non-decreasing). */
int oracle_spmm(int64_t i0, int64_t i1, const int32_t *row_ind, const int32_t *col_ind,
                const float *val, int64_t K, const float *A, int64_t lda, int64_t r0,
                int64_t nrows, double *O, double *T) {
  if (i0 < 0 || i1 < i0 || K < 1 || lda < K || nrows < 0) return -1;
  memset(O, 0, sizeof(double) * (size_t)(nrows * K));
  if (T) memset(T, 0, sizeof(double) * (size_t)(nrows * K));
  int nt = 1;
#ifdef _OPENMP
  nt = omp_get_max_threads();
  if ((i1 - i0) < 65536) nt = 1;
#endif
  int rc = 0;
#pragma omp parallel num_threads(nt) reduction(| : rc)
  {
    int t = 0;
#ifdef _OPENMP
    t = omp_get_thread_num();
#endif
    int64_t s = i0 + (i1 - i0) * t / nt, e = i0 + (i1 - i0) * (t + 1) / nt;
    while (s > i0 && s < i1 && row_ind[s] == row_ind[s - 1]) ++s;  /* own whole rows */
    while (e > i0 && e < i1 && row_ind[e] == row_ind[e - 1]) ++e;
    if (s < e) rc |= spmm_range(s, e, row_ind, col_ind, val, K, A, lda, r0, nrows, O, T);
  }
  return rc ? -1 : 0;
}

/* ------------------------------------------------ aggregated SpMM ------ */
/* Eq. 1 with f_n = v * X_u and (+) = sum / mean / max / min. */
int oracle_spmm_agg(int64_t i0, int64_t i1, const int32_t *row_ind, const int32_t *col_ind,
                    const float *val, int64_t K, const float *A, int64_t lda, int64_t r0,
                    int64_t nrows, int32_t agg, double *O, double *T) {
  if (agg < 0 || agg > 3) return -1;
  if (agg <= 1) {
    int rc = oracle_spmm(i0, i1, row_ind, col_ind, val, K, A, lda, r0, nrows, O, T);
    if (rc != 0 || agg == 0) return rc;
    /* mean: divide each row by its number of terms */
    for (int64_t r = 0; r < nrows; ++r) {
      int64_t cnt = 0;
      for (int64_t i = i0; i < i1; ++i) cnt += (row_ind[i] == r0 + r);
      if (cnt == 0) continue;
      for (int64_t k = 0; k < K; ++k) {
        O[r * K + k] /= (double)cnt;
        if (T) T[r * K + k] /= (double)cnt;
      }
    }
    return 0;
  }
  if (i0 < 0 || i1 < i0 || K < 1 || lda < K || nrows < 0) return -1;
  char *seen = (char *)calloc((size_t)nrows + 1, 1);
  memset(O, 0, sizeof(double) * (size_t)(nrows * K));
  if (T) memset(T, 0, sizeof(double) * (size_t)(nrows * K));
  for (int64_t i = i0; i < i1; ++i) {
    int64_t r = row_ind[i], c = col_ind[i];
    double v = val ? (double)val[i] : 1.0;
    if (r < r0 || r >= r0 + nrows || c < 0) { free(seen); return -1; }
    double *o = O + (r - r0) * K;
    const float *a = A + c * lda;
    for (int64_t k = 0; k < K; ++k) {
      double term = v * (double)a[k];
      if (!seen[r - r0]) o[k] = term;
      else if (agg == 2 ? term > o[k] : term < o[k]) o[k] = term;
      if (T && fabs(term) > T[(r - r0) * K + k]) T[(r - r0) * K + k] = fabs(term);
    }
    seen[r - r0] = 1;
  }
  free(seen);
  return 0;
}

/* Backward of the max / min node-wise op (Eq. 1; the subgradient rule is
 * DESIGN.md reading 26).  The forward keeps one fp32 product fl(v_i * A[c_i][k]) per
 * (r, k) -- the decision is taken in the kernel's precision (fp32 products, exact
 * comparisons), the gradients are accumulated in fp64:
 *   1. E[r][k] = max (min) over the row's nonzeros of the fp32 product;
 *   2. the first nonzero i of row r (storage order) whose product equals E[r][k] gets
 *      dA[c_i][k] += v_i * dO[r][k] and dval[i - i0] += A[c_i][k] * dO[r][k].
 * dA (N x K, zeroed here) and dval (i1 - i0, zeroed here; may be NULL). */
int oracle_spmm_extremum_backward(int64_t i0, int64_t i1, const int32_t *row_ind,
                                  const int32_t *col_ind, const float *val, int64_t K,
                                  const float *A, int64_t lda, int64_t N, int64_t r0,
                                  int64_t nrows, int32_t agg, const float *dO, double *dA,
                                  double *dval) {
  if (i0 < 0 || i1 < i0 || K < 1 || lda < K || nrows < 0 || N < 0 || (agg != 2 && agg != 3))
    return -1;
  memset(dA, 0, sizeof(double) * (size_t)(N * K));
  if (dval) memset(dval, 0, sizeof(double) * (size_t)(i1 - i0));
  float *E = (float *)malloc(sizeof(float) * (size_t)(nrows * K + 1));
  char *seen = (char *)calloc((size_t)nrows + 1, 1);
  char *taken = (char *)calloc((size_t)(nrows * K + 1), 1);
  if (!E || !seen || !taken) { free(E); free(seen); free(taken); return -1; }
  for (int64_t i = i0; i < i1; ++i) {                       /* step 1 */
    int64_t r = row_ind[i] - r0, c = col_ind[i];
    if (r < 0 || r >= nrows || c < 0 || c >= N) { free(E); free(seen); free(taken); return -1; }
    float v = val ? val[i] : 1.0f;
    for (int64_t k = 0; k < K; ++k) {
      float p = v * A[c * lda + k];
      float *e = E + r * K + k;
      if (!seen[r] || (agg == 2 ? p > *e : p < *e)) *e = p;
    }
    seen[r] = 1;
  }
  for (int64_t i = i0; i < i1; ++i) {                       /* step 2, storage order */
    int64_t r = row_ind[i] - r0, c = col_ind[i];
    float v = val ? val[i] : 1.0f;
    for (int64_t k = 0; k < K; ++k) {
      float p = v * A[c * lda + k];
      if (taken[r * K + k] || p != E[r * K + k]) continue;
      taken[r * K + k] = 1;
      double g = (double)dO[r * K + k];
      dA[c * K + k] += (double)v * g;
      if (dval) dval[i - i0] += (double)A[c * lda + k] * g;
    }
  }
  free(E); free(seen); free(taken);
  return 0;
}

/* ----------------------------------------------------------- SDDMM ------ */
/* Algorithm 2. */
int oracle_sddmm(int64_t i0, int64_t i1, const int32_t *row_ind, const int32_t *col_ind,
                 const float *val, int64_t K, const float *A1, int64_t lda1,
                 const float *A2T, int64_t lda2, double *out, double *T) {
  if (i0 < 0 || i1 < i0 || K < 1 || lda1 < K || lda2 < K) return -1;
  int rc = 0;
  /* every output is independent: OpenMP over the nonzeros changes no arithmetic */
#pragma omp parallel for schedule(static) reduction(| : rc) if (i1 - i0 >= 16384)
  for (int64_t i = i0; i < i1; ++i) {                       /* line 1 */
    int64_t r = row_ind[i], c = col_ind[i];                 /* line 2 */
    double v = val ? (double)val[i] : 1.0;
    if (r < 0 || c < 0) { rc |= 1; continue; }
    const float *a1 = A1 + r * lda1;
    const float *a2 = A2T + c * lda2;                       /* A2[k][c] = A2T[c][k] */
    double acc = 0.0, tabs = 0.0;
    for (int64_t k = 0; k < K; ++k) {                       /* line 3 */
      double term = (double)a1[k] * (double)a2[k];
      acc += term;                                          /* line 4 */
      tabs += fabs(term);
    }
    out[i - i0] = acc * v;                                  /* line 6 */
    if (T) T[i - i0] = fabs(v) * tabs;
  }
  return rc ? -1 : 0;
}

/* ------------------------------------------------------------ plan ------ */
/* NnzPerWarp candidate set. */
static const int32_t kCandidates[6] = {8, 32, 64, 128, 256, 512};

static int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

/* Right-hand side of InEq. (5) in integer form: the number of thread
 * blocks launched when every chunk of C nnz is cut into S K-slices, each slice
 * is one lane group's work item, G groups share a warp, WPB warps a block. */
static int64_t blocks_for(int64_t nnz, int64_t C, int64_t S, int64_t G, int64_t WPB) {
  int64_t chunks = cdiv(nnz, C);
  int64_t items = chunks * S;
  int64_t warps = cdiv(items, G);
  return cdiv(warps, WPB);
}

int oracle_plan(int64_t nnz, const int32_t *row_ind, int32_t K, int32_t alpha,
                int32_t warps_per_block, int32_t force_chunk, int32_t force_vw,
                int32_t feature_dtype, int32_t num_sms, int32_t active_blocks_per_sm,
                int64_t M, int64_t l2_bytes, oracle_plan_info_t *info,
                int32_t *row_first, int32_t *row_last, uint8_t *flags) {
  if (nnz < 0 || K < 1 || alpha < 1 || warps_per_block < 1 || num_sms < 1 ||
      active_blocks_per_sm < 1 || force_chunk < 0 || M < 0 || l2_bytes < 0 || !info)
    return -1;
  /* step 1: feature vector width in elements of the feature dtype (0 fp32: 8,4,2,1;
   * 1 bf16: 16,8,4,2): the widest that divides K, or forced */
  int32_t vmax, vmin, vw = 0;
  if (feature_dtype == 0) { vmax = 8; vmin = 1; }
  else if (feature_dtype == 1) { vmax = 16; vmin = 2; }
  else return -1;
  if (force_vw > 0) {
    int ok = 0;
    for (int32_t v = vmin; v <= vmax; v *= 2) ok |= (force_vw == v);
    if (!ok || K % force_vw != 0) return -1;
    vw = force_vw;
  } else {
    for (int32_t v = vmax; v >= vmin; v /= 2)
      if (vw == 0 && K % v == 0) vw = v;
    if (vw == 0) return -1;
  }
  /* step 2: vectors per lane, lanes per chunk-slice, slices, groups per warp */
  int64_t need = cdiv(K, vw);          /* VW-wide vectors in a feature row */
  int32_t R = need >= 16 ? 2 : 1;
  int32_t L = 1;
  while (L < cdiv(need, R) && L < 32) L *= 2;
  int32_t S = (int32_t)cdiv(K, (int64_t)L * R * vw);
  int32_t G = 32 / L;
  /* step 3: FullWaveSize = NumSM x ActiveblocksPerSM (Eqs. 3-4) */
  int64_t FW = (int64_t)num_sms * active_blocks_per_sm;
  /* steps 4-5: largest candidate satisfying InEq. (5), else 8 */
  int32_t C = 8;
  for (int j = 0; j < 6; ++j) {
    if (blocks_for(nnz, kCandidates[j], S, G, warps_per_block) >= (int64_t)alpha * FW)
      C = kCandidates[j];
  }
  int32_t C_dtp = C;
  /* step 5b (a B200 reading -- not in the paper): the locality
   * cap.  One full wave holds FW x WarpsPerBlock x G / S chunks; with C nonzeros each
   * that is (FW x WPB x G x C) / S nonzeros in flight, covering about
   * nonzeros x M / nnz rows (at most M).  Their feature rows, rows x K x eb bytes
   * (eb = 4 fp32, 2 bf16), must fit a quarter of L2: compared without overflow as
   * rows <= floor(floor(L2 / 4) / (K x eb)).  The largest candidate <= C_dtp that fits
   * wins; if none fits, 8.  l2_bytes == 0 switches the cap off. */
  if (l2_bytes > 0 && nnz > 0 && M > 0) {
    int64_t eb = feature_dtype == 1 ? 2 : 4;
    int64_t rows_that_fit = (l2_bytes / 4) / ((int64_t)K * eb);
    int32_t capped = 8;
    for (int j = 0; j < 6; ++j) {
      int32_t cand = kCandidates[j];
      if (cand > C_dtp) continue;
      int64_t chunks_in_flight_x_C = FW * warps_per_block * G * cand;
      int64_t nnz_in_flight = chunks_in_flight_x_C / S;
      int64_t rows_in_flight = nnz_in_flight * M / nnz;
      if (rows_in_flight > M) rows_in_flight = M;
      if (rows_in_flight <= rows_that_fit) capped = cand;
    }
    C = capped;
    /* step 5c (a B200 reading -- not in the paper; on with the
     * cap): where InEq. (5) itself chose fewer than 64 nonzeros per chunk, C = 64. */
    if (C_dtp < 64) C = 64;
  }
  if (force_chunk > 0) C = force_chunk;
  /* step 6: sparse-load vector width (HVMA) */
  int32_t vws = 1;
  if (C >= 128 && C % 4 == 0) vws = 4;
  else if (C >= 64 && C % 2 == 0) vws = 2;
  /* step 7: chunks (Algo 3 lines 2-3: warp_start = id x NnzPerWarp, end clamped) */
  int64_t nch = nnz > 0 ? cdiv(nnz, C) : 0;
  info->chunk = C;
  info->vw_feat = vw;
  info->vw_sparse = vws;
  info->lanes = L;
  info->vecs = R;
  info->slices = S;
  info->groups = G;
  info->warps_per_block = warps_per_block;
  info->active_blocks_per_sm = active_blocks_per_sm;
  info->num_sms = num_sms;
  info->alpha = alpha;
  info->K = K;
  info->feature_dtype = feature_dtype;
  info->chunk_dtp = C_dtp;
  info->M = M;
  info->l2_bytes = l2_bytes;
  info->nnz = nnz;
  info->num_chunks = nch;
  info->num_blocks = nnz > 0 ? blocks_for(nnz, C, S, G, warps_per_block) : 0;
  for (int64_t c = 0; c < nch; ++c) {
    int64_t s = c * C;
    int64_t e = s + C < nnz ? s + C : nnz;
    if (row_first) row_first[c] = row_ind[s];
    if (row_last) row_last[c] = row_ind[e - 1];
    if (flags) {
      uint8_t f = 0;
      if (s > 0 && row_ind[s - 1] == row_ind[s]) f |= 1;      /* head continues */
      if (e < nnz && row_ind[e] == row_ind[e - 1]) f |= 2;    /* tail continues */
      flags[c] = f;
    }
  }
  return 0;
}

/* ---------------------------------------------------------- shards ------ */
int oracle_shard_rows(const int32_t *row_ptr, int64_t M, int32_t P, int64_t *bounds) {
  if (!row_ptr || M < 0 || P < 1 || !bounds) return -1;
  int64_t base = row_ptr[0];
  int64_t nnz = (int64_t)row_ptr[M] - base;
  bounds[0] = 0;
  for (int32_t p = 1; p < P; ++p) {
    int64_t t = (int64_t)p * nnz / P;
    int64_t lo = 0, hi = M; /* first r in [0, M] with row_ptr[r] - base >= t */
    while (lo < hi) {
      int64_t mid = lo + (hi - lo) / 2;
      if ((int64_t)row_ptr[mid] - base >= t) hi = mid; else lo = mid + 1;
    }
    bounds[p] = lo < bounds[p - 1] ? bounds[p - 1] : lo;
  }
  bounds[P] = M;
  return 0;
}

int oracle_shard_edges(int64_t nnz, int32_t P, int64_t *bounds) {
  if (nnz < 0 || P < 1 || !bounds) return -1;
  for (int32_t p = 0; p <= P; ++p) bounds[p] = (int64_t)p * nnz / P;
  return 0;
}

int oracle_csr_to_coo(const int32_t *row_ptr, int64_t M, int32_t *row_ind) {
  if (!row_ptr || M < 0) return -1;
  int64_t base = row_ptr[0];
  for (int64_t r = 0; r < M; ++r)
    for (int64_t i = row_ptr[r]; i < row_ptr[r + 1]; ++i) row_ind[i - base] = (int32_t)r;
  return 0;
}

/* ------------------------------------------------------- modularity ------ */
#include <stdlib.h>
double oracle_modularity(const int32_t *row_ptr, const int32_t *col_ind, int64_t n,
                         const int32_t *comm, int32_t skip_self) {
  double *in = (double *)calloc((size_t)n + 1, sizeof(double));
  double *tot = (double *)calloc((size_t)n + 1, sizeof(double));
  double m2 = 0.0;
  int64_t base = row_ptr[0];
  for (int64_t i = 0; i < n; ++i) {
    for (int64_t e = row_ptr[i] - base; e < row_ptr[i + 1] - base; ++e) {
      int64_t j = col_ind[e];
      if (skip_self && j == i) continue;
      m2 += 1.0;                      /* sum_i k_i = 2m */
      tot[comm[i]] += 1.0;            /* k_i accumulated into tot_{c_i} */
      if (comm[j] == comm[i]) in[comm[i]] += 1.0;
    }
  }
  double q = 0.0;
  if (m2 > 0)
    for (int64_t c = 0; c < n; ++c) q += in[c] / m2 - (tot[c] / m2) * (tot[c] / m2);
  free(in);
  free(tot);
  return q;
}
