/* Host-side sanitizer driver (SURVEY.md §5 "Race detection / sanitizers"): the oracle and
 * the generators compiled with -fsanitize=address,undefined and exercised on small
 * cases, including the edge shapes (empty graph, single hub row, rectangular sub-ranges,
 * NULL values, every aggregator, P > nnz shards).  Exit 0 = no sanitizer report and
 * every self-check held.  Built and run by tests/test_sanitize_host.py. */
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "../../gen/gen.h"
#include "../../oracle/oracle.h"

#define CHECK(c)                                                  \
  do {                                                            \
    if (!(c)) {                                                   \
      fprintf(stderr, "check failed: %s (line %d)\n", #c, __LINE__); \
      return 1;                                                   \
    }                                                             \
  } while (0)

static int run_graph(int64_t n, int64_t nnz_target, int32_t n_comm, uint64_t seed) {
  gen_graph_params_t p = {n, nnz_target, 2.3, 0.0, n_comm, 0.3, 1, 1, seed};
  int64_t cap = gen_graph_nnz(&p);
  int32_t *rp = malloc(sizeof(int32_t) * (n + 1)), *ri = malloc(sizeof(int32_t) * cap),
          *ci = malloc(sizeof(int32_t) * cap), *comm = malloc(sizeof(int32_t) * n);
  float *val = malloc(sizeof(float) * cap);
  int64_t nnz = 0;
  CHECK(gen_graph(&p, rp, ri, ci, val, comm, cap, &nnz) == 0);
  CHECK(nnz <= cap && rp[n] == nnz);
  const int32_t Ks[] = {1, 3, 8, 32, 64};
  for (int q = 0; q < 5; ++q) {
    const int32_t K = Ks[q];
    float *X = malloc(sizeof(float) * n * K);
    gen_features(seed + K, 0, n, K, K, X);
    double *O = malloc(sizeof(double) * n * K), *T = malloc(sizeof(double) * n * K);
    CHECK(oracle_spmm(0, nnz, ri, ci, val, K, X, K, 0, n, O, T) == 0);
    CHECK(oracle_spmm(0, nnz, ri, ci, NULL, K, X, K, 0, n, O, T) == 0);
    for (int agg = 0; agg < 4; ++agg)
      CHECK(oracle_spmm_agg(0, nnz, ri, ci, val, K, X, K, 0, n, agg, O, T) == 0);
    if (nnz > 0) {  /* a sub-range of rows */
      const int64_t i0 = rp[n / 3], i1 = rp[n / 2];
      CHECK(oracle_spmm(i0, i1, ri, ci, val, K, X, K, n / 3, n / 2 - n / 3, O, T) == 0);
    }
    double *E = malloc(sizeof(double) * (nnz + 1)), *TE = malloc(sizeof(double) * (nnz + 1));
    CHECK(oracle_sddmm(0, nnz, ri, ci, val, K, X, K, X, K, E, TE) == 0);
    for (int dt = 0; dt < 2; ++dt) {
      if (dt == 1 && K % 2) continue;
      oracle_plan_info_t info;
      const int64_t nch_max = nnz / 8 + 2;
      int32_t *rf = malloc(sizeof(int32_t) * nch_max), *rl = malloc(sizeof(int32_t) * nch_max);
      uint8_t *fl = malloc(nch_max);
      CHECK(oracle_plan(nnz, ri, K, 2, 8, 0, 0, dt, 148, 2, n, 132644864, &info, rf, rl, fl) == 0);
      CHECK(info.num_chunks <= nch_max);
      CHECK(oracle_plan(nnz, ri, K, 2, 8, 8, 0, dt, 148, 2, n, 0, &info, rf, rl, fl) == 0);
      free(rf); free(rl); free(fl);
    }
    free(X); free(O); free(T); free(E); free(TE);
  }
  int64_t b[65];
  for (int P = 1; P <= 64; P *= 2) {
    CHECK(oracle_shard_rows(rp, n, P, b) == 0);
    CHECK(b[0] == 0 && b[P] == n);
    CHECK(oracle_shard_edges(nnz, P, b) == 0);
  }
  int32_t *ri2 = malloc(sizeof(int32_t) * (nnz + 1));
  CHECK(oracle_csr_to_coo(rp, n, ri2) == 0);
  CHECK(memcmp(ri, ri2, sizeof(int32_t) * nnz) == 0);
  const double Q = oracle_modularity(rp, ci, n, comm, 1);
  CHECK(Q > -1.0 && Q <= 1.0);
  free(rp); free(ri); free(ci); free(comm); free(val); free(ri2);
  return 0;
}

int main(void) {
  int rc = 0;
  rc |= run_graph(1, 1, 1, 1);          /* a single self-loop */
  rc |= run_graph(2, 2, 1, 2);
  rc |= run_graph(100, 1000, 3, 3);
  rc |= run_graph(1000, 10000, 4, 4);   /* C1-sized */
  rc |= run_graph(3000, 200000, 5, 5);  /* dense-ish, hub rows span many chunks */
  if (rc == 0) printf("sanitize driver ok\n");
  return rc;
}
