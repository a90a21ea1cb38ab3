/*
 * gen.h -- seeded synthetic-input generators shared by the oracle side and the
 * CUDA side (the ONLY code both sides use).  Nothing here implements any of the
 * method's arithmetic (no SpMM / SDDMM / plan / shard math): it only produces
 * graphs in hybrid CSR/COO form (Fig. 2d) and dense feature
 * matrices, deterministically from a seed.
 *
 * Randomness is counter based: every random draw is mix64(seed, stream, index)
 * (a splitmix64 finaliser chain), so results do not depend on thread count or
 * call order.  The recipe (degree law, communities, relabelling, values) is
 * documented in DESIGN.md "Input recipe".
 */
#ifndef GNN_GEN_H
#define GNN_GEN_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
  int64_t n;            /* nodes; the adjacency is square n x n (M = N)            */
  int64_t target_nnz;   /* nnz incl. the n self-loops; produced nnz is
                           n + 2*floor((target_nnz - n)/2) exactly                  */
  double gamma;         /* power-law exponent of the expected-degree law (> 1)     */
  double max_deg;       /* cap on the expected degree (<= 0: n - 1)                 */
  int32_t n_comm;       /* planted communities (>= 1)                               */
  double mu;            /* mixing: prob. the 2nd endpoint is drawn graph-wide        */
  int32_t relabel;      /* 1: random node relabelling (scatters hubs/communities)   */
  int32_t val_mode;     /* 0: U(0,1]  1: GCN 1/sqrt(deg_r*deg_c)  2: all ones      */
  uint64_t seed;
} gen_graph_params_t;

/* Upper bound on the nnz gen_graph() produces for these params. */
int64_t gen_graph_nnz(const gen_graph_params_t *p);

/* Generate a symmetric, self-looped, deduplicated graph sorted by (row, col).
 * Outputs (caller-allocated, host): row_ptr[n+1], row_ind[nnz], col_ind[nnz],
 * val[nnz] (val may be NULL), community of each (relabelled) node comm[n] (may be
 * NULL).  cap = capacity of the nnz arrays.  Returns 0 on success, <0 on error.
 * *nnz_out receives the produced nnz. */
int gen_graph(const gen_graph_params_t *p, int32_t *row_ptr, int32_t *row_ind,
              int32_t *col_ind, float *val, int32_t *comm, int64_t cap,
              int64_t *nnz_out);

/* Dense feature matrix, row-major rows x K with leading dimension ld >= K:
 * X[i][k] = U(-1,1) drawn from counter (seed, i*K + k).  Independent of ld and of
 * which row block is generated, so shards / gathers can regenerate any block:
 * rows [row0, row0 + rows). */
void gen_features(uint64_t seed, int64_t row0, int64_t rows, int64_t K, int64_t ld,
                  float *out);

/* Edge values only (used to re-value a graph): val[i] = U(0,1] from (seed, i). */
void gen_values_uniform(uint64_t seed, int64_t nnz, float *val);

#ifdef __cplusplus
}
#endif
#endif
