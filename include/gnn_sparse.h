/*
 * gnn_sparse.h -- C ABI of libgnnsparse.so, the B200 (sm_100a) hybrid-parallel
 * SpMM / SDDMM library for GNN message passing.
 *
 * Paper: R. Fan, W. Wang, X. Chu, "Fast Sparse GPU Kernels for Accelerated Training
 * of Graph Neural Networks", IPDPS 2023.  "P:n" below is /root/reference/PAPER.md
 * line n (the paper text; not needed at run time).
 *
 * Conventions for every entry point
 *   - All array pointers are DEVICE pointers unless the name ends in _host.
 *   - Sparse input is hybrid CSR/COO (Fig. 2d): row_ind[nnz] is the fully
 *     decoded, NON-DECREASING row index; col_ind[nnz], val[nnz] (val may be NULL,
 *     meaning every value is 1).  int32 indices, int64 sizes/offsets (P:295 max nnz
 *     264M fits int32).  Row r is a destination node, column c a source node
 *     (Table I).
 *   - Dense matrices are row-major fp32 with a leading dimension (pitch, in
 *     elements) >= K ("row-major ... FP32").
 *   - The caller owns every buffer (graph arrays, features, outputs and the plan
 *     workspace); the library never allocates device memory, except gnn_validate (an
 *     8-byte stream-ordered result flag, freed before it returns).
 *   - GNN_VALIDATE=1 in the environment makes gnn_plan_create (and everything built on
 *     it) run gnn_validate on the graph first -- a debug switch that synchronises.
 *   - Every call is asynchronous on the given stream (a cudaStream_t; NULL = the
 *     legacy default stream) and never synchronises the host, except
 *     gnn_validate().  Launch errors are returned as GNN_ERR_CUDA; faults inside a
 *     kernel surface at the caller's next synchronisation.
 *   - Calls return a gnn_status_t; no C++ exception crosses the ABI.  A thread-local
 *     message for the last failure is available from gnn_last_error().
 *   - There is no CPU fallback: without a usable sm_100 device every compute entry
 *     point returns GNN_ERR_CUDA.
 */
#ifndef GNN_SPARSE_H
#define GNN_SPARSE_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(_WIN32)
#define GNN_API
#else
#define GNN_API __attribute__((visibility("default")))
#endif

typedef enum {
  GNN_OK = 0,
  GNN_ERR_INVALID_ARG = 1,   /* NULL pointer, negative size, K < 1, bad option   */
  GNN_ERR_UNSUPPORTED = 2,   /* alignment/pitch not compatible with the plan's VW */
  GNN_ERR_CUDA = 3,          /* CUDA runtime / launch error or no sm_100 device   */
  GNN_ERR_WORKSPACE = 4,     /* workspace too small or misaligned                 */
  GNN_ERR_INPUT_CHECK = 5    /* gnn_validate found an invalid graph               */
} gnn_status_t;

typedef void *gnn_stream_t; /* a cudaStream_t */

/* Element type of the gathered feature matrices (A, A1, A2T).  Accumulation and the
 * outputs (O, S_O) are fp32 for both (bf16 halves the gathered bytes). */
typedef enum { GNN_F32 = 0, GNN_BF16 = 1 } gnn_dtype_t;

/* A hybrid CSR/COO adjacency S (M x N) or a row/edge shard of one.
 * A shard's row_ind holds GLOBAL row ids in [row_base, row_base + M); its
 * row_ind/col_ind/val pointers are sub-views starting at the shard's first nnz.
 * Kernels write output row r at O[(r - row_base) * ldo]. */
typedef struct {
  int64_t M, N, nnz;
  const int32_t *row_ptr;  /* [M+1] CSR offsets, read relative to row_ptr[0]; only
                              used by gnn_validate / gnn_csr_to_coo; may be NULL   */
  const int32_t *row_ind;  /* [nnz] non-decreasing, in [row_base, row_base + M)     */
  const int32_t *col_ind;  /* [nnz] in [0, N)                                       */
  const float *val;        /* [nnz] or NULL (all ones)                              */
  int64_t row_base;
} gnn_graph_t;

/* Plan options; zero-initialised fields take defaults. */
typedef struct {
  int32_t alpha;           /* InEq. (5) scale factor; default 2             */
  int32_t warps_per_block; /* WarpsPerBlock; 1..16, default 2               */
  int32_t force_chunk;     /* 0 = DTP choice; >0 forces NnzPerWarp (ablation/tests) */
  int32_t force_vw;        /* 0 = from K; 1/2/4/8 forces the feature vector width   */
  int32_t deterministic;   /* 1: SpMM sums rows split across chunks in chunk order
                              through per-chunk partials in the workspace (no atomics:
                              bit-reproducible; workspace grows by 8*K B per chunk)     */
  int32_t feature_dtype;   /* gnn_dtype_t of the feature matrices; default GNN_F32   */
  int32_t no_locality;     /* 1: plain DTP exactly as InEq. (5): skips
                              the L2 locality cap (DESIGN.md §3 step 5b) AND the chunk
                              floor (step 5c); 0 (default) applies both              */
  /* Device-parameter overrides (0 = query the current device).  They change only the
   * plan's arithmetic (DTP's NumSM, ActiveblocksPerSM and the cap's L2 size), never the
   * launch: tests use them to feed identical inputs to the library and the oracle. */
  int32_t num_sms;              /* NumSM of Eq. 4                                      */
  int32_t active_blocks_per_sm; /* ActiveblocksPerSM of Eq. 3 (else the occupancy API) */
  int64_t l2_bytes;             /* L2 bytes of step 5b (no_locality still disables it) */
} gnn_plan_opts_t;

/* What the plan decided (all integers; bit-exact with the oracle's plan). */
typedef struct {
  int32_t chunk;           /* C*: nnz per work chunk ("NnzPerWarp")    */
  int32_t vw_feat;         /* feature-row vector width VW (elements per lane-vector) */
  int32_t vw_sparse;       /* sparse-array vector width (HVMA): 1, 2 or 4     */
  int32_t lanes;           /* L: lanes per chunk-slice                              */
  int32_t vecs;            /* R: VW-wide vectors per lane per slice (1 or 2)         */
  int32_t slices;          /* S: K-slices per chunk                                 */
  int32_t groups;          /* G = 32 / L chunk-slices per warp                      */
  int32_t warps_per_block;
  int32_t active_blocks_per_sm; /* occupancy API value for the SpMM kernel (Eq. 3)  */
  int32_t num_sms;         /* NumSM (Eq. 4)                                         */
  int32_t alpha;
  int32_t K;
  int32_t feature_dtype;   /* gnn_dtype_t the plan was built for                    */
  int32_t chunk_dtp;       /* the plain-DTP choice before the locality cap           */
  int64_t nnz;
  int64_t num_chunks;      /* ceil(nnz / chunk)                                     */
  int64_t num_blocks;      /* SpMM grid size (integer form of InEq. (5) RHS)         */
  int64_t M;               /* rows of the planned graph (locality cap input)        */
  int64_t l2_bytes;        /* device L2 size the locality cap used (0: cap off)     */
} gnn_plan_info_t;

typedef struct gnn_plan *gnn_plan_t;

/* ---------------------------------------------------------------- plan ---- */
/* Bytes of device workspace gnn_plan_create needs for a graph of M rows and nnz
 * nonzeros at width K with opts on the current device (exact; 0 when nnz == 0).
 * Returns (size_t)-1 on invalid arguments. */
GNN_API size_t gnn_plan_workspace_bytes(int64_t M, int64_t nnz, int32_t K,
                                        const gnn_plan_opts_t *opts);

/* Dynamic Task Partition + Hierarchical Vectorized Memory Access and the
 * per-chunk boundary table of the hybrid-parallel strategy (Algo 3 lines
 * 2-3 P:175-176).  Host part: C* from InEq. (5) over the candidate set
 * {8,32,64,128,256,512}, capped so that the feature rows of the rows in flight fit a
 * quarter of L2 (DESIGN.md §3 step 5b, a B200 addition to DTP), then raised to 64 where
 * InEq. (5) itself chose 8 or 32 (step 5c, B200 addition); no_locality skips 5b and 5c.
 * Scalar integer arithmetic only -- no device read, no sync.
 * Device part: one launch writing, for every chunk c (nnz [c*C*, min((c+1)*C*, nnz))),
 *   row_first[c] = row_ind[start], row_last[c] = row_ind[end-1],
 *   flags[c] = (head row continues from chunk c-1) | (tail row continues into c+1) << 1.
 * workspace: device memory of gnn_plan_workspace_bytes() bytes, 256-byte aligned,
 * owned by the caller; it must outlive every use of the plan.  The plan is bound to
 * (graph arrays, nnz, K, device) and immutable; it may be used concurrently.
 * opts may be NULL (defaults).  *out receives a host handle (free with
 * gnn_plan_destroy). */
GNN_API gnn_status_t gnn_plan_create(const gnn_graph_t *graph, int32_t K,
                                     const gnn_plan_opts_t *opts, void *workspace,
                                     size_t ws_bytes, gnn_stream_t stream, gnn_plan_t *out);
GNN_API gnn_status_t gnn_plan_info(gnn_plan_t plan, gnn_plan_info_t *info);
/* Device views of the plan's per-chunk arrays (inside the workspace). */
GNN_API gnn_status_t gnn_plan_arrays(gnn_plan_t plan, const int32_t **row_first,
                                     const int32_t **row_last, const uint8_t **flags);
GNN_API void gnn_plan_destroy(gnn_plan_t plan);

/* ------------------------------------------------------------- kernels ---- */
/* SpMM, O = S A (Algorithm 1), hybrid-parallel (Algorithm 3
 * P:168-195): O[r - row_base][k] = sum_{i : row_ind[i] = r} val[i] * A[col_ind[i]][k]
 * for every r in [row_base, row_base + M), k in [0, K).  OVERWRITES O (rows without
 * nnz become +0).  A: N x K (lda >= K), O: M x K (ldo >= K), fp32 accumulation.
 * A, O must be 4*vw_feat-byte aligned and lda, ldo multiples of vw_feat, else
 * GNN_ERR_UNSUPPORTED (re-plan with force_vw).  A and O must not overlap.
 * Rows split across chunks are combined with vector atomic adds, so the fp32
 * summation order of such rows is not deterministic (tolerance: DESIGN.md), and the
 * vector atomics flush SUBNORMAL partial sums to zero: for data whose partial sums can be
 * subnormal use a deterministic plan (plain fp32 adds, exact for subnormals). */
GNN_API gnn_status_t gnn_spmm(gnn_plan_t plan, const gnn_graph_t *graph, const float *A,
                              int64_t lda, float *O, int64_t ldo, gnn_stream_t stream);

/* gnn_spmm with bf16 features A (raw bf16 bit patterns, N x K, lda >= K elements;
 * A 2*vw_feat-byte aligned, lda a multiple of vw_feat), fp32 accumulation, fp32 O.
 * The plan must have been built with feature_dtype = GNN_BF16. */
GNN_API gnn_status_t gnn_spmm_bf16(gnn_plan_t plan, const gnn_graph_t *graph,
                                   const uint16_t *A, int64_t lda, float *O, int64_t ldo,
                                   gnn_stream_t stream);

/* Aggregators of the MPP node-wise op (Eq. 1: "max, min, sum"), f_n = v * X_u. */
typedef enum { GNN_AGG_SUM = 0, GNN_AGG_MEAN = 1, GNN_AGG_MAX = 2, GNN_AGG_MIN = 3 } gnn_agg_t;

/* Generalised SpMM: O[r] = (+)_{i : row_ind[i] = r} val[i] * A[col_ind[i]]
 * with (+) = sum, mean (sum / number of nonzeros of the row; needs graph->row_ptr), max or
 * min (elementwise over the row's terms); rows without nonzeros give 0.  A's element type
 * is the plan's feature_dtype (max / min: fp32 only).  accumulate = 1 (sum only) computes
 * O += S A and leaves rows without nonzeros untouched (beta = 1, used to sum partial
 * products, e.g. per column block).  Other rules as gnn_spmm. */
GNN_API gnn_status_t gnn_spmm_ex(gnn_plan_t plan, const gnn_graph_t *graph, const void *A,
                                 int64_t lda, float *O, int64_t ldo, int32_t agg,
                                 int32_t accumulate, gnn_stream_t stream);

/* Backward of gnn_spmm_ex with agg = GNN_AGG_MAX / GNN_AGG_MIN (fp32).  The forward keeps,
 * for every (r, k), exactly one fp32 product fl(val[i] * A[col_ind[i]][k]); the gradient
 * of O[r][k] flows to the FIRST nonzero i of row r (storage order) whose product equals
 * O[r][k] (recomputed in the same fp32 arithmetic, so it is the term the forward kept;
 * ties, e.g. zeros of a ReLU'd input, go to the first):
 *   dA[col_ind[i]][k] += val[i] * dO[r][k]      dval[i] += A[col_ind[i]][k] * dO[r][k]
 * ACCUMULATES into dA (N x K, pitch ldda) and, if dval is non-NULL, into dval (nnz, in
 * col_ind order): zero them first for a plain gradient.  Needs graph->row_ptr (read
 * relative to row_ptr[0]); O is the forward's output (M x K, pitch ldo), dO the incoming
 * gradient (M x K, pitch lddo).  val NULL means all ones.  Float atomics make dA / dval
 * order-dependent within fp32 rounding.  Device pointers; asynchronous on `stream`. */
GNN_API gnn_status_t gnn_spmm_extremum_backward(const gnn_graph_t *graph, int32_t agg, int32_t K,
                                                const float *A, int64_t lda, const float *O,
                                                int64_t ldo, const float *dO, int64_t lddo,
                                                float *dA, int64_t ldda, float *dval,
                                                gnn_stream_t stream);

/* SDDMM, S_O = (A1 A2) (.) S (Algorithm 2), hybrid-parallel
 * (Algorithm 4): out[i] = val[i] * sum_k A1[row_ind[i] - row_base][k] *
 * A2T[col_ind[i]][k] for i in [0, nnz).  A1: M x K (destination rows, lda1 >= K);
 * A2T: N x K, the transpose of Table I's K x N A2 (source rows, lda2 >= K);
 * out: nnz fp32 in col_ind order, each written exactly once (deterministic).
 * Same alignment rules as gnn_spmm; uses the same plan. */
GNN_API gnn_status_t gnn_sddmm(gnn_plan_t plan, const gnn_graph_t *graph, const float *A1,
                               int64_t lda1, const float *A2T, int64_t lda2, float *out,
                               gnn_stream_t stream);

/* gnn_sddmm with bf16 A1 / A2T (raw bf16 bit patterns), fp32 products and sums, fp32
 * out.  Plan built with feature_dtype = GNN_BF16. */
GNN_API gnn_status_t gnn_sddmm_bf16(gnn_plan_t plan, const gnn_graph_t *graph,
                                    const uint16_t *A1, int64_t lda1, const uint16_t *A2T,
                                    int64_t lda2, float *out, gnn_stream_t stream);

/* -------------------------------------------------------------- shards ---- */
/* nnz-balanced contiguous row shards for P GPUs (HOST arrays; DESIGN.md
 * "Multi-GPU"): t_p = floor(p * nnz / P), bounds[p] = first r with
 * row_ptr[r] - row_ptr[0] >= t_p, bounds[0] = 0, bounds[P] = M (monotone).
 * row_ptr_host: [M+1]; bounds: [P+1]. */
GNN_API gnn_status_t gnn_shard_rows(const int32_t *row_ptr_host, int64_t M, int32_t P,
                                    int64_t *bounds);
/* Equal edge-range shards: bounds[p] = floor(p * nnz / P), [P+1] host array. */
GNN_API gnn_status_t gnn_shard_edges(int64_t nnz, int32_t P, int64_t *bounds);

/* ----------------------------------------------------------- transpose ---- */
/* S^T (N x M) in hybrid CSR/COO on the device, for the backward pass dX = S^T dO
 * (SURVEY §8(f) f3).  Outputs (caller-allocated, device): row_ptr_t[N+1], row_ind_t[nnz]
 * (= columns of S), col_ind_t[nnz] (= rows of S minus row_base), val_t[nnz] (may be NULL;
 * ones when graph->val is NULL), edge_perm[nnz] (may be NULL: original edge id of each
 * transposed entry).  Rows of S^T ascending, then S's rows ascending (stable: duplicates
 * keep their order).  workspace: gnn_transpose_workspace_bytes(nnz) bytes, 256-B aligned. */
GNN_API size_t gnn_transpose_workspace_bytes(int64_t nnz);
GNN_API gnn_status_t gnn_transpose(const gnn_graph_t *graph, void *workspace, size_t ws_bytes,
                                   int32_t *row_ptr_t, int32_t *row_ind_t, int32_t *col_ind_t,
                                   float *val_t, int32_t *edge_perm, gnn_stream_t stream);

/* ------------------------------------------------------------- reorder ---- */
/* Graph Clustering based Reordering (GCR, Fig. 8) -- optional, HOST side,
 * offline (it is not part of the timed kernels, P:323 / P:275).  Louvain community
 * detection (refs [29][30]) on the symmetric square graph given as HOST CSR
 * (row_ptr[n+1], col_ind[nnz]; self-loops ignored), then a hierarchical node order
 * (DESIGN.md §2 item 23).  Outputs perm[old] = new (a bijection of [0,n)), optionally
 * the top-level community of each ORIGINAL node and the modularity of that partition.
 * Zero-initialised option fields take the defaults (3 levels, 20 passes per level,
 * min_gain 1e-6, resolution 1.0).  Single-threaded; deterministic. */
typedef struct {
  int32_t max_levels;
  int32_t max_passes;
  double min_gain;
  double resolution;
  int64_t hub_rows;  /* > 0: the hub_rows nodes of largest degree (ties: smaller id) are
                        placed first, in the community order among themselves, so their
                        feature rows form one contiguous block X[0, hub_rows) (DESIGN.md §5:
                        measured on C5 with and without an L2 evict_last hint on that block:
                        no gain; kept for experiments) */
} gnn_reorder_opts_t;
GNN_API gnn_status_t gnn_reorder_gcr(const int32_t *row_ptr_host, const int32_t *col_ind_host,
                                     int64_t n, const gnn_reorder_opts_t *opts,
                                     int32_t *perm_host, int32_t *comm_host,
                                     double *modularity);
/* Apply a node permutation to a square hybrid CSR/COO (HOST arrays): S' = P S P^T with
 * new row perm[r] holding new columns perm[c] sorted ascending (ties keep the original
 * order), values carried along; row_ind_out (the decoded RowInd) may be NULL,
 * val/val_out may be NULL.  Output arrays are caller-allocated (n+1 / nnz entries). */
GNN_API gnn_status_t gnn_permute_graph(const int32_t *row_ptr_host, const int32_t *col_ind_host,
                                       const float *val_host, int64_t n, const int32_t *perm_host,
                                       int32_t *row_ptr_out, int32_t *row_ind_out,
                                       int32_t *col_ind_out, float *val_out);
/* Permute dense rows on the device: Y[perm[i]][:K] = X[i][:K] for i in [0, n) (X' = P X,
 * so SpMM(P S P^T, P X) = P SpMM(S, X)).  perm is a DEVICE array; X and Y must not
 * overlap. */
GNN_API gnn_status_t gnn_permute_rows(const float *X, int64_t ldx, int64_t n, int64_t K,
                                      const int32_t *perm, float *Y, int64_t ldy,
                                      gnn_stream_t stream);

/* ------------------------------------------------------------ end to end ---- */
/* The whole path on HOST buffers (bench.py's "e2e" number): copies the hybrid CSR/COO
 * arrays (if upload_graph) and X from host memory into the caller's device workspace,
 * builds the plan (GPU plan kernel), runs SpMM (O = S X, if O_host) and SDDMM
 * (S_O[i] = v_i <X_r, X_c>, i.e. A1 = A2T = X, if out_host), and copies O (M x K, pitch K)
 * and S_O (nnz) back.  Everything is enqueued asynchronously and the call returns without
 * waiting; `stream` is ordered after every copy of the call, so synchronise it before
 * reading O_host / out_host or reusing X_host (pinned host memory gives asynchronous DMA;
 * pageable memory works but copies synchronously).  Internally the nonzeros are cut into
 * pieces (about one per 4 Mi nonzeros, at most 32; env GNN_HOST_PIECES overrides): the
 * graph uploads piece by piece on a copy-in stream (RowInd/ColInd/Value of the piece plus
 * the next piece's first RowInd entry), each piece is planned as it lands (the plan
 * kernel over the chunks that end inside it, then the pre-zero of its split rows, on a
 * prep stream in piece order), earlier pieces compute (alternating between `stream` and a
 * second compute stream) and finished O rows / S_O values download on a copy-out stream,
 * so the call costs about max(upload, compute, download) instead of their sum.
 * Deterministic plans run as one piece.  Reads the host row_ind to find the rows each
 * piece completes.  GNN_HOST_TRACE=1 prints a per-piece timeline to stderr (synchronises;
 * a measurement aid).
 * graph_host: host pointers, a square N-node graph or a row shard of one (rows
 * [row_base, row_base + M) with row_base + M <= N; SDDMM then uses A1 = those rows of X, O
 * holds the shard's M rows).  If graph_host->row_ptr is given ([M+1], read relative to
 * row_ptr[0], consistent with row_ind), each piece uploads the CSR offsets of the rows it
 * spans instead of its RowInd, which is decoded on the device (4 B per nonzero less over
 * PCIe; row_ind is still read on the host for the piece bookkeeping).  fp32 only.
 * upload_graph = 0 reuses the graph already in this workspace from an earlier call (the
 * graph's offsets do not depend on K, so one workspace sized for the largest K serves all).
 * workspace: gnn_run_host_workspace_bytes(M, N, nnz, K, opts) bytes, 256-B aligned, device. */
GNN_API size_t gnn_run_host_workspace_bytes(int64_t M, int64_t N, int64_t nnz, int32_t K,
                                            const gnn_plan_opts_t *opts);
GNN_API gnn_status_t gnn_run_host(const gnn_graph_t *graph_host, int32_t upload_graph,
                                  const float *X_host, int32_t K, float *O_host,
                                  float *out_host, const gnn_plan_opts_t *opts, void *workspace,
                                  size_t ws_bytes, gnn_stream_t stream);

/* gnn_run_host for nk feature widths K[0..nk) on one graph in ONE pipelined call
 * (1 <= nk <= 16): X_host[k] (N x K[k]), O_host[k] (M x K[k], or O_host / O_host[k] NULL
 * to skip that SpMM), out_host[k] (nnz, or NULL to skip that SDDMM).  Copy-in order:
 * the narrower widths' X interleaved with the first pieces (narrowest first), the widest
 * width's X half-way (env GNN_HOST_WIDE_X_AT = piece index overrides); a width computes every piece that has landed once its X has
 * (catching up on earlier pieces), so downloads start after the first X and piece, and
 * the call costs about max(total upload, total compute, total download).  Each width has its own plan and workspace region, so no width waits for
 * an earlier width's download.  Same ordering, ownership and error rules as gnn_run_host
 * (gnn_run_host is this call with nk = 1).  workspace:
 * gnn_run_host_multi_workspace_bytes(M, N, nnz, nk, K, opts) bytes ((size_t)-1 on
 * invalid arguments), 256-B aligned, device. */
GNN_API size_t gnn_run_host_multi_workspace_bytes(int64_t M, int64_t N, int64_t nnz, int32_t nk,
                                                  const int32_t *K, const gnn_plan_opts_t *opts);
GNN_API gnn_status_t gnn_run_host_multi(const gnn_graph_t *graph_host, int32_t upload_graph,
                                        int32_t nk, const int32_t *K,
                                        const float *const *X_host, float *const *O_host,
                                        float *const *out_host, const gnn_plan_opts_t *opts,
                                        void *workspace, size_t ws_bytes, gnn_stream_t stream);

/* One message-passing step on DEVICE data in one call (BJ configs[2]: a new sampled
 * subgraph every step, re-planned every step): the host half of gnn_plan_create (DTP:
 * C* and the launch shape, no sync), then O = S X (gnn_spmm, if O) and
 * out[i] = val[i] <X[row_i], X[col_i]> (gnn_sddmm with A1 = the graph's rows of X, i.e.
 * X + row_base * ldx, A2T = X, if out).  The per-chunk boundary table the plan kernel
 * would write (row_first / row_last / flags, Algo 3 lines 2-3) is recomputed
 * from row_ind inside the kernels instead, so no plan kernel runs and `workspace`'s
 * plan arrays are NOT written (deterministic plans excepted: they run the plan kernel
 * for their fix-up pass).  The SDDMM runs on a per-thread side stream forked from
 * `stream` and joined back, so the two kernels overlap; the SpMM is a programmatic
 * dependent launch of its split-row pre-zero.  `stream` is ordered after both.
 * workspace: gnn_plan_workspace_bytes bytes.  fp32; same alignment and error rules as
 * gnn_spmm / gnn_sddmm.  Device pointers. */
GNN_API gnn_status_t gnn_plan_spmm_sddmm(const gnn_graph_t *graph, int32_t K,
                                         const gnn_plan_opts_t *opts, const float *X,
                                         int64_t ldx, float *O, int64_t ldo, float *out,
                                         void *workspace, size_t ws_bytes,
                                         gnn_stream_t stream);

/* ----------------------------------------------------------- measurement --- */
/* Roofline probe (not part of the method): gathers rows X[idx[i]][0:K] for i in [0, n)
 * with the same 256-bit row loads the kernels use and no other work (sums are folded
 * into *sink so the loads are live).  Timing it on an L1-, L2- or HBM-resident X gives
 * the on-chip / off-chip gather ceilings bench.py reports beside the HBM roofline.
 * K in {32, 64, 128, 256}; X 32-byte aligned with ld % 8 == 0; idx in [0, rows). */
GNN_API gnn_status_t gnn_probe_gather(const float *X, int64_t ld, const int32_t *idx, int64_t n,
                                      int32_t K, float *sink, gnn_stream_t stream);
/* The same pure gather in the kernels' traversal order: one lane group (K/8 lanes, 8 fp32
 * per lane) per `chunk` consecutive entries of idx, one group per chunk over the whole
 * grid of 4-warp blocks (as gnn_spmm / gnn_sddmm launch a plan of chunk size C*), so the
 * rows in flight -- and the L2 hit rate on a workload's own index stream -- are the
 * kernels'.  Same argument rules as gnn_probe_gather; chunk >= 1. */
GNN_API gnn_status_t gnn_probe_gather_chunked(const float *X, int64_t ld, const int32_t *idx,
                                              int64_t n, int32_t K, int32_t chunk, float *sink,
                                              gnn_stream_t stream);

/* Split a (row-shard) hybrid CSR/COO by the owner of each column, for overlapping the
 * X all-gather with SpMM: column c belongs to block c / blk, P blocks.
 * HOST arrays.  The nonzeros are stably partitioned by block (so every block is again a
 * hybrid CSR/COO with non-decreasing rows): block q occupies
 * [bounds[q], bounds[q+1]) of row_ind_out / col_ind_out / val_out (val may be NULL).
 * Columns keep their global ids.  bounds: [P+1]. */
GNN_API gnn_status_t gnn_split_col_blocks(const int32_t *row_ind_host, const int32_t *col_ind_host,
                                          const float *val_host, int64_t nnz, int32_t P,
                                          int64_t blk, int32_t *row_ind_out,
                                          int32_t *col_ind_out, float *val_out,
                                          int64_t *bounds);

/* --------------------------------------------------------- autograd helpers -- */
/* dst[i] = src[idx[i]] for i in [0, n) (device arrays): the edge values of S^T in the
 * transposed order (idx = gnn_transpose's edge_perm) for the backward dX = S^T dO with
 * trainable edge values. */
GNN_API gnn_status_t gnn_gather_f32(const float *src, const int32_t *idx, int64_t n, float *dst,
                                    gnn_stream_t stream);
/* Y[r][0:K] = X[r][0:K] / max(1, row_ptr[r+1] - row_ptr[r]) for r in [0, M) (device; Y may
 * be X): the backward of the mean aggregator, dX = S^T (dO / deg) (Eq. 1 with (+) = mean,
 * P:23-31; rows without nonzeros carry no gradient). */
GNN_API gnn_status_t gnn_scale_rows_inv_degree(const int32_t *row_ptr, int64_t M, int32_t K,
                                               const float *X, int64_t ldx, float *Y,
                                               int64_t ldy, gnn_stream_t stream);

/* ------------------------------------------------------------- helpers ---- */
/* Decode CSR offsets into the hybrid format's RowInd (Fig. 2d):
 * row_ind[i - row_ptr[0]] = r + row_base for row_ptr[r] <= i < row_ptr[r+1]. */
GNN_API gnn_status_t gnn_csr_to_coo(const int32_t *row_ptr, int64_t M, int64_t row_base,
                                    int32_t *row_ind, gnn_stream_t stream);
/* Debug check of a graph's contents (row_ind non-decreasing and in range, col_ind
 * in [0,N), row_ptr consistent when given).  SYNCHRONISES the stream.  Returns
 * GNN_OK or GNN_ERR_INPUT_CHECK (message in gnn_last_error()). */
GNN_API gnn_status_t gnn_validate(const gnn_graph_t *graph, gnn_stream_t stream);
/* Thread-local description of the last failure on this thread ("" if none). */
GNN_API const char *gnn_last_error(void);
/* Library version string. */
GNN_API const char *gnn_version(void);

#ifdef __cplusplus
}
#endif
#endif /* GNN_SPARSE_H */
