// internal.cuh -- shared internals of libgnnsparse.so (not part of the ABI).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "gnn_sparse.h"

namespace gnn {

// Per-thread error message + status helpers (gnn_last_error()).
gnn_status_t fail(gnn_status_t st, const char *fmt, ...);
gnn_status_t cuda_fail(cudaError_t e, const char *what);
void clear_error();

// Cached per-device properties (queried once per device, no sync).
struct DeviceInfo {
  int device;
  int num_sms;
  int cc_major, cc_minor;
  int64_t l2_bytes;
};
gnn_status_t device_info(DeviceInfo *out);

// The plan handle (host struct; arrays live in the caller's workspace).
struct Plan {
  gnn_plan_info_t info;
  int device;
  const int32_t *row_ind;  // graph arrays the plan was built for
  int32_t *row_first;
  int32_t *row_last;
  uint8_t *flags;
  float *carry;  // deterministic plans: [num_chunks][2][K] split-row partials, else null
  int64_t M;
  int64_t row_base;
  bool inline_plan = false;  // kernels recompute the boundary table (gnn_plan_spmm_sddmm)
};

// Kernel parameter block shared by the SpMM / SDDMM launchers.
struct SparseArgs {
  const int32_t *__restrict__ row_ind;
  const int32_t *__restrict__ col_ind;
  const float *__restrict__ val;  // may be null
  const int32_t *__restrict__ row_first;
  const int32_t *__restrict__ row_last;
  const uint8_t *__restrict__ flags;
  int64_t nnz;
  int64_t num_chunks;
  int64_t row_base;
  int64_t M;
  int32_t chunk;
  int32_t K;
  int32_t slices;
  int32_t vecs;
  int32_t accum;  // 1: O += S A (beta = 1), rows without nonzeros untouched
  float *carry;   // deterministic: split-row partials [chunk][first|last][K] (no atomics)
  int64_t c_begin, c_end;  // chunk range of this launch (default [0, num_chunks)); the
                           // pipelined host path launches a plan piece by piece
  int32_t inline_plan;     // 1: no plan arrays -- each chunk derives its boundary rows and
                           // flags from row_ind (the plan kernel's arithmetic) itself
};

#ifdef __CUDACC__
// Boundary rows and continuation flags of chunk c (Algo 3 lines 2-3): from the
// plan arrays, or -- inline plans -- recomputed from row_ind exactly as plan_kernel does.
__device__ __forceinline__ void chunk_rows(const SparseArgs &a, int64_t c, int32_t &rf,
                                           int32_t &rl, uint32_t &fl) {
  if (a.inline_plan) {
    const int64_t s = c * a.chunk;
    const int64_t e = s + a.chunk < a.nnz ? s + a.chunk : a.nnz;
    rf = __ldg(a.row_ind + s);
    rl = __ldg(a.row_ind + e - 1);
    fl = (s > 0 && __ldg(a.row_ind + s - 1) == rf ? 1u : 0u) |
         (e < a.nnz && __ldg(a.row_ind + e) == rl ? 2u : 0u);
  } else {
    rf = a.row_first[c];
    rl = a.row_last[c];
    fl = a.flags[c];
  }
}
// last row of chunk c - 1 (c > 0)
__device__ __forceinline__ int32_t prev_chunk_last_row(const SparseArgs &a, int64_t c) {
  return a.inline_plan ? __ldg(a.row_ind + c * a.chunk - 1) : a.row_last[c - 1];
}
#endif

// Occupancy (active blocks / SM) of the SpMM kernel for a feature width/lane count;
// DTP's ActiveblocksPerSM (Eq. 3) -- defined in spmm.cu.
int spmm_active_blocks_per_sm(int dtype, int vw, int lanes, int vecs, int warps_per_block);

// Shared launcher helpers (spmm.cu).
gnn_status_t check_common(const Plan *p, const gnn_graph_t *g, const char *who);
int effective_vws(int vws, const gnn_graph_t *g, const void *extra);
SparseArgs make_args(const Plan *p, const gnn_graph_t *g);

// Launchers (spmm.cu / sddmm.cu); c0 < 0 = every chunk of the plan, else chunks [c0, c1).
gnn_status_t launch_spmm(const Plan *p, const gnn_graph_t *g, const void *A, int64_t lda,
                         float *O, int64_t ldo, gnn_stream_t stream, int dtype, int agg_api,
                         int accumulate, const char *who, int64_t c0, int64_t c1);
// Pre-zero of the rows split across chunks, for the chunks [c0, c1) (c0 < 0: all).
gnn_status_t launch_spmm_prezero(const Plan *p, const gnn_graph_t *g, float *O, int64_t ldo,
                                 gnn_stream_t stream, int64_t c0 = -1, int64_t c1 = 0);
// gnn_plan_create with launch = false: the host half only (C*, info, workspace views);
// the caller fills the plan arrays with launch_plan_range as the row array arrives.
gnn_status_t plan_create(const gnn_graph_t *g, int32_t K, const gnn_plan_opts_t *opts,
                         void *workspace, size_t ws_bytes, gnn_stream_t stream, gnn_plan_t *out,
                         bool launch);
gnn_status_t launch_plan_range(const Plan *p, gnn_stream_t stream, int64_t c0, int64_t c1);
// The one-call step as one launch (step_fused.cu); GNN_ERR_UNSUPPORTED = no fused instance
// for this shape (nothing launched).
gnn_status_t launch_step_fused(const Plan *p, const gnn_graph_t *g, const float *X,
                               int64_t ldx, float *O, int64_t ldo, float *out,
                               gnn_stream_t stream);
gnn_status_t launch_sddmm(const Plan *p, const gnn_graph_t *g, const void *A1, int64_t lda1,
                          const void *A2T, int64_t lda2, float *out, gnn_stream_t stream,
                          int dtype, const char *who, int64_t c0, int64_t c1);

// Valid warps_per_block range; block size = 32 * wpb <= kMaxThreads.
constexpr int kMaxThreads = 512;

inline bool aligned(const void *p, size_t a) { return (reinterpret_cast<uintptr_t>(p) % a) == 0; }

}  // namespace gnn
