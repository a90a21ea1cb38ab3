// sddmm.cu -- hybrid-parallel SDDMM for sm_100a (S_O = (A1 A2) (.) S, P:96;
// Algorithm 2 P:112-131 is the definition, Algorithm 4 P:211-232 the prior-art GPU
// design).
//
// Same plan, chunks and lane groups as SpMM (one hybrid node/edge partition).  A lane
// group owns a whole chunk (all K-slices, so no cross-group reduction is needed).
// Per nonzero i of the chunk: gather the A2T[col_i] slice (U rows in flight per
// lane), multiply with the register-cached A1[row_i] slice -- reloaded only on a row
// switch, the reuse Algorithm 4 lines 8-11 describe -- reduce over the L lanes
// with a transposed butterfly that reduces U nonzeros at once (WarpReduce, line 12),
// scale by val_i after the sum (Algo 2 line 6) and store: the U results of a
// batch land in consecutive lanes, so the store is coalesced; each output is written
// exactly once (plain stores, deterministic).  The sparse entries come from the same
// per-warp cp.async shared-memory ring as SpMM's (one tile ahead of use); tiles whose
// nonzeros all share one row (for every group of the warp) take a fast path with no
// per-nonzero row or bounds logic, and single-slice rows issue the next batch's gathers
// before this batch's butterfly (software pipelining).  SDDMM never reads the plan's
// boundary table, only its chunk size and lane shape.
#include "sddmm_kernel.cuh"

namespace gnn {
// c0 < 0: the whole plan; else chunks [c0, c1) only (the pipelined host path).
gnn_status_t launch_sddmm(const Plan *p, const gnn_graph_t *g, const void *A1, int64_t lda1,
                          const void *A2T, int64_t lda2, float *out, gnn_stream_t stream,
                          int dtype, const char *who, int64_t c0, int64_t c1) {
  if (gnn_status_t st = check_common(p, g, who)) return st;
  const gnn_plan_info_t &in = p->info;
  if (in.feature_dtype != dtype)
    return fail(GNN_ERR_INVALID_ARG, "%s: plan was built for feature_dtype %d", who,
                in.feature_dtype);
  const int K = in.K, VW = in.vw_feat;
  const int ES = dtype == GNN_BF16 ? 2 : 4;
  if (g->nnz == 0) return GNN_OK;
  if (!A1 || !A2T || !out || lda1 < K || lda2 < K || lda2 >= (int64_t(1) << 29))
    return fail(GNN_ERR_INVALID_ARG, "%s: bad dense operand", who);
  if (!aligned(A1, (size_t)ES * VW) || !aligned(A2T, (size_t)ES * VW) || lda1 % VW || lda2 % VW)
    return fail(GNN_ERR_UNSUPPORTED,
                "%s: A1/A2T must be %d-byte aligned with pitches multiple of %d", who, ES * VW,
                VW);
  const int vws = effective_vws(in.vw_sparse, g, out);
  int V = in.lanes * in.vecs;  // vectors per K-slice
  int VWk = VW;
#if GNN_SDDMM_BF16_NARROW
  // bf16 single-slice rows held as two 16-element vectors (K = 32): a 2-lane dot product
  // leaves the butterfly nothing to batch; as four 8-element vectors (4-lane dot
  // products) the kernel measured 0.82 -> 0.69 ms on C4 (profiles/r01_sweep36).  SpMM
  // keeps the plan's 16-wide vectors (faster there).  The plan's alignment check for 16
  // elements covers 8.
  if (dtype == GNN_BF16 && in.slices == 1 && VW == 16 && V == 2) {
    VWk = 8;
    V = 4;
  }
#endif
#if GNN_SDDMM_NARROW_LG8
  // single-slice rows of four 32-byte vectors (fp32 K = 32, bf16 K = 64): a 4-lane dot
  // product takes the unpipelined path; as eight 16-byte vectors (8-lane dot products) the
  // next batch's gathers are issued before this batch's butterfly (run_fast_pipelined)
  if (in.slices == 1 && V == 4 && VWk * ES >= GNN_SDDMM_NARROW_MIN_BYTES) {
    VWk /= 2;
    V = 8;
  }
#endif
  SddmmFn f = dtype == GNN_BF16 ? pick_sddmm_bf16(VWk, V, vws, in.slices)
                                : pick_sddmm_f32(VWk, V, vws, in.slices);
  if (!f)
    return fail(GNN_ERR_UNSUPPORTED, "%s: K=%d needs %d slices (max 4 at vw=%d)", who, K,
                in.slices, VW);
  SparseArgs a = make_args(p, g);
  if (c0 >= 0) {
    if (c1 < c0 || c1 > a.num_chunks)
      return fail(GNN_ERR_INVALID_ARG, "%s: bad chunk range [%lld, %lld)", who, (long long)c0,
                  (long long)c1);
    if (c1 == c0) return GNN_OK;
    a.c_begin = c0;
    a.c_end = c1;
  }
  const int threads = in.warps_per_block * 32;
  const int lg = sddmm_group_lanes(V, in.slices);
  const int64_t per_block = (int64_t)(32 / lg) * in.warps_per_block;
  const int64_t blocks = (a.c_end - a.c_begin + per_block - 1) / per_block;
  const size_t smem = (size_t)in.warps_per_block *
                      sddmm_tile_bytes_per_warp(lg, sddmm_effective_vws(V, in.slices, vws));
  if (smem > 48 * 1024) {
    cudaError_t e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return cuda_fail(e, "gnn_sddmm smem attribute");
  }
  f<<<(unsigned)blocks, threads, smem, (cudaStream_t)stream>>>(a, A1, lda1, A2T, lda2, out);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GNN_OK : cuda_fail(e, "gnn_sddmm launch");
}
}  // namespace gnn

using namespace gnn;

extern "C" GNN_API gnn_status_t gnn_sddmm(gnn_plan_t plan, const gnn_graph_t *g,
                                          const float *A1, int64_t lda1, const float *A2T,
                                          int64_t lda2, float *out, gnn_stream_t stream) {
  return launch_sddmm(reinterpret_cast<const Plan *>(plan), g, A1, lda1, A2T, lda2, out, stream,
                      GNN_F32, "gnn_sddmm", -1, 0);
}

extern "C" GNN_API gnn_status_t gnn_sddmm_bf16(gnn_plan_t plan, const gnn_graph_t *g,
                                               const uint16_t *A1, int64_t lda1,
                                               const uint16_t *A2T, int64_t lda2, float *out,
                                               gnn_stream_t stream) {
  return launch_sddmm(reinterpret_cast<const Plan *>(plan), g, A1, lda1, A2T, lda2, out, stream,
                      GNN_BF16, "gnn_sddmm_bf16", -1, 0);
}
