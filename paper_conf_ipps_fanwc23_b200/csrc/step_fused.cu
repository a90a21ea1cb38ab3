// step_fused.cu -- the one-call message-passing step (gnn_plan_spmm_sddmm, BJ configs[2]:
// a new sampled subgraph and a new plan every step) as ONE kernel launch: blocks
// [0, nb_spmm) run the SpMM body (O = S X, Algorithm 1, hybrid-parallel per
// Algorithm 3) and blocks [nb_spmm, nb_spmm + nb_sddmm) the SDDMM body (out = v <X_r, X_c>,
// Algorithm 2 P:112-131 / Algorithm 4) over the same plan's chunks.  On the 1-3-wave
// graphs of graph sampling one grid has one launch latency and one tail instead of two
// kernels on two streams joined by events.  The launch is a programmatic dependent of the
// split-row pre-zero: SDDMM blocks never wait for it, SpMM blocks wait only before their
// first atomic flush (spmm_body).  Boundary rows are recomputed in-kernel (inline plan).
// fp32, VW = 8, K in {32, 64, 128, 256}; other shapes use the two-kernel path.
#include "sddmm_kernel.cuh"
#include "spmm_kernel.cuh"

namespace gnn {
namespace {

// K8 = K / 8: SpMM lanes per group (rows of one 256-bit vector per lane, after the
// widen remap) and SDDMM vectors per slice.
#ifndef GNN_STEP_FUSED_REGS
#define GNN_STEP_FUSED_REGS 128
#endif
template <int K8, int VWS_SP, int VWS_SD>
__global__ void __maxnreg__(GNN_STEP_FUSED_REGS)
    step_fused_kernel(const SparseArgs a, const float *__restrict__ X, const int64_t ldx,
                      const float *__restrict__ A1, float *__restrict__ O, const int64_t ldo,
                      float *__restrict__ out, const int64_t nb_spmm) {
  if ((int64_t)blockIdx.x < nb_spmm)
    spmm_body<F32, 8, K8, 1, VWS_SP, kAggSum>(a, X, ldx, O, ldo, blockIdx.x);
  else
    sddmm_body<F32, 8, K8, VWS_SD, 1>(a, A1, ldx, X, ldx, out, (int64_t)blockIdx.x - nb_spmm);
}

using StepFn = void (*)(const SparseArgs, const float *__restrict__, const int64_t,
                        const float *__restrict__, float *__restrict__, const int64_t,
                        float *__restrict__, const int64_t);

template <int K8, int VWS_SP>
StepFn pick_sd(int vws_sd) {
  switch (vws_sd) {
    case 2: return step_fused_kernel<K8, VWS_SP, 2>;
    case 4: return step_fused_kernel<K8, VWS_SP, 4>;
  }
  return nullptr;
}
template <int K8>
StepFn pick_sp(int vws_sp, int vws_sd) {
  switch (vws_sp) {
    case 2: return pick_sd<K8, 2>(vws_sd);
    case 4: return pick_sd<K8, 4>(vws_sd);
  }
  return nullptr;
}
StepFn pick_step(int K, int vws_sp, int vws_sd) {
  switch (K) {
    case 32: return pick_sp<4>(vws_sp, vws_sd);
    case 64: return pick_sp<8>(vws_sp, vws_sd);
    case 128: return pick_sp<16>(vws_sp, vws_sd);
    case 256: return pick_sp<32>(vws_sp, vws_sd);
  }
  return nullptr;
}

}  // namespace

// Returns GNN_ERR_UNSUPPORTED (nothing launched) when the shape has no fused instance;
// the caller then runs the two-kernel path.
gnn_status_t launch_step_fused(const Plan *p, const gnn_graph_t *g, const float *X,
                               int64_t ldx, float *O, int64_t ldo, float *out,
                               gnn_stream_t stream) {
  const gnn_plan_info_t &in = p->info;
  const int K = in.K;
  if (!p->inline_plan || in.feature_dtype != GNN_F32 || in.vw_feat != 8 || in.slices != 1 ||
      in.lanes * in.vecs != K / 8 || g->nnz == 0 || !X || !O || !out || ldx < K || ldo < K ||
      ldx >= (int64_t(1) << 29) || !aligned(X, 32) || ldx % 8 || !aligned(O, 32) || ldo % 8 ||
      !aligned(X + g->row_base * ldx, 32))
    return GNN_ERR_UNSUPPORTED;
  if (gnn_status_t st = check_common(p, g, "gnn_plan_spmm_sddmm (fused)")) return st;
  // sparse vector widths as the two launchers pick them
  int vws_sp = effective_vws(in.vw_sparse, g, nullptr);
  if (in.vecs == 2 && vws_sp > 2) vws_sp = 2;  // widened rows: 2-wide sparse copies
  const int vws_sd = sddmm_effective_vws(K / 8, 1, effective_vws(in.vw_sparse, g, out));
  StepFn f = pick_step(K, vws_sp, vws_sd);
  if (!f) return GNN_ERR_UNSUPPORTED;
  SparseArgs a = make_args(p, g);
  const int wpb = in.warps_per_block;
  const int64_t per_sp = (int64_t)(32 / (K / 8)) * wpb;  // SpMM work items per block
  const int lg = sddmm_group_lanes(K / 8, 1);
  const int64_t per_sd = (int64_t)(32 / lg) * wpb;       // SDDMM chunks per block
  const int64_t nb_sp = (a.num_chunks + per_sp - 1) / per_sp;
  const int64_t nb_sd = (a.num_chunks + per_sd - 1) / per_sd;
  const int b_sp = spmm_tile_bytes_per_warp(K / 8, vws_sp);
  const int b_sd = sddmm_tile_bytes_per_warp(lg, vws_sd);
  const size_t smem = (size_t)wpb * (b_sp > b_sd ? b_sp : b_sd);
  cudaStream_t s = (cudaStream_t)stream;
  if (gnn_status_t st = launch_spmm_prezero(p, g, O, ldo, stream)) return st;
  if (smem > 48 * 1024) {
    cudaError_t e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return cuda_fail(e, "fused step smem attribute");
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(nb_sp + nb_sd));
  cfg.blockDim = dim3(wpb * 32);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  const float *A1 = X + g->row_base * ldx;  // the graph's own rows of X
  cudaError_t e = cudaLaunchKernelEx(&cfg, f, a, X, ldx, A1, O, ldo, out, nb_sp);
  return e == cudaSuccess ? GNN_OK : cuda_fail(e, "fused step launch");
}

}  // namespace gnn
