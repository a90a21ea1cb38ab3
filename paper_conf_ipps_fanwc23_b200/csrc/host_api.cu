// host_api.cu -- the end-to-end entry point on HOST buffers (bench.py's e2e path): the
// caller hands host arrays and one device workspace; the library copies the graph and X
// in, plans (GPU plan kernel), runs SpMM and SDDMM, and copies O and S_O out, all
// asynchronously on one stream.
#include <cuda_runtime.h>

#include "internal.cuh"

namespace gnn {
namespace {
inline size_t a256(size_t b) { return (b + 255) & ~size_t(255); }

struct HostLayout {  // offsets inside the workspace; the graph part does not depend on K
  size_t row_ind, col_ind, val, X, O, out, plan, total;
};

HostLayout layout(int64_t M, int64_t N, int64_t nnz, int32_t K, size_t plan_bytes) {
  HostLayout l{};
  size_t o = 0;
  l.row_ind = o; o += a256(4 * (size_t)nnz);
  l.col_ind = o; o += a256(4 * (size_t)nnz);
  l.val = o;     o += a256(4 * (size_t)nnz);
  l.X = o;       o += a256(4 * (size_t)N * K);
  l.O = o;       o += a256(4 * (size_t)M * K);
  l.out = o;     o += a256(4 * (size_t)nnz);
  l.plan = o;    o += a256(plan_bytes);
  l.total = o;
  return l;
}
}  // namespace
}  // namespace gnn

using namespace gnn;

extern "C" {

GNN_API size_t gnn_run_host_workspace_bytes(int64_t M, int64_t N, int64_t nnz, int32_t K,
                                            const gnn_plan_opts_t *opts) {
  if (M < 0 || N < 0 || nnz < 0 || K < 1) return (size_t)-1;
  const size_t pb = gnn_plan_workspace_bytes(nnz, K, opts);
  if (pb == (size_t)-1) return (size_t)-1;
  return layout(M, N, nnz, K, pb).total;
}

GNN_API gnn_status_t gnn_run_host(const gnn_graph_t *gh, int32_t upload_graph, const float *X_host,
                                  int32_t K, float *O_host, float *out_host,
                                  const gnn_plan_opts_t *opts, void *workspace, size_t ws_bytes,
                                  gnn_stream_t stream) {
  if (!gh || gh->M < 0 || gh->N < 0 || gh->nnz < 0 || K < 1 || !X_host || gh->M != gh->N ||
      gh->row_base != 0 || (gh->nnz > 0 && (!gh->row_ind || !gh->col_ind)))
    return fail(GNN_ERR_INVALID_ARG,
                "gnn_run_host: bad arguments (square graph with host arrays, K >= 1)");
  if (opts && opts->feature_dtype != GNN_F32)
    return fail(GNN_ERR_UNSUPPORTED, "gnn_run_host: fp32 features only");
  const size_t pb = gnn_plan_workspace_bytes(gh->nnz, K, opts);
  if (pb == (size_t)-1) return fail(GNN_ERR_INVALID_ARG, "gnn_run_host: %s", gnn_last_error());
  const HostLayout l = layout(gh->M, gh->N, gh->nnz, K, pb);
  if (!workspace || ws_bytes < l.total || !aligned(workspace, 256))
    return fail(GNN_ERR_WORKSPACE, "gnn_run_host: workspace %zu B (need %zu B, 256-B aligned)",
                ws_bytes, l.total);
  char *w = (char *)workspace;
  cudaStream_t s = (cudaStream_t)stream;
  const int64_t nnz = gh->nnz, M = gh->M, N = gh->N;
  cudaError_t e = cudaSuccess;
  if (upload_graph && nnz > 0) {
    e = cudaMemcpyAsync(w + l.row_ind, gh->row_ind, 4 * nnz, cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess)
      e = cudaMemcpyAsync(w + l.col_ind, gh->col_ind, 4 * nnz, cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess && gh->val)
      e = cudaMemcpyAsync(w + l.val, gh->val, 4 * nnz, cudaMemcpyHostToDevice, s);
    if (e != cudaSuccess) return cuda_fail(e, "gnn_run_host graph upload");
  }
  if (N > 0) {
    e = cudaMemcpyAsync(w + l.X, X_host, 4 * (size_t)N * K, cudaMemcpyHostToDevice, s);
    if (e != cudaSuccess) return cuda_fail(e, "gnn_run_host X upload");
  }
  gnn_graph_t gd = *gh;
  gd.row_ptr = nullptr;
  gd.row_ind = (const int32_t *)(w + l.row_ind);
  gd.col_ind = (const int32_t *)(w + l.col_ind);
  gd.val = gh->val ? (const float *)(w + l.val) : nullptr;
  gnn_plan_t plan = nullptr;
  if (gnn_status_t st = gnn_plan_create(&gd, K, opts, w + l.plan, pb, stream, &plan)) return st;
  const float *X = (const float *)(w + l.X);
  gnn_status_t st = GNN_OK;
  if (O_host) {
    st = gnn_spmm(plan, &gd, X, K, (float *)(w + l.O), K, stream);
    if (st == GNN_OK && M > 0) {
      e = cudaMemcpyAsync(O_host, w + l.O, 4 * (size_t)M * K, cudaMemcpyDeviceToHost, s);
      if (e != cudaSuccess) st = cuda_fail(e, "gnn_run_host O download");
    }
  }
  if (st == GNN_OK && out_host) {
    st = gnn_sddmm(plan, &gd, X, K, X, K, (float *)(w + l.out), stream);
    if (st == GNN_OK && nnz > 0) {
      e = cudaMemcpyAsync(out_host, w + l.out, 4 * (size_t)nnz, cudaMemcpyDeviceToHost, s);
      if (e != cudaSuccess) st = cuda_fail(e, "gnn_run_host S_O download");
    }
  }
  gnn_plan_destroy(plan);
  return st;
}

}  // extern "C"
