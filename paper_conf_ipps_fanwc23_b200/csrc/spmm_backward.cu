// spmm_backward.cu -- backward of the max / min aggregators of the node-wise op (Eq. 1,
// (+) in {max, min}).
//
// Forward (gnn_spmm_ex): O[r][k] = (+)_{i : row_i = r} fl(v_i * A[c_i][k]) -- each output is
// exactly one of the fp32 products (fmaxf / fminf), and 0 for rows without nonzeros.
// Backward: the gradient of O[r][k] flows to ONE term, the first nonzero of row r (in
// storage order) whose product equals O[r][k] (a valid subgradient; ties -- e.g. the zeros
// of a ReLU'd input -- are resolved deterministically):
//     dA[c_i][k] += v_i * dO[r][k]        dval[i] += A[c_i][k] * dO[r][k]
// The selection recomputes the forward's products in the same fp32 arithmetic, so it
// picks exactly the term the forward kept.
//
// Layout: one warp per (row, 32-column block); lanes own the block's columns and walk the
// row's nonzeros in order until every lane has found its term (__all_sync early exit).
// A rows gathered per nonzero are coalesced 128-byte loads; the scatter into dA is a
// float atomic (several rows can select the same source row), dval gets one atomic per
// nonzero that any lane selected (warp-reduced first).  This is a backward-only path
// sized for correctness and coalescing, not a DTP-balanced kernel: hub rows serialise on
// one warp per column block.
#include <cuda_runtime.h>

#include "internal.cuh"

namespace gnn {
namespace {

__global__ void __launch_bounds__(256)
    spmm_extremum_backward_kernel(const int32_t *__restrict__ row_ptr, int64_t M,
                                  const int32_t *__restrict__ col_ind,
                                  const float *__restrict__ val, int32_t K,
                                  const float *__restrict__ A, int64_t lda,
                                  const float *__restrict__ O, int64_t ldo,
                                  const float *__restrict__ dO, int64_t lddo,
                                  float *__restrict__ dA, int64_t ldda,
                                  float *__restrict__ dval) {
  const int lane = threadIdx.x & 31;
  const int64_t nkb = (K + 31) / 32;
  const int64_t nwarps = (int64_t)gridDim.x * (blockDim.x >> 5);
  const int32_t base = row_ptr[0];
  for (int64_t w = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); w < M * nkb;
       w += nwarps) {
    const int64_t r = w / nkb;
    const int k = (int)(w - r * nkb) * 32 + lane;
    const int64_t i0 = row_ptr[r] - base, i1 = row_ptr[r + 1] - base;
    bool done = k >= K;
    const float o = done ? 0.f : O[r * ldo + k];
    const float g = done ? 0.f : dO[r * lddo + k];
    for (int64_t i = i0; i < i1; ++i) {
      if (__all_sync(0xffffffffu, done)) break;
      const int32_t c = col_ind[i];
      const float v = val ? val[i] : 1.f;
      float part = 0.f;
      if (!done) {
        const float x = A[(int64_t)c * lda + k];
        if (v * x == o) {  // the forward's product, same fp32 rounding
          done = true;
          atomicAdd(dA + (int64_t)c * ldda + k, v * g);
          part = x * g;
        }
      }
      if (dval) {
        const unsigned hit = __ballot_sync(0xffffffffu, part != 0.f);
        if (hit) {
#pragma unroll
          for (int s = 16; s >= 1; s >>= 1) part += __shfl_xor_sync(0xffffffffu, part, s);
          if (lane == 0) atomicAdd(dval + i, part);
        }
      }
    }
  }
}

}  // namespace
}  // namespace gnn

using namespace gnn;

extern "C" GNN_API gnn_status_t gnn_spmm_extremum_backward(
    const gnn_graph_t *g, int32_t agg, int32_t K, const float *A, int64_t lda, const float *O,
    int64_t ldo, const float *dO, int64_t lddo, float *dA, int64_t ldda, float *dval,
    gnn_stream_t stream) {
  if (!g || g->M < 0 || g->N < 0 || g->nnz < 0 || K < 1 ||
      (agg != GNN_AGG_MAX && agg != GNN_AGG_MIN))
    return fail(GNN_ERR_INVALID_ARG, "gnn_spmm_extremum_backward: bad graph / K / agg %d", agg);
  if (g->M == 0 || g->nnz == 0) return GNN_OK;
  if (!g->row_ptr || !g->col_ind || !A || !O || !dO || !dA || lda < K || ldo < K || lddo < K ||
      ldda < K)
    return fail(GNN_ERR_INVALID_ARG,
                "gnn_spmm_extremum_backward: needs row_ptr, col_ind, A, O, dO, dA with pitches "
                ">= K");
  DeviceInfo d;
  if (gnn_status_t st = device_info(&d)) return st;
  const int64_t warps = g->M * ((K + 31) / 32);
  int64_t blocks = (warps + 7) / 8;
  if (blocks > (int64_t)d.num_sms * 16) blocks = (int64_t)d.num_sms * 16;
  cudaStream_t s = (cudaStream_t)stream;
  const float *val = g->val;  // sub-view starting at the graph's first nonzero
  // max and min select the same way (the term equal to the forward's output)
  spmm_extremum_backward_kernel<<<(unsigned)blocks, 256, 0, s>>>(
      g->row_ptr, g->M, g->col_ind, val, K, A, lda, O, ldo, dO, lddo, dA, ldda, dval);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GNN_OK : cuda_fail(e, "gnn_spmm_extremum_backward launch");
}
