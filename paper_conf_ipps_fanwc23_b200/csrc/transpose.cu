// transpose.cu -- S^T in hybrid CSR/COO on the device (the backward
// pass of SpMM is dX = S^T dO, an SpMM on the transposed graph).
//
// One stable radix sort of (col << bits(M) | local row) keys carrying the edge ids
// (CUB, part of the CUDA toolkit), then an unpack kernel and a lower-bound kernel for the
// row offsets.  Deterministic: duplicates keep their original order.
#include <cub/device/device_radix_sort.cuh>

#include "internal.cuh"

namespace gnn {
namespace {

inline size_t align256(size_t b) { return (b + 255) & ~size_t(255); }

// key = col << rb | local row (rb = bits of M): one radix pass per 8 key bits used
__global__ void make_keys_kernel(const int32_t *__restrict__ row_ind,
                                 const int32_t *__restrict__ col_ind, int64_t nnz,
                                 int64_t row_base, int rb, uint64_t *__restrict__ keys,
                                 int32_t *__restrict__ ids) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nnz; i += stride) {
    keys[i] = ((uint64_t)(uint32_t)col_ind[i] << rb) | (uint64_t)(uint32_t)(row_ind[i] - row_base);
    ids[i] = (int32_t)i;
  }
}

__global__ void unpack_kernel(const uint64_t *__restrict__ keys, const int32_t *__restrict__ ids,
                              int64_t nnz, int rb, const float *__restrict__ val,
                              int32_t *__restrict__ row_ind_t, int32_t *__restrict__ col_ind_t,
                              float *__restrict__ val_t, int32_t *__restrict__ perm) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < nnz; j += stride) {
    const uint64_t k = keys[j];
    row_ind_t[j] = (int32_t)(k >> rb);
    col_ind_t[j] = (int32_t)(k & ((uint64_t(1) << rb) - 1));
    const int32_t id = ids[j];
    if (val_t) val_t[j] = val ? val[id] : 1.0f;
    if (perm) perm[j] = id;
  }
}

// row_ptr_t[c] = first j with row_ind_t[j] >= c, for c in [0, N]
__global__ void offsets_kernel(const int32_t *__restrict__ row_ind_t, int64_t nnz, int64_t N,
                               int32_t *__restrict__ row_ptr_t) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c <= N; c += stride) {
    int64_t lo = 0, hi = nnz;
    while (lo < hi) {
      const int64_t mid = (lo + hi) >> 1;
      if (row_ind_t[mid] < c) lo = mid + 1;
      else hi = mid;
    }
    row_ptr_t[c] = (int32_t)lo;
  }
}

size_t cub_temp_bytes(int64_t nnz) {
  size_t t = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, t, (uint64_t *)nullptr, (uint64_t *)nullptr,
                                  (int32_t *)nullptr, (int32_t *)nullptr, (int)nnz, 0, 64);
  return t;
}

}  // namespace
}  // namespace gnn

using namespace gnn;

extern "C" {

GNN_API size_t gnn_transpose_workspace_bytes(int64_t nnz) {
  if (nnz < 0 || nnz >= (int64_t(1) << 31)) return (size_t)-1;
  if (nnz == 0) return 0;
  return 2 * align256(sizeof(uint64_t) * nnz) + 2 * align256(sizeof(int32_t) * nnz) +
         align256(cub_temp_bytes(nnz));
}

GNN_API gnn_status_t gnn_transpose(const gnn_graph_t *g, void *workspace, size_t ws_bytes,
                                   int32_t *row_ptr_t, int32_t *row_ind_t, int32_t *col_ind_t,
                                   float *val_t, int32_t *edge_perm, gnn_stream_t stream) {
  if (!g || g->M < 0 || g->N < 0 || g->nnz < 0 || !row_ptr_t ||
      (g->nnz > 0 && (!g->row_ind || !g->col_ind || !row_ind_t || !col_ind_t)))
    return fail(GNN_ERR_INVALID_ARG, "gnn_transpose: bad arguments");
  if (g->M >= (int64_t(1) << 31) || g->N >= (int64_t(1) << 31) || g->nnz >= (int64_t(1) << 31))
    return fail(GNN_ERR_INVALID_ARG, "gnn_transpose: sizes exceed int32 indices");
  DeviceInfo d;
  if (gnn_status_t st = device_info(&d)) return st;
  cudaStream_t s = (cudaStream_t)stream;
  const int64_t nnz = g->nnz;
  const unsigned grid = (unsigned)d.num_sms * 8;
  if (nnz == 0) {
    cudaError_t e = cudaMemsetAsync(row_ptr_t, 0, sizeof(int32_t) * (g->N + 1), s);
    return e == cudaSuccess ? GNN_OK : cuda_fail(e, "gnn_transpose memset");
  }
  const size_t need = gnn_transpose_workspace_bytes(nnz);
  if (!workspace || ws_bytes < need || !aligned(workspace, 256))
    return fail(GNN_ERR_WORKSPACE, "gnn_transpose: workspace %zu B (need %zu B, 256-B aligned)",
                ws_bytes, need);
  char *w = (char *)workspace;
  uint64_t *k_in = (uint64_t *)w;
  w += align256(sizeof(uint64_t) * nnz);
  uint64_t *k_out = (uint64_t *)w;
  w += align256(sizeof(uint64_t) * nnz);
  int32_t *id_in = (int32_t *)w;
  w += align256(sizeof(int32_t) * nnz);
  int32_t *id_out = (int32_t *)w;
  w += align256(sizeof(int32_t) * nnz);
  size_t temp = cub_temp_bytes(nnz);
  int rb = 1, cb = 1;
  while (rb < 31 && ((int64_t)1 << rb) < g->M) ++rb;
  while (cb < 31 && ((int64_t)1 << cb) < g->N) ++cb;
  make_keys_kernel<<<grid, 256, 0, s>>>(g->row_ind, g->col_ind, nnz, g->row_base, rb, k_in, id_in);
  cudaError_t e = cub::DeviceRadixSort::SortPairs(w, temp, k_in, k_out, id_in, id_out, (int)nnz, 0,
                                                  rb + cb, s);
  if (e != cudaSuccess) return cuda_fail(e, "gnn_transpose sort");
  unpack_kernel<<<grid, 256, 0, s>>>(k_out, id_out, nnz, rb, g->val, row_ind_t, col_ind_t, val_t,
                                     edge_perm);
  offsets_kernel<<<grid, 256, 0, s>>>(row_ind_t, nnz, g->N, row_ptr_t);
  e = cudaGetLastError();
  return e == cudaSuccess ? GNN_OK : cuda_fail(e, "gnn_transpose launch");
}

}  // extern "C"
