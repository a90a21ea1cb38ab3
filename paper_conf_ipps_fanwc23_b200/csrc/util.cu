// util.cu -- errors, device info, shards, CSR->COO, validation (C ABI).
#include <cuda_runtime.h>
#include <stdarg.h>
#include <stdio.h>
#include <string.h>

#include <mutex>

#include "internal.cuh"

namespace gnn {

static thread_local char g_err[512] = "";

gnn_status_t fail(gnn_status_t st, const char *fmt, ...) {
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(g_err, sizeof(g_err), fmt, ap);
  va_end(ap);
  return st;
}

gnn_status_t cuda_fail(cudaError_t e, const char *what) {
  return fail(GNN_ERR_CUDA, "%s: %s (%s)", what, cudaGetErrorName(e), cudaGetErrorString(e));
}

void clear_error() { g_err[0] = '\0'; }

gnn_status_t device_info(DeviceInfo *out) {
  static std::mutex mu;
  static DeviceInfo cache[64];
  static bool have[64] = {false};
  int dev = -1;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return cuda_fail(e, "cudaGetDevice (no usable CUDA device)");
  if (dev < 0 || dev >= 64) return fail(GNN_ERR_CUDA, "device ordinal %d out of range", dev);
  std::lock_guard<std::mutex> lk(mu);
  if (!have[dev]) {
    DeviceInfo d{};
    d.device = dev;
    if ((e = cudaDeviceGetAttribute(&d.num_sms, cudaDevAttrMultiProcessorCount, dev)) !=
        cudaSuccess)
      return cuda_fail(e, "cudaDeviceGetAttribute(SM count)");
    cudaDeviceGetAttribute(&d.cc_major, cudaDevAttrComputeCapabilityMajor, dev);
    cudaDeviceGetAttribute(&d.cc_minor, cudaDevAttrComputeCapabilityMinor, dev);
    int l2 = 0;
    cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev);
    d.l2_bytes = l2;
    if (d.cc_major != 10 || d.cc_minor != 0)
      return fail(GNN_ERR_CUDA, "device %d is sm_%d%d; this library is built for sm_100a only",
                  dev, d.cc_major, d.cc_minor);
    cache[dev] = d;
    have[dev] = true;
  }
  *out = cache[dev];
  return GNN_OK;
}

// ------------------------------------------------------------- kernels ----
__global__ void csr_to_coo_kernel(const int32_t *__restrict__ row_ptr, int64_t M,
                                  int64_t row_base, int32_t *__restrict__ row_ind) {
  // one warp per row: coalesced writes of the row's run
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  const int64_t base = row_ptr[0];
  for (int64_t r = warp; r < M; r += nwarps) {
    const int64_t b = row_ptr[r] - base, e = row_ptr[r + 1] - base;
    for (int64_t i = b + lane; i < e; i += 32) row_ind[i] = (int32_t)(r + row_base);
  }
}

// err[0]: first offending nnz index (or -1), err[1]: kind
__global__ void validate_kernel(gnn_graph_t g, unsigned long long *bad) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t base = g.row_ptr ? g.row_ptr[0] : 0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < g.nnz; i += stride) {
    const int64_t r = g.row_ind[i], c = g.col_ind[i];
    unsigned long long kind = 0;
    if (r < g.row_base || r >= g.row_base + g.M) kind = 1;
    else if (c < 0 || c >= g.N) kind = 2;
    else if (i > 0 && g.row_ind[i - 1] > r) kind = 3;
    else if (g.row_ptr && !((int64_t)g.row_ptr[r - g.row_base] - base <= i &&
                            i < (int64_t)g.row_ptr[r - g.row_base + 1] - base))
      kind = 4;
    if (kind) atomicMin(bad, ((unsigned long long)i << 3) | kind);
  }
}

// one warp per row: coalesced copy of K floats to the permuted row
__global__ void permute_rows_kernel(const float *__restrict__ X, int64_t ldx, int64_t n,
                                    int64_t K, const int32_t *__restrict__ perm,
                                    float *__restrict__ Y, int64_t ldy) {
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t i = warp; i < n; i += nwarps) {
    const float *x = X + i * ldx;
    float *y = Y + (int64_t)perm[i] * ldy;
    for (int64_t k = lane; k < K; k += 32) y[k] = x[k];
  }
}

// dst[i] = src[idx[i]] (grid-stride, coalesced over i)
__global__ void gather_f32_kernel(const float *__restrict__ src, const int32_t *__restrict__ idx,
                                  int64_t n, float *__restrict__ dst) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride)
    dst[i] = src[idx[i]];
}

// Y[r][:K] = X[r][:K] / max(1, row_ptr[r+1] - row_ptr[r]); one warp per row
__global__ void scale_rows_inv_degree_kernel(const int32_t *__restrict__ row_ptr, int64_t M,
                                             int32_t K, const float *__restrict__ X,
                                             int64_t ldx, float *__restrict__ Y, int64_t ldy) {
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t r = warp; r < M; r += nwarps) {
    const int32_t cnt = row_ptr[r + 1] - row_ptr[r];
    const float s = 1.0f / (float)(cnt > 1 ? cnt : 1);
    for (int k = lane; k < K; k += 32) Y[r * ldy + k] = X[r * ldx + k] * s;
  }
}

}  // namespace gnn

using namespace gnn;

extern "C" {

GNN_API const char *gnn_last_error(void) { return g_err; }

#ifndef GNN_GIT_SHA
#define GNN_GIT_SHA "unknown"
#endif
// the commit the library was built from (Makefile: git rev-parse; "+dirty" for a tree with
// uncommitted changes) -- the GPU box's snapshot has no .git, bench.py reports this
GNN_API const char *gnn_version(void) { return "gnnsparse 0.2 (sm_100a) git " GNN_GIT_SHA; }

GNN_API gnn_status_t gnn_shard_rows(const int32_t *row_ptr_host, int64_t M, int32_t P,
                                    int64_t *bounds) {
  if (!row_ptr_host || M < 0 || P < 1 || !bounds)
    return fail(GNN_ERR_INVALID_ARG, "gnn_shard_rows: bad arguments");
  const int64_t base = row_ptr_host[0];
  const int64_t nnz = (int64_t)row_ptr_host[M] - base;
  bounds[0] = 0;
  for (int32_t p = 1; p < P; ++p) {
    const int64_t t = (int64_t)p * nnz / P;
    // lower_bound over r in [0, M] of row_ptr[r] - base >= t
    int64_t lo = 0, n = M + 1;
    while (n > 0) {
      const int64_t half = n / 2;
      if ((int64_t)row_ptr_host[lo + half] - base < t) {
        lo += half + 1;
        n -= half + 1;
      } else {
        n = half;
      }
    }
    bounds[p] = lo > bounds[p - 1] ? lo : bounds[p - 1];
  }
  bounds[P] = M;
  return GNN_OK;
}

GNN_API gnn_status_t gnn_shard_edges(int64_t nnz, int32_t P, int64_t *bounds) {
  if (nnz < 0 || P < 1 || !bounds) return fail(GNN_ERR_INVALID_ARG, "gnn_shard_edges: bad arguments");
  for (int32_t p = 0; p <= P; ++p) bounds[p] = (int64_t)((__int128)p * nnz / P);
  return GNN_OK;
}

GNN_API gnn_status_t gnn_split_col_blocks(const int32_t *row_ind, const int32_t *col_ind,
                                          const float *val, int64_t nnz, int32_t P, int64_t blk,
                                          int32_t *row_out, int32_t *col_out, float *val_out,
                                          int64_t *bounds) {
  if (nnz < 0 || P < 1 || blk < 1 || !bounds ||
      (nnz > 0 && (!row_ind || !col_ind || !row_out || !col_out || (val && !val_out))))
    return fail(GNN_ERR_INVALID_ARG, "gnn_split_col_blocks: bad arguments");
  for (int32_t q = 0; q <= P; ++q) bounds[q] = 0;
  for (int64_t i = 0; i < nnz; ++i) {  // counting pass
    const int64_t q = col_ind[i] / blk;
    if (col_ind[i] < 0 || q >= P)
      return fail(GNN_ERR_INVALID_ARG, "gnn_split_col_blocks: column %d outside %d blocks of %lld",
                  col_ind[i], P, (long long)blk);
    bounds[q + 1]++;
  }
  for (int32_t q = 0; q < P; ++q) bounds[q + 1] += bounds[q];
  int64_t fill[1024];
  if (P > 1024) return fail(GNN_ERR_INVALID_ARG, "gnn_split_col_blocks: P > 1024");
  for (int32_t q = 0; q < P; ++q) fill[q] = bounds[q];
  for (int64_t i = 0; i < nnz; ++i) {  // stable scatter
    const int64_t j = fill[col_ind[i] / blk]++;
    row_out[j] = row_ind[i];
    col_out[j] = col_ind[i];
    if (val) val_out[j] = val[i];
  }
  return GNN_OK;
}

GNN_API gnn_status_t gnn_csr_to_coo(const int32_t *row_ptr, int64_t M, int64_t row_base,
                                    int32_t *row_ind, gnn_stream_t stream) {
  if (M < 0 || (M > 0 && (!row_ptr || !row_ind)))
    return fail(GNN_ERR_INVALID_ARG, "gnn_csr_to_coo: bad arguments");
  if (M == 0) return GNN_OK;
  DeviceInfo d;
  if (gnn_status_t st = device_info(&d)) return st;
  const int threads = 256;
  int64_t blocks = (M * 32 + threads - 1) / threads;
  const int64_t cap = (int64_t)d.num_sms * 16;
  if (blocks > cap) blocks = cap;
  csr_to_coo_kernel<<<(unsigned)blocks, threads, 0, (cudaStream_t)stream>>>(row_ptr, M, row_base,
                                                                           row_ind);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GNN_OK : cuda_fail(e, "csr_to_coo launch");
}

GNN_API gnn_status_t gnn_permute_rows(const float *X, int64_t ldx, int64_t n, int64_t K,
                                      const int32_t *perm, float *Y, int64_t ldy,
                                      gnn_stream_t stream) {
  if (n < 0 || K < 1 || (n > 0 && (!X || !Y || !perm || ldx < K || ldy < K)))
    return fail(GNN_ERR_INVALID_ARG, "gnn_permute_rows: bad arguments");
  if (n == 0) return GNN_OK;
  DeviceInfo d;
  if (gnn_status_t st = device_info(&d)) return st;
  int64_t blocks = (n * 32 + 255) / 256;
  if (blocks > (int64_t)d.num_sms * 32) blocks = (int64_t)d.num_sms * 32;
  permute_rows_kernel<<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>(X, ldx, n, K, perm, Y,
                                                                         ldy);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GNN_OK : cuda_fail(e, "permute_rows launch");
}

GNN_API gnn_status_t gnn_gather_f32(const float *src, const int32_t *idx, int64_t n, float *dst,
                                    gnn_stream_t stream) {
  if (n < 0 || (n > 0 && (!src || !idx || !dst)))
    return fail(GNN_ERR_INVALID_ARG, "gnn_gather_f32: bad arguments");
  if (n == 0) return GNN_OK;
  DeviceInfo d;
  if (gnn_status_t st = device_info(&d)) return st;
  int64_t blocks = (n + 255) / 256;
  if (blocks > (int64_t)d.num_sms * 16) blocks = (int64_t)d.num_sms * 16;
  gather_f32_kernel<<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>(src, idx, n, dst);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GNN_OK : cuda_fail(e, "gather launch");
}

GNN_API gnn_status_t gnn_scale_rows_inv_degree(const int32_t *row_ptr, int64_t M, int32_t K,
                                               const float *X, int64_t ldx, float *Y,
                                               int64_t ldy, gnn_stream_t stream) {
  if (M < 0 || K < 1 || (M > 0 && (!row_ptr || !X || !Y || ldx < K || ldy < K)))
    return fail(GNN_ERR_INVALID_ARG, "gnn_scale_rows_inv_degree: bad arguments");
  if (M == 0) return GNN_OK;
  DeviceInfo d;
  if (gnn_status_t st = device_info(&d)) return st;
  int64_t blocks = (M * 32 + 255) / 256;
  if (blocks > (int64_t)d.num_sms * 16) blocks = (int64_t)d.num_sms * 16;
  scale_rows_inv_degree_kernel<<<(unsigned)blocks, 256, 0, (cudaStream_t)stream>>>(
      row_ptr, M, K, X, ldx, Y, ldy);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GNN_OK : cuda_fail(e, "scale rows launch");
}

GNN_API gnn_status_t gnn_validate(const gnn_graph_t *g, gnn_stream_t stream) {
  if (!g || g->M < 0 || g->N < 0 || g->nnz < 0 ||
      (g->nnz > 0 && (!g->row_ind || !g->col_ind)))
    return fail(GNN_ERR_INVALID_ARG, "gnn_validate: bad graph descriptor");
  if (g->nnz == 0) return GNN_OK;
  DeviceInfo d;
  if (gnn_status_t st = device_info(&d)) return st;
  cudaStream_t s = (cudaStream_t)stream;
  unsigned long long *bad = nullptr, h = ~0ull;
  cudaError_t e = cudaMallocAsync((void **)&bad, sizeof(*bad), s);
  if (e != cudaSuccess) return cuda_fail(e, "gnn_validate alloc");
  cudaMemcpyAsync(bad, &h, sizeof(h), cudaMemcpyHostToDevice, s);
  validate_kernel<<<d.num_sms * 8, 256, 0, s>>>(*g, bad);
  cudaMemcpyAsync(&h, bad, sizeof(h), cudaMemcpyDeviceToHost, s);
  cudaFreeAsync(bad, s);
  e = cudaStreamSynchronize(s);
  if (e != cudaSuccess) return cuda_fail(e, "gnn_validate");
  if (h == ~0ull) return GNN_OK;
  static const char *kinds[] = {"", "row_ind out of [row_base, row_base+M)",
                                "col_ind out of [0, N)", "row_ind decreasing",
                                "row_ptr inconsistent with row_ind"};
  return fail(GNN_ERR_INPUT_CHECK, "gnn_validate: nnz %lld: %s", (long long)(h >> 3),
              kinds[h & 7]);
}

}  // extern "C"
