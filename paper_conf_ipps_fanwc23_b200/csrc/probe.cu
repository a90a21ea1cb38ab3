// probe.cu -- gnn_probe_gather: the pure random-row gather the SpMM/SDDMM kernels are
// built from (no sparse values, no row logic, no stores), for measured gather ceilings.
#include "device.cuh"
#include "internal.cuh"

namespace gnn {
namespace {

template <int L, int U>
__global__ void __launch_bounds__(256) probe_gather_kernel(const float *__restrict__ X,
                                                           uint32_t ldB,
                                                           const int32_t *__restrict__ idx,
                                                           int64_t n, float *__restrict__ sink) {
  constexpr int G = 32 / L;
  const int lane = threadIdx.x & 31, g = lane / L, l = lane % L;
  const int64_t gid = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * G + g;
  const int64_t ngroups = (int64_t)gridDim.x * (blockDim.x >> 5) * G;
  const char *Xb = reinterpret_cast<const char *>(X + l * 8);
  float acc[8] = {};
  for (int64_t base = gid * U; base < n; base += ngroups * U) {
    float x[U][8];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t i = base + u;
      const uint32_t c = i < n ? (uint32_t)__ldg(idx + i) : 0u;
      ld_feat<8>(reinterpret_cast<const float *>(Xb + (uint64_t)c * ldB), x[u]);
    }
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int v = 0; v < 8; ++v) acc[v] += x[u][v];
  }
  float s = 0.f;
#pragma unroll
  for (int v = 0; v < 8; ++v) s += acc[v];
  if (s == 1234.5f) sink[0] = s;  // practically never: keeps the loads live
}

// The same gather in the kernels' traversal order: lane group q (of L lanes) owns the
// `chunk` consecutive entries [q * chunk, (q + 1) * chunk), U loads in flight per lane,
// 4-warp blocks, one group per chunk over the whole grid (as the SpMM / SDDMM launch), so
// the set of rows in flight -- and with it the L2 hit rate -- is the kernels'.
template <int L, int U>
__global__ void __launch_bounds__(128) probe_gather_chunked_kernel(
    const float *__restrict__ X, uint32_t ldB, const int32_t *__restrict__ idx, int64_t n,
    int32_t chunk, float *__restrict__ sink) {
  constexpr int G = 32 / L;
  const int lane = threadIdx.x & 31, g = lane / L, l = lane % L;
  const int64_t q = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * G + g;
  const char *Xb = reinterpret_cast<const char *>(X + l * 8);
  float acc[8] = {};
  const int64_t s = q * chunk;
  const int64_t e = s + chunk < n ? s + chunk : n;
  for (int64_t base = s; base < e; base += U) {
    float x[U][8];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t i = base + u;
      const uint32_t c = i < e ? (uint32_t)__ldg(idx + i) : 0u;
      ld_feat<8>(reinterpret_cast<const float *>(Xb + (uint64_t)c * ldB), x[u]);
    }
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int v = 0; v < 8; ++v) acc[v] += x[u][v];
  }
  float t = 0.f;
#pragma unroll
  for (int v = 0; v < 8; ++v) t += acc[v];
  if (t == 1234.5f) sink[0] = t;  // practically never: keeps the loads live
}

}  // namespace
}  // namespace gnn

using namespace gnn;

extern "C" GNN_API gnn_status_t gnn_probe_gather(const float *X, int64_t ld, const int32_t *idx,
                                                 int64_t n, int32_t K, float *sink,
                                                 gnn_stream_t stream) {
  if (!X || !idx || !sink || n < 0 || ld < K || ld % 8 || !aligned(X, 32) ||
      !(K == 32 || K == 64 || K == 128 || K == 256) || ld >= (int64_t(1) << 30))
    return fail(GNN_ERR_INVALID_ARG, "gnn_probe_gather: bad arguments");
  DeviceInfo d;
  if (gnn_status_t st = device_info(&d)) return st;
  const uint32_t ldB = (uint32_t)(ld * 4);
  const unsigned blocks = d.num_sms * 8;
  cudaStream_t s = (cudaStream_t)stream;
  switch (K) {
    case 32: probe_gather_kernel<4, 8><<<blocks, 256, 0, s>>>(X, ldB, idx, n, sink); break;
    case 64: probe_gather_kernel<8, 8><<<blocks, 256, 0, s>>>(X, ldB, idx, n, sink); break;
    case 128: probe_gather_kernel<16, 8><<<blocks, 256, 0, s>>>(X, ldB, idx, n, sink); break;
    default: probe_gather_kernel<32, 8><<<blocks, 256, 0, s>>>(X, ldB, idx, n, sink); break;
  }
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GNN_OK : cuda_fail(e, "gnn_probe_gather launch");
}

extern "C" GNN_API gnn_status_t gnn_probe_gather_chunked(const float *X, int64_t ld,
                                                         const int32_t *idx, int64_t n,
                                                         int32_t K, int32_t chunk, float *sink,
                                                         gnn_stream_t stream) {
  if (!X || !idx || !sink || n < 0 || ld < K || ld % 8 || !aligned(X, 32) || chunk < 1 ||
      !(K == 32 || K == 64 || K == 128 || K == 256) || ld >= (int64_t(1) << 30))
    return fail(GNN_ERR_INVALID_ARG, "gnn_probe_gather_chunked: bad arguments");
  if (n == 0) return GNN_OK;
  const uint32_t ldB = (uint32_t)(ld * 4);
  const int L = K / 8, G = 32 / L;
  const int64_t chunks = (n + chunk - 1) / chunk;
  const int64_t per_block = 4 * G;
  const unsigned blocks = (unsigned)((chunks + per_block - 1) / per_block);
  cudaStream_t s = (cudaStream_t)stream;
  switch (K) {
    case 32: probe_gather_chunked_kernel<4, 4><<<blocks, 128, 0, s>>>(X, ldB, idx, n, chunk, sink); break;
    case 64: probe_gather_chunked_kernel<8, 4><<<blocks, 128, 0, s>>>(X, ldB, idx, n, chunk, sink); break;
    case 128: probe_gather_chunked_kernel<16, 4><<<blocks, 128, 0, s>>>(X, ldB, idx, n, chunk, sink); break;
    default: probe_gather_chunked_kernel<32, 4><<<blocks, 128, 0, s>>>(X, ldB, idx, n, chunk, sink); break;
  }
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GNN_OK : cuda_fail(e, "gnn_probe_gather_chunked launch");
}
