// locality_probe.cu -- does SM-local traversal buy L1 hits on the gathers?  (experiment)
//
// The SpMM / SDDMM kernels run at 0.86-0.93 of a pure gather of their own index stream in
// chunk order (bench.py roofline), with the L1 hit rate at ~6% (ncu): the hardware block
// scheduler deals consecutive blocks to different SMs, so the blocks resident on one SM
// gather from rows ~148 blocks apart and the SM's L1 sees the whole community's X.  Here
// the same pure gather (no values, no stores) runs three ways:
//   lp_chunked : the kernels' order (one lane group per chunk over a non-persistent grid)
//   lp_smlocal : persistent grid; SM s owns a contiguous range of chunks (%smid) and its
//                blocks claim (chunk, K-slice) items from it slice-major, so the X working
//                set of one SM at a time is (columns its rows touch) x (slice width);
//                idle SMs then steal from the others' ranges
// Built into variants/liblocprobe.so (not part of the product ABI).
#include <cuda_runtime.h>
#include <stdint.h>

namespace {

__device__ __forceinline__ void ld8(const float *p, float (&x)[8]) {
  asm volatile("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=f"(x[0]), "=f"(x[1]), "=f"(x[2]), "=f"(x[3]), "=f"(x[4]), "=f"(x[5]),
                 "=f"(x[6]), "=f"(x[7])
               : "l"(p));
}

__device__ __forceinline__ uint32_t smid() {
  uint32_t s;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
  return s;
}

// gather entries [s, e) of idx, columns [col0, col0 + 8L) of X, U loads in flight per lane
template <int L, int U>
__device__ __forceinline__ void gather_range(const char *Xb, uint32_t ldB,
                                             const int32_t *__restrict__ idx, int64_t s,
                                             int64_t e, float (&acc)[8]) {
  for (int64_t base = s; base < e; base += U) {
    float x[U][8];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t i = base + u;
      const uint32_t c = i < e ? (uint32_t)__ldg(idx + i) : 0u;
      ld8(reinterpret_cast<const float *>(Xb + (uint64_t)c * ldB), x[u]);
    }
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int v = 0; v < 8; ++v) acc[v] += x[u][v];
  }
}

template <int L, int U>
__global__ void __launch_bounds__(128) lp_chunked_kernel(const float *__restrict__ X,
                                                         uint32_t ldB,
                                                         const int32_t *__restrict__ idx,
                                                         int64_t n, int32_t chunk, int K,
                                                         float *__restrict__ sink) {
  constexpr int G = 32 / L;
  const int lane = threadIdx.x & 31, g = lane / L, l = lane % L;
  const int64_t q = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * G + g;
  float acc[8] = {};
  const int64_t s = q * chunk;
  const int64_t e = s + chunk < n ? s + chunk : n;
  for (int col0 = 0; col0 < K; col0 += 8 * L)
    gather_range<L, U>(reinterpret_cast<const char *>(X + col0 + l * 8), ldB, idx, s, e, acc);
  float t = 0.f;
#pragma unroll
  for (int v = 0; v < 8; ++v) t += acc[v];
  if (t == 1234.5f) sink[0] = t;
}

// counters[2 * nsm]: [0, nsm) next item of SM s's range, [nsm, 2 nsm) unused padding
template <int L, int U>
__global__ void __launch_bounds__(128) lp_smlocal_kernel(const float *__restrict__ X,
                                                         uint32_t ldB,
                                                         const int32_t *__restrict__ idx,
                                                         int64_t n, int32_t chunk, int K,
                                                         int nsm, int slice_major,
                                                         unsigned long long *counters,
                                                         float *__restrict__ sink) {
  constexpr int G = 32 / L;
  constexpr int KS = 8 * L;
  const int lane = threadIdx.x & 31, g = lane / L, l = lane % L;
  const int64_t nch = (n + chunk - 1) / chunk;
  const int S = K / KS;
  const uint32_t me = smid() % (uint32_t)nsm;
  float acc[8] = {};
  for (int k = 0; k < nsm; ++k) {
    const uint32_t sm = (me + k) % (uint32_t)nsm;
    const int64_t c0 = nch * sm / nsm, c1 = nch * (sm + 1) / nsm;
    const int64_t items = (c1 - c0) * S;
    for (;;) {
      unsigned long long t0 = 0;
      if (lane == 0) t0 = atomicAdd(counters + sm, (unsigned long long)G);
      t0 = __shfl_sync(0xffffffffu, t0, 0);
      if ((int64_t)t0 >= items) break;
      const int64_t t = (int64_t)t0 + g;
      if (t < items) {
        int64_t c, sl;
        if (slice_major) {
          sl = t / (c1 - c0);
          c = c0 + t % (c1 - c0);
        } else {
          c = c0 + t / S;
          sl = t % S;
        }
        const int64_t s = c * chunk, e = s + chunk < n ? s + chunk : n;
        gather_range<L, U>(reinterpret_cast<const char *>(X + sl * KS + l * 8), ldB, idx, s, e,
                           acc);
      }
    }
  }
  float t = 0.f;
#pragma unroll
  for (int v = 0; v < 8; ++v) t += acc[v];
  if (t == 1234.5f) sink[0] = t;
}

// lp_front: persistent blocks of W warps (36 warps per SM, as many as lp_chunked keeps resident) claim batches of W*G consecutive chunks from one
// global counter (one chunk per lane group), so the global sweep order is the kernels' but
// the warps resident on one SM work on adjacent chunks (adjacent rows, shared columns)
template <int L, int U>
__global__ void __launch_bounds__(576) lp_front_kernel(const float *__restrict__ X, uint32_t ldB,
                                                       const int32_t *__restrict__ idx,
                                                       int64_t n, int32_t chunk, int K,
                                                       unsigned long long *counter,
                                                       float *__restrict__ sink) {
  constexpr int G = 32 / L;
  const int lane = threadIdx.x & 31, g = lane / L, l = lane % L;
  const int W = blockDim.x >> 5, w = threadIdx.x >> 5;
  const int64_t nch = (n + chunk - 1) / chunk;
  __shared__ unsigned long long base_s;
  float acc[8] = {};
  for (;;) {
    __syncthreads();
    if (threadIdx.x == 0) base_s = atomicAdd(counter, (unsigned long long)(W * G));
    __syncthreads();
    const int64_t b = (int64_t)base_s;
    if (b >= nch) break;
    const int64_t c = b + w * G + g;
    if (c < nch) {
      const int64_t s = c * chunk, e = s + chunk < n ? s + chunk : n;
      gather_range<L, U>(reinterpret_cast<const char *>(X + l * 8), ldB, idx, s, e, acc);
    }
  }
  float t = 0.f;
#pragma unroll
  for (int v = 0; v < 8; ++v) t += acc[v];
  if (t == 1234.5f) sink[0] = t;
}

// lp_chunked with U loads in flight per lane and at least MINB resident 4-warp blocks per SM
// (register cap 65536 / (128 MINB)): how the gather rate scales with bytes in flight
template <int L, int U, int MINB>
__global__ void __launch_bounds__(128, MINB) lp_mlp_kernel(const float *__restrict__ X,
                                                           uint32_t ldB,
                                                           const int32_t *__restrict__ idx,
                                                           int64_t n, int32_t chunk,
                                                           float *__restrict__ sink) {
  constexpr int G = 32 / L;
  const int lane = threadIdx.x & 31, g = lane / L, l = lane % L;
  const int64_t q = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * G + g;
  float acc[8] = {};
  const int64_t s = q * chunk;
  const int64_t e = s + chunk < n ? s + chunk : n;
  gather_range<L, U>(reinterpret_cast<const char *>(X + l * 8), ldB, idx, s, e, acc);
  float t = 0.f;
#pragma unroll
  for (int v = 0; v < 8; ++v) t += acc[v];
  if (t == 1234.5f) sink[0] = t;
}

template <int L, int U, int MINB>
cudaError_t launch_mlp(const float *X, uint32_t ldB, const int32_t *idx, int64_t n, int chunk,
                       float *sink, cudaStream_t st) {
  constexpr int G = 32 / L;
  const int64_t chunks = (n + chunk - 1) / chunk;
  const unsigned blocks = (unsigned)((chunks + 4 * G - 1) / (4 * G));
  lp_mlp_kernel<L, U, MINB><<<blocks, 128, 0, st>>>(X, ldB, idx, n, chunk, sink);
  return cudaGetLastError();
}

template <int L>
cudaError_t launch_mlp_sel(const float *X, uint32_t ldB, const int32_t *idx, int64_t n,
                           int chunk, int U, int minb, float *sink, cudaStream_t st) {
#define LP_MLP(u, b) if (U == u && minb == b) return launch_mlp<L, u, b>(X, ldB, idx, n, chunk, sink, st);
  LP_MLP(2, 1) LP_MLP(4, 1) LP_MLP(8, 1) LP_MLP(2, 12) LP_MLP(4, 12) LP_MLP(2, 16) LP_MLP(4, 16)
  LP_MLP(8, 6) LP_MLP(8, 9) LP_MLP(6, 9) LP_MLP(6, 12)
#undef LP_MLP
  return cudaErrorInvalidValue;
}

template <int L>
cudaError_t launch_chunked(const float *X, uint32_t ldB, const int32_t *idx, int64_t n,
                           int chunk, int K, float *sink, cudaStream_t st) {
  constexpr int G = 32 / L;
  const int64_t chunks = (n + chunk - 1) / chunk;
  const unsigned blocks = (unsigned)((chunks + 4 * G - 1) / (4 * G));
  lp_chunked_kernel<L, 4><<<blocks, 128, 0, st>>>(X, ldB, idx, n, chunk, K, sink);
  return cudaGetLastError();
}

template <int L>
cudaError_t launch_smlocal(const float *X, uint32_t ldB, const int32_t *idx, int64_t n,
                           int chunk, int K, int blocks_per_sm, int slice_major, int carveout,
                           unsigned long long *counters, float *sink, cudaStream_t st) {
  int dev = 0, nsm = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  if (carveout >= 0)
    cudaFuncSetAttribute(lp_smlocal_kernel<L, 4>, cudaFuncAttributePreferredSharedMemoryCarveout,
                         carveout);
  cudaMemsetAsync(counters, 0, sizeof(unsigned long long) * 2 * nsm, st);
  lp_smlocal_kernel<L, 4><<<nsm * blocks_per_sm, 128, 0, st>>>(
      X, ldB, idx, n, chunk, K, nsm, slice_major, counters, sink);
  return cudaGetLastError();
}

template <int L>
cudaError_t launch_front(const float *X, uint32_t ldB, const int32_t *idx, int64_t n, int chunk,
                         int K, int warps, int carveout, unsigned long long *counter,
                         float *sink, cudaStream_t st) {
  int dev = 0, nsm = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
  if (carveout >= 0)
    cudaFuncSetAttribute(lp_front_kernel<L, 4>, cudaFuncAttributePreferredSharedMemoryCarveout,
                         carveout);
  cudaMemsetAsync(counter, 0, sizeof(unsigned long long), st);
  lp_front_kernel<L, 4><<<nsm * (36 / warps), 32 * warps, 0, st>>>(X, ldB, idx, n, chunk, K,
                                                                  counter, sink);
  return cudaGetLastError();
}

}  // namespace

extern "C" int lp_front(const float *X, int64_t ld, const int32_t *idx, int64_t n, int K,
                        int chunk, int warps, int carveout, unsigned long long *counter,
                        float *sink, void *stream) {
  const uint32_t ldB = (uint32_t)(ld * 4);
  cudaStream_t st = (cudaStream_t)stream;
  switch (K) {
    case 32: return launch_front<4>(X, ldB, idx, n, chunk, K, warps, carveout, counter, sink, st);
    case 64: return launch_front<8>(X, ldB, idx, n, chunk, K, warps, carveout, counter, sink, st);
    case 128: return launch_front<16>(X, ldB, idx, n, chunk, K, warps, carveout, counter, sink, st);
    case 256: return launch_front<32>(X, ldB, idx, n, chunk, K, warps, carveout, counter, sink, st);
  }
  return -1;
}

extern "C" int lp_mlp(const float *X, int64_t ld, const int32_t *idx, int64_t n, int K,
                      int chunk, int U, int minb, float *sink, void *stream) {
  const uint32_t ldB = (uint32_t)(ld * 4);
  cudaStream_t st = (cudaStream_t)stream;
  switch (K) {
    case 32: return launch_mlp_sel<4>(X, ldB, idx, n, chunk, U, minb, sink, st);
    case 64: return launch_mlp_sel<8>(X, ldB, idx, n, chunk, U, minb, sink, st);
    case 128: return launch_mlp_sel<16>(X, ldB, idx, n, chunk, U, minb, sink, st);
    case 256: return launch_mlp_sel<32>(X, ldB, idx, n, chunk, U, minb, sink, st);
  }
  return -1;
}

extern "C" int lp_chunked(const float *X, int64_t ld, const int32_t *idx, int64_t n, int K,
                          int chunk, float *sink, void *stream) {
  const uint32_t ldB = (uint32_t)(ld * 4);
  cudaStream_t st = (cudaStream_t)stream;
  switch (K) {  // lane group = whole row (one vector of 8 per lane), as the kernels
    case 32: return launch_chunked<4>(X, ldB, idx, n, chunk, K, sink, st);
    case 64: return launch_chunked<8>(X, ldB, idx, n, chunk, K, sink, st);
    case 128: return launch_chunked<16>(X, ldB, idx, n, chunk, K, sink, st);
    case 256: return launch_chunked<32>(X, ldB, idx, n, chunk, K, sink, st);
  }
  return -1;
}

// KS = slice width in fp32 columns (32, 64, 128, 256; <= K)
extern "C" int lp_smlocal(const float *X, int64_t ld, const int32_t *idx, int64_t n, int K,
                          int KS, int chunk, int blocks_per_sm, int slice_major, int carveout,
                          unsigned long long *counters, float *sink, void *stream) {
  const uint32_t ldB = (uint32_t)(ld * 4);
  cudaStream_t st = (cudaStream_t)stream;
  switch (KS) {
    case 32: return launch_smlocal<4>(X, ldB, idx, n, chunk, K, blocks_per_sm, slice_major, carveout, counters, sink, st);
    case 64: return launch_smlocal<8>(X, ldB, idx, n, chunk, K, blocks_per_sm, slice_major, carveout, counters, sink, st);
    case 128: return launch_smlocal<16>(X, ldB, idx, n, chunk, K, blocks_per_sm, slice_major, carveout, counters, sink, st);
    case 256: return launch_smlocal<32>(X, ldB, idx, n, chunk, K, blocks_per_sm, slice_major, carveout, counters, sink, st);
  }
  return -1;
}
