// microbench.cu -- measured peaks for the roofline discussion:
//   mb_gather: pure random-row gather of X[idx[i]][0:K] (K fp32 columns), the memory
//              operation SpMM/SDDMM are built from, with no sparse values, rows or
//              stores: a lane group of L = K/VW lanes per row, U rows in flight/lane.
//   mb_copy  : streaming copy (HBM read+write).
//   mb_shfl  : warp-shuffle issue rate (8 independent xor-shuffle chains per thread):
//              the cost of a shuffle-based segmented reduction in SpMM.
//   mb_fma   : fp32 FMA throughput, scalar FFMA vs packed FFMA2 (fma.rn.f32x2), 16
//              independent accumulator pairs per thread (SURVEY §8(d) peak #4).
// Not part of the product ABI (built into variants/libgnnmicro.so).
#include <cuda_runtime.h>
#include <stdint.h>

template <int VW>
__device__ __forceinline__ void ldv(const float *p, float (&x)[VW]) {
  if constexpr (VW == 4) {
    asm("ld.global.nc.v4.f32 {%0,%1,%2,%3}, [%4];" : "=f"(x[0]), "=f"(x[1]), "=f"(x[2]), "=f"(x[3]) : "l"(p));
  } else {
    asm("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
        : "=f"(x[0]), "=f"(x[1]), "=f"(x[2]), "=f"(x[3]), "=f"(x[4]), "=f"(x[5]), "=f"(x[6]), "=f"(x[7])
        : "l"(p));
  }
}

template <int VW, int L, int U>
__global__ void __launch_bounds__(256) gather_kernel(const float *__restrict__ X, uint32_t ldB,
                                                     const int32_t *__restrict__ idx, int64_t n,
                                                     float *__restrict__ out) {
  constexpr int G = 32 / L;
  const int lane = threadIdx.x & 31, g = lane / L, l = lane % L;
  const int64_t gid = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * G + g;
  const int64_t ngroups = (int64_t)gridDim.x * (blockDim.x >> 5) * G;
  const char *Xb = reinterpret_cast<const char *>(X + l * VW);
  float acc[VW] = {};
  for (int64_t base = gid * U; base < n; base += ngroups * U) {
    float x[U][VW];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t i = base + u;
      const uint32_t c = i < n ? (uint32_t)__ldg(idx + i) : 0u;
      ldv<VW>(reinterpret_cast<const float *>(Xb + (uint64_t)c * ldB), x[u]);
    }
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int v = 0; v < VW; ++v) acc[v] += x[u][v];
  }
  float s = 0.f;
#pragma unroll
  for (int v = 0; v < VW; ++v) s += acc[v];
  if (s == 1234.5f) out[0] = s;  // keep the loads alive
}

__global__ void copy_kernel(const float4 *__restrict__ a, float4 *__restrict__ b, int64_t n) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    b[i] = a[i];
}

__global__ void shfl_kernel(int iters, float *__restrict__ out) {
  float v[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) v[j] = threadIdx.x + j;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 8; ++j) v[j] = __shfl_xor_sync(0xffffffffu, v[j], 1 + (j & 3));
  }
  float s = 0.f;
#pragma unroll
  for (int j = 0; j < 8; ++j) s += v[j];
  if (s == 1234.5f) out[0] = s;
}

template <bool PACKED>
__global__ void fma_kernel(int iters, float *__restrict__ out) {
  float a[32];
#pragma unroll
  for (int j = 0; j < 32; ++j) a[j] = threadIdx.x * 1e-3f + j;
  const float x0 = 1.0001f, x1 = 0.9999f, s = 1e-7f;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 32; j += 2) {
      if constexpr (PACKED) {
        uint64_t d, xx, ss;
        asm("mov.b64 %0, {%1,%2};" : "=l"(d) : "f"(a[j]), "f"(a[j + 1]));
        asm("mov.b64 %0, {%1,%2};" : "=l"(xx) : "f"(x0), "f"(x1));
        asm("mov.b64 %0, {%1,%1};" : "=l"(ss) : "f"(s));
        asm volatile("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(d) : "l"(xx), "l"(ss));
        asm("mov.b64 {%0,%1}, %2;" : "=f"(a[j]), "=f"(a[j + 1]) : "l"(d));
      } else {
        asm volatile("fma.rn.f32 %0, %1, %2, %0;" : "+f"(a[j]) : "f"(x0), "f"(s));
        asm volatile("fma.rn.f32 %0, %1, %2, %0;" : "+f"(a[j + 1]) : "f"(x1), "f"(s));
      }
    }
  }
  float t = 0.f;
#pragma unroll
  for (int j = 0; j < 32; ++j) t += a[j];
  if (t == 1234.5f) out[0] = t;
}

extern "C" {
// 32 fp32 FMAs per thread per iteration either way (16 FFMA2 or 32 FFMA instructions)
__attribute__((visibility("default"))) int mb_fma(int packed, int blocks, int iters, float *out,
                                                  void *stream) {
  if (packed) fma_kernel<true><<<blocks, 256, 0, (cudaStream_t)stream>>>(iters, out);
  else fma_kernel<false><<<blocks, 256, 0, (cudaStream_t)stream>>>(iters, out);
  return cudaGetLastError() == cudaSuccess ? 0 : 2;
}
__attribute__((visibility("default"))) int mb_shfl(int blocks, int iters, float *out, void *stream) {
  shfl_kernel<<<blocks, 256, 0, (cudaStream_t)stream>>>(iters, out);
  return cudaGetLastError() == cudaSuccess ? 0 : 2;
}
__attribute__((visibility("default"))) int mb_gather(const float *X, int64_t ld, const int32_t *idx,
                                                     int64_t n, int K, float *out, void *stream,
                                                     int blocks) {
  cudaStream_t s = (cudaStream_t)stream;
  const uint32_t ldB = (uint32_t)(ld * 4);
  switch (K) {
    case 32: gather_kernel<4, 8, 8><<<blocks, 256, 0, s>>>(X, ldB, idx, n, out); break;
    case 64: gather_kernel<4, 16, 8><<<blocks, 256, 0, s>>>(X, ldB, idx, n, out); break;
    case 128: gather_kernel<4, 32, 8><<<blocks, 256, 0, s>>>(X, ldB, idx, n, out); break;
    case 256: gather_kernel<8, 32, 8><<<blocks, 256, 0, s>>>(X, ldB, idx, n, out); break;
    default: return 1;
  }
  return cudaGetLastError() == cudaSuccess ? 0 : 2;
}
__attribute__((visibility("default"))) int mb_copy(const void *a, void *b, int64_t bytes, void *stream,
                                                   int blocks) {
  copy_kernel<<<blocks, 256, 0, (cudaStream_t)stream>>>((const float4 *)a, (float4 *)b, bytes / 16);
  return cudaGetLastError() == cudaSuccess ? 0 : 2;
}
}
