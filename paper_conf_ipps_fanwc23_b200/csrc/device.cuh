// device.cuh -- sm_100a load/store/atomic primitives used by the hot kernels.
//
// Feature rows (X / A2T / A1): read-only, re-read by many nnz -> L1-allocating
//   non-coherent loads, 128-bit (VW=4) or 256-bit (VW=8, LDG.E.ENL2.256, new on
//   sm_100) so one lane moves 16/32 B per instruction (HVMA, widened).
// Sparse arrays (row_ind / col_ind / val): streamed once -> L1::no_allocate, vector
//   width vw_sparse (int2/int4).
// Split-row flushes (Algo 3 "AtomicStore" P:188): red.global.add.v{2,4}.f32
//   (REDG.E.ADD.F32x4 -- note the hardware flushes subnormals).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace gnn {

constexpr unsigned kFull = 0xffffffffu;

#ifndef GNN_SPARSE_EVICT_FIRST
#define GNN_SPARSE_EVICT_FIRST 0  // L2 evict_first hint on the streamed sparse arrays
#endif
#ifndef GNN_FEAT_EVICT_LAST
#define GNN_FEAT_EVICT_LAST 0     // L2 evict_last hint on gathered feature rows
#endif

__device__ __forceinline__ uint64_t l2_evict_first() {
  uint64_t pol;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}
__device__ __forceinline__ uint64_t l2_evict_last() {
  uint64_t pol;
  asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(pol));
  return pol;
}

#ifndef GNN_USE_FFMA2
#define GNN_USE_FFMA2 1
#endif

// ------------------------------------------------------------ features ----
template <int VW>
__device__ __forceinline__ void ld_feat(const float *p, float (&x)[VW]);

template <>
__device__ __forceinline__ void ld_feat<1>(const float *p, float (&x)[1]) {
  asm("ld.global.nc.f32 %0, [%1];" : "=f"(x[0]) : "l"(p));
}
template <>
__device__ __forceinline__ void ld_feat<2>(const float *p, float (&x)[2]) {
  asm("ld.global.nc.v2.f32 {%0,%1}, [%2];" : "=f"(x[0]), "=f"(x[1]) : "l"(p));
}
template <>
__device__ __forceinline__ void ld_feat<4>(const float *p, float (&x)[4]) {
#if GNN_FEAT_EVICT_LAST
  asm("ld.global.nc.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
      : "=f"(x[0]), "=f"(x[1]), "=f"(x[2]), "=f"(x[3])
      : "l"(p), "l"(l2_evict_last()));
#else
  asm("ld.global.nc.v4.f32 {%0,%1,%2,%3}, [%4];"
               : "=f"(x[0]), "=f"(x[1]), "=f"(x[2]), "=f"(x[3])
               : "l"(p));
#endif
}
template <>
__device__ __forceinline__ void ld_feat<8>(const float *p, float (&x)[8]) {
#if GNN_FEAT_EVICT_LAST
  asm("ld.global.nc.L2::cache_hint.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
      : "=f"(x[0]), "=f"(x[1]), "=f"(x[2]), "=f"(x[3]), "=f"(x[4]), "=f"(x[5]), "=f"(x[6]),
        "=f"(x[7])
      : "l"(p), "l"(l2_evict_last()));
#else
  asm("ld.global.nc.v8.f32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=f"(x[0]), "=f"(x[1]), "=f"(x[2]), "=f"(x[3]), "=f"(x[4]), "=f"(x[5]),
                 "=f"(x[6]), "=f"(x[7])
               : "l"(p));
#endif
}

// ------------------------------------------------------------- outputs ----
template <int VW>
__device__ __forceinline__ void st_vec(float *p, const float (&x)[VW]) {
  if constexpr (VW == 1) {
    p[0] = x[0];
  } else if constexpr (VW == 2) {
    *reinterpret_cast<float2 *>(p) = make_float2(x[0], x[1]);
  } else if constexpr (VW == 4) {
    *reinterpret_cast<float4 *>(p) = make_float4(x[0], x[1], x[2], x[3]);
  } else {
    asm volatile("st.global.v8.f32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "f"(x[0]),
                 "f"(x[1]), "f"(x[2]), "f"(x[3]), "f"(x[4]), "f"(x[5]), "f"(x[6]), "f"(x[7])
                 : "memory");
  }
}

template <int VW>
__device__ __forceinline__ void st_zero(float *p) {
  float z[VW];
#pragma unroll
  for (int v = 0; v < VW; ++v) z[v] = 0.f;
  st_vec<VW>(p, z);
}

template <int VW>
__device__ __forceinline__ void red_add(float *p, const float (&x)[VW]) {
  if constexpr (VW == 1) {
    atomicAdd(p, x[0]);
  } else if constexpr (VW == 2) {
    asm volatile("red.global.add.v2.f32 [%0], {%1,%2};" ::"l"(p), "f"(x[0]), "f"(x[1])
                 : "memory");
  } else {
#pragma unroll
    for (int h = 0; h < VW; h += 4)
      asm volatile("red.global.add.v4.f32 [%0], {%1,%2,%3,%4};" ::"l"(p + h), "f"(x[h]),
                   "f"(x[h + 1]), "f"(x[h + 2]), "f"(x[h + 3])
                   : "memory");
  }
}

// ------------------------------------------------------------------ math ----
// d[0..1] += s * x[0..1] as one packed FFMA2 (fma.rn.f32x2: two IEEE fp32 FMAs, the
// same rounding as two fmaf calls).
__device__ __forceinline__ void fma2_bcast(float &d0, float &d1, float s, float x0, float x1) {
  uint64_t d, xx, ss;
  asm("mov.b64 %0, {%1,%2};" : "=l"(d) : "f"(d0), "f"(d1));
  asm("mov.b64 %0, {%1,%2};" : "=l"(xx) : "f"(x0), "f"(x1));
  asm("mov.b64 %0, {%1,%1};" : "=l"(ss) : "f"(s));
  asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(d) : "l"(ss), "l"(xx));
  asm("mov.b64 {%0,%1}, %2;" : "=f"(d0), "=f"(d1) : "l"(d));
}
// d[0..1] += a[0..1] * x[0..1] (element-wise, packed)
__device__ __forceinline__ void fma2_pair(float &d0, float &d1, float a0, float a1, float x0,
                                          float x1) {
  uint64_t d, aa, xx;
  asm("mov.b64 %0, {%1,%2};" : "=l"(d) : "f"(d0), "f"(d1));
  asm("mov.b64 %0, {%1,%2};" : "=l"(aa) : "f"(a0), "f"(a1));
  asm("mov.b64 %0, {%1,%2};" : "=l"(xx) : "f"(x0), "f"(x1));
  asm("fma.rn.f32x2 %0, %1, %2, %0;" : "+l"(d) : "l"(aa), "l"(xx));
  asm("mov.b64 {%0,%1}, %2;" : "=f"(d0), "=f"(d1) : "l"(d));
}

// acc[v] += s * x[v] for v < VW (FFMA2 for pairs)
template <int VW>
__device__ __forceinline__ void axpy(float (&acc)[VW], float s, const float (&x)[VW]) {
#if GNN_USE_FFMA2
  if constexpr (VW >= 2) {
#pragma unroll
    for (int v = 0; v < VW; v += 2) fma2_bcast(acc[v], acc[v + 1], s, x[v], x[v + 1]);
    return;
  }
#endif
#pragma unroll
  for (int v = 0; v < VW; ++v) acc[v] = fmaf(s, x[v], acc[v]);
}

// d + sum_v a[v] * x[v] (sequential fp32 chain, or two interleaved FFMA2 chains)
template <int VW>
__device__ __forceinline__ float dot_acc(float d, const float (&a)[VW], const float (&x)[VW]) {
#if GNN_USE_FFMA2
  if constexpr (VW >= 4) {
    float e0 = 0.f, e1 = 0.f;
#pragma unroll
    for (int v = 0; v < VW; v += 2) fma2_pair(e0, e1, a[v], a[v + 1], x[v], x[v + 1]);
    return d + (e0 + e1);
  }
#endif
#pragma unroll
  for (int v = 0; v < VW; ++v) d = fmaf(a[v], x[v], d);
  return d;
}

// -------------------------------------------------------------- sparse ----
// Load VWS consecutive entries starting at index i (vector when the whole vector is
// in range; element-wise with a default otherwise).  The base pointer + i is
// 4*VWS-byte aligned by construction (chunk/tile/lane offsets are multiples of VWS
// and the launcher checks the base pointers).
template <int VWS>
__device__ __forceinline__ void ld_sparse_i32(const int32_t *p, int64_t i, int64_t end,
                                              int32_t dflt, int32_t (&x)[VWS]) {
  if (i + VWS <= end) {
#if GNN_SPARSE_EVICT_FIRST
    const uint64_t pol = l2_evict_first();
    if constexpr (VWS == 4) {
      asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.s32 {%0,%1,%2,%3}, [%4], %5;"
          : "=r"(x[0]), "=r"(x[1]), "=r"(x[2]), "=r"(x[3])
          : "l"(p + i), "l"(pol));
    } else if constexpr (VWS == 2) {
      asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.s32 {%0,%1}, [%2], %3;"
          : "=r"(x[0]), "=r"(x[1])
          : "l"(p + i), "l"(pol));
    } else {
      asm("ld.global.nc.L1::no_allocate.L2::cache_hint.s32 %0, [%1], %2;"
          : "=r"(x[0])
          : "l"(p + i), "l"(pol));
    }
#else
    if constexpr (VWS == 4) {
      asm("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
                   : "=r"(x[0]), "=r"(x[1]), "=r"(x[2]), "=r"(x[3])
                   : "l"(p + i));
    } else if constexpr (VWS == 2) {
      asm("ld.global.nc.L1::no_allocate.v2.s32 {%0,%1}, [%2];"
                   : "=r"(x[0]), "=r"(x[1])
                   : "l"(p + i));
    } else {
      asm("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(x[0]) : "l"(p + i));
    }
#endif
  } else {
#pragma unroll
    for (int q = 0; q < VWS; ++q) x[q] = (i + q < end) ? __ldg(p + i + q) : dflt;
  }
}

template <int VWS>
__device__ __forceinline__ void ld_sparse_f32(const float *p, int64_t i, int64_t end,
                                              float (&x)[VWS]) {
  if (p == nullptr) {
#pragma unroll
    for (int q = 0; q < VWS; ++q) x[q] = 1.f;
    return;
  }
  int32_t (&xi)[VWS] = reinterpret_cast<int32_t (&)[VWS]>(x);
  if (i + VWS <= end) {
    ld_sparse_i32<VWS>(reinterpret_cast<const int32_t *>(p), i, end, 0, xi);
  } else {
#pragma unroll
    for (int q = 0; q < VWS; ++q) x[q] = (i + q < end) ? __ldg(p + i + q) : 0.f;
  }
}

}  // namespace gnn
