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

#include <type_traits>

namespace gnn {

constexpr unsigned kFull = 0xffffffffu;

#ifndef GNN_SPARSE_EVICT_FIRST
#define GNN_SPARSE_EVICT_FIRST 1  // L2 evict_first hint on the streamed sparse arrays
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
#ifndef GNN_BF16_FHFMA
#define GNN_BF16_FHFMA 1  // bf16 dot products (SDDMM) on the mixed-precision FMA
#endif

// ------------------------------------------------------------ features ----
// address of feature row c: base + c * ldB as ONE mad.wide.u32 (IMAD.WIDE.U32 with the
// 64-bit base as addend); written as C++ the compiler splits it into IMAD.WIDE + IADD3 +
// IADD3.X and, under the tight register budgets, reloads the base from the constant bank
// inside the gather loop
__device__ __forceinline__ const char *row_addr(const char *base, uint32_t c, uint32_t ldB) {
  const char *p;
  asm("mad.wide.u32 %0, %1, %2, %3;" : "=l"(p) : "r"(c), "r"(ldB), "l"(base));
  return p;
}

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
#ifndef GNN_OUT_STREAMING
#define GNN_OUT_STREAMING 0  // outputs stored with the streaming (.cs, evict-first) policy
#endif
template <int VW>
__device__ __forceinline__ void st_vec(float *p, const float (&x)[VW]) {
#if GNN_OUT_STREAMING
  // written once, never re-read by the kernel: keep them from displacing gathered rows
  if constexpr (VW == 1) {
    __stcs(p, x[0]);
  } else if constexpr (VW == 2) {
    __stcs(reinterpret_cast<float2 *>(p), make_float2(x[0], x[1]));
  } else if constexpr (VW == 4) {
    __stcs(reinterpret_cast<float4 *>(p), make_float4(x[0], x[1], x[2], x[3]));
  } else {
#pragma unroll
    for (int h = 0; h < VW; h += 8)
      asm volatile("st.global.cs.v8.f32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p + h),
                   "f"(x[h]), "f"(x[h + 1]), "f"(x[h + 2]), "f"(x[h + 3]), "f"(x[h + 4]),
                   "f"(x[h + 5]), "f"(x[h + 6]), "f"(x[h + 7])
                   : "memory");
  }
#else
  if constexpr (VW == 1) {
    p[0] = x[0];
  } else if constexpr (VW == 2) {
    *reinterpret_cast<float2 *>(p) = make_float2(x[0], x[1]);
  } else if constexpr (VW == 4) {
    *reinterpret_cast<float4 *>(p) = make_float4(x[0], x[1], x[2], x[3]);
  } else {
#pragma unroll
    for (int h = 0; h < VW; h += 8)
      asm volatile("st.global.v8.f32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p + h),
                   "f"(x[h]), "f"(x[h + 1]), "f"(x[h + 2]), "f"(x[h + 3]), "f"(x[h + 4]),
                   "f"(x[h + 5]), "f"(x[h + 6]), "f"(x[h + 7])
                   : "memory");
  }
#endif
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

// ---------------------------------------------------------- feature types ----
// Gathered feature rows are fp32 or bf16; arithmetic and outputs are
// fp32 either way.  FeatVec<TF, VW> holds one VW-element vector as loaded (bf16 stays
// packed two per register, widened exactly to fp32 when consumed: bf16 -> fp32 is a
// 16-bit shift).
struct F32 {
  static constexpr int bytes = 4;
};
struct BF16 {
  static constexpr int bytes = 2;
};

template <typename TF, int VW>
struct FeatVec;

template <int VW>
struct FeatVec<F32, VW> {
  float r[VW];
  __device__ __forceinline__ void load(const char *p) {
    ld_feat<VW>(reinterpret_cast<const float *>(p), r);
  }
  __device__ __forceinline__ void zero() {
#pragma unroll
    for (int v = 0; v < VW; ++v) r[v] = 0.f;
  }
  __device__ __forceinline__ float get(int v) const { return r[v]; }
};

template <int VW>
struct FeatVec<BF16, VW> {
  static_assert(VW % 2 == 0 && VW <= 16, "bf16 vectors hold 2..16 elements");
  uint32_t r[VW / 2];
  __device__ __forceinline__ void load(const char *p) {
    if constexpr (VW == 16) {
      asm("ld.global.nc.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
          : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
            "=r"(r[7])
          : "l"(p));
    } else if constexpr (VW == 8) {
      asm("ld.global.nc.v4.b32 {%0,%1,%2,%3}, [%4];"
          : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3])
          : "l"(p));
    } else if constexpr (VW == 4) {
      asm("ld.global.nc.v2.b32 {%0,%1}, [%2];" : "=r"(r[0]), "=r"(r[1]) : "l"(p));
    } else {
      asm("ld.global.nc.b32 %0, [%1];" : "=r"(r[0]) : "l"(p));
    }
  }
  __device__ __forceinline__ void zero() {
#pragma unroll
    for (int v = 0; v < VW / 2; ++v) r[v] = 0u;
  }
  __device__ __forceinline__ float get(int v) const {
    return (v & 1) ? __uint_as_float(r[v >> 1] & 0xffff0000u) : __uint_as_float(r[v >> 1] << 16);
  }
};

// acc[v] += s * x[v] (FFMA2 pairs)
template <typename TF, int VW>
__device__ __forceinline__ void axpy_f(float (&acc)[VW], float s, const FeatVec<TF, VW> &x) {
#if GNN_USE_FFMA2
  if constexpr (VW >= 2) {
#pragma unroll
    for (int v = 0; v < VW; v += 2) fma2_bcast(acc[v], acc[v + 1], s, x.get(v), x.get(v + 1));
    return;
  }
#endif
#pragma unroll
  for (int v = 0; v < VW; ++v) acc[v] = fmaf(s, x.get(v), acc[v]);
}

// d + sum_v a[v] * x[v] (two interleaved FFMA2 chains for VW >= 4)
template <typename TF, int VW>
__device__ __forceinline__ float dot_f(float d, const FeatVec<TF, VW> &a,
                                       const FeatVec<TF, VW> &x) {
#if GNN_BF16_FHFMA
  if constexpr (std::is_same<TF, BF16>::value && VW >= 4) {
    // bf16 x bf16 products accumulated in fp32 by the mixed-precision FMA (FHFMA.BF16,
    // half selectors straight from the packed words): no widening instructions.  The
    // product of two bf16 values is exact in fp32, so e0 / e1 (even / odd elements) round
    // exactly like the FFMA2 pair chains on widened operands below: identical results.
    float e0 = 0.f, e1 = 0.f;
#pragma unroll
    for (int w = 0; w < VW / 2; ++w)
      asm("{.reg .b16 al, ah, xl, xh;\n\t"
          "mov.b32 {al, ah}, %2;\n\t"
          "mov.b32 {xl, xh}, %3;\n\t"
          "fma.rn.f32.bf16 %0, al, xl, %0;\n\t"
          "fma.rn.f32.bf16 %1, ah, xh, %1;}"
          : "+f"(e0), "+f"(e1)
          : "r"(a.r[w]), "r"(x.r[w]));
    return d + (e0 + e1);
  }
#endif
#if GNN_USE_FFMA2
  if constexpr (VW >= 4) {
    float e0 = 0.f, e1 = 0.f;
#pragma unroll
    for (int v = 0; v < VW; v += 2) fma2_pair(e0, e1, a.get(v), a.get(v + 1), x.get(v), x.get(v + 1));
    return d + (e0 + e1);
  }
#endif
#pragma unroll
  for (int v = 0; v < VW; ++v) d = fmaf(a.get(v), x.get(v), d);
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

// ------------------------------------------------------- sparse tiles ----
// The streamed sparse arrays are staged through a per-warp, double-buffered shared
// memory ring with cp.async (LDGSTS, L1-bypassing for 16-byte copies): the next tile
// is in flight while the current one is consumed, and no registers hold tiles.  Each
// lane group's tile of T = L * VWS nonzeros sits at a padded stride of T + 4 words so
// that the groups of a warp hit different banks when they read "their" nonzero.
template <int BYTES>
__device__ __forceinline__ void cp_async(void *smem_dst, const void *gsrc, int src_bytes) {
  const uint32_t d = (uint32_t)__cvta_generic_to_shared(smem_dst);
  if constexpr (BYTES == 16) {
#if GNN_SPARSE_EVICT_FIRST
    // streamed once: ask L2 to evict these lines first (keeps the gathered rows of X)
    asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2, %3;" ::"r"(d),
                 "l"(gsrc), "r"(src_bytes), "l"(l2_evict_first())
                 : "memory");
#else
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(d), "l"(gsrc),
                 "r"(src_bytes)
                 : "memory");
#endif
  } else {
    asm volatile("cp.async.ca.shared.global [%0], [%1], %2, %3;" ::"r"(d), "l"(gsrc),
                 "n"(BYTES), "r"(src_bytes)
                 : "memory");
  }
}
__device__ __forceinline__ void cp_async_commit() {
  asm volatile("cp.async.commit_group;" ::: "memory");
}
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

template <int L, int VWS>
struct SparseTiles {
  static constexpr int G = 32 / L;
  static constexpr int T = L * VWS;        // nonzeros per tile per lane group
  static constexpr int STRIDE = T + 4;     // words per group (bank padding, 16-B aligned)
  static constexpr int WORDS = G * STRIDE;  // words per array per stage
  static constexpr int WARP_WORDS = 2 * 3 * WORDS;
  static constexpr int BYTES_PER_WARP = WARP_WORDS * 4;
  int32_t *w;  // this warp's region: [stage][row|col|val][G * STRIDE]
  __device__ __forceinline__ int32_t *rows(int st, int g) const { return w + (st * 3 + 0) * WORDS + g * STRIDE; }
  __device__ __forceinline__ int32_t *cols(int st, int g) const { return w + (st * 3 + 1) * WORDS + g * STRIDE; }
  __device__ __forceinline__ float *vals(int st, int g) const {
    return reinterpret_cast<float *>(w + (st * 3 + 2) * WORDS + g * STRIDE);
  }
  // Lane l of group g copies entries [tb + l*VWS, +VWS) of its chunk (n valid entries;
  // the rest zero-filled) into stage st.
  __device__ __forceinline__ void load(int st, int g, int l, const int32_t *ri, const int32_t *ci,
                                       const float *vi, int tb, int n) const {
    const int i = tb + l * VWS;
    int cnt = n - i;
    cnt = cnt < 0 ? 0 : (cnt > VWS ? VWS : cnt);
    const int bytes = cnt * 4;
    const int off = cnt > 0 ? i : 0;  // no bytes are read when cnt == 0
    cp_async<4 * VWS>(rows(st, g) + l * VWS, ri + off, bytes);
    cp_async<4 * VWS>(cols(st, g) + l * VWS, ci + off, bytes);
    if (vi) cp_async<4 * VWS>(vals(st, g) + l * VWS, vi + off, bytes);
  }
};


// ------------------------------------------------- TMA-staged sparse tiles ----
// ncu on the cp.async ring (C4, K = 32) showed the LDGSTS copies costing ~27 L1 data-pipe
// wavefronts per warp instruction -- ~40% of the wavefronts of a data pipe running at
// 70-83% of its peak, the busiest unit of both kernels.  With vw_sparse = 4 (16-byte
// aligned chunk bases) the tiles can instead be filled by the TMA unit: one bulk copy
// (cp.async.bulk, global -> shared, completion counted on a per-warp mbarrier) per
// (group, array) and tile, issued by one lane each, which bypasses the LSU data pipe.
// Tile T = L * 4 * TM nonzeros per group (TM: tile multiplier), stride T + 4 words
// (bank padding, keeps 16-byte destination alignment).  Entries past the chunk end are
// left stale (the kernels never use them); a tail that is not a multiple of 16 bytes is
// copied with plain loads by the issuing lane.
// MEASURED SLOWER (profiles/r01_sweep31_tma_tiles.txt, C4 GCR): SpMM K=32 0.93 -> 1.16 ms,
// SDDMM 1.06 -> 1.24 ms at TM = 1, no gain at K = 256 either: the many small (64-256 B)
// bulk copies and the mbarrier round trip one tile ahead cost more than the LDGSTS
// wavefronts they remove, so the data pipe is busy but not the binding limit (the L2 ->
// SM return path is).  Kept as an opt-in build (-DGNN_TMA_TILES=1) for that record.
#ifndef GNN_TMA_TILES
#define GNN_TMA_TILES 0  // measured slower (profiles/r01_sweep31_tma_tiles.txt): opt-in
#endif
#ifndef GNN_TILE_MULT
#define GNN_TILE_MULT 1
#endif

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count)
               : "memory");
}
__device__ __forceinline__ void mbar_fence_init() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // (a cluster-scope fence would emit CCTL.IVALL: an L1 flush per warp)
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t *bar, uint32_t tx) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(tx)
               : "memory");
}
__device__ __forceinline__ void mbar_wait_parity(uint64_t *bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n"
      "LAB_WAIT:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@P1 bra DONE;\n\t"
      "bra LAB_WAIT;\n"
      "DONE:\n\t}" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes,
                                         uint64_t *bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::
          "r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

template <int L, int TM>
struct TmaTiles {
  static constexpr int G = 32 / L;
  static constexpr int T = L * 4 * TM;       // nonzeros per tile per lane group
  static constexpr int STRIDE = T + 4;       // words per group
  static constexpr int WORDS = G * STRIDE;   // words per array per stage
  static constexpr int SLOTS = (3 * G + 31) / 32;  // copies issued per lane per tile
  static constexpr int WARP_WORDS = 4 + 2 * 3 * WORDS;  // 2 mbarriers + ring
  static constexpr int BYTES_PER_WARP = WARP_WORDS * 4;
  int32_t *w;
  const int32_t *src[SLOTS];  // this lane's copy slots: source of (array, group) at tile 0
  int doff[SLOTS];            // ... destination (words into the warp region, stage 0)
  int n[SLOTS];               // ... valid entries of that group's chunk (0: no copy)
  __device__ __forceinline__ uint64_t *bar(int st) const { return reinterpret_cast<uint64_t *>(w) + st; }
  __device__ __forceinline__ int32_t *arr(int st, int a, int g) const {
    return w + 4 + (st * 3 + a) * WORDS + g * STRIDE;
  }
  __device__ __forceinline__ int32_t *rows(int st, int g) const { return arr(st, 0, g); }
  __device__ __forceinline__ int32_t *cols(int st, int g) const { return arr(st, 1, g); }
  __device__ __forceinline__ float *vals(int st, int g) const {
    return reinterpret_cast<float *>(arr(st, 2, g));
  }
  // chunk_of(gg, &cs, &n): first nonzero and count of group gg's chunk (n = 0: none);
  // (own_cs, own_n: the calling lane's own group's, unused here)
  template <typename ChunkOf>
  __device__ __forceinline__ void init(int32_t *warp_smem, int lane, const int32_t *ri0,
                                       const int32_t *ci0, const float *vi0, ChunkOf chunk_of,
                                       int64_t, int) {
    w = warp_smem;
#pragma unroll
    for (int q = 0; q < SLOTS; ++q) {
      const int j = lane + 32 * q;
      const int a = j / G, gg = j % G;
      n[q] = 0;
      src[q] = ri0;
      doff[q] = 4 + ((a < 3 ? a : 0) * WORDS + gg * STRIDE);
      if (j < 3 * G && (a != 2 || vi0)) {
        int64_t cs;
        int cnt;
        chunk_of(gg, cs, cnt);
        n[q] = cnt;
        src[q] = (a == 0 ? ri0 : a == 1 ? ci0 : reinterpret_cast<const int32_t *>(vi0)) + cs;
      }
    }
    if (!vi0)  // v = 1: value slots hold 1.0 for good (never copied), as AsyncTiles
      for (int e = lane; e < WORDS; e += 32) vals(0, 0)[e] = vals(1, 0)[e] = 1.f;
    if (lane == 0) {
      mbar_init(bar(0), 1);
      mbar_init(bar(1), 1);
      mbar_fence_init();
    }
    __syncwarp();
  }
  // fill stage st with entries [tb, tb + T) of every group's chunk
  __device__ __forceinline__ void issue(int st, int tb, int lane) const {
    uint32_t bulk[SLOTS], mine = 0;
#pragma unroll
    for (int q = 0; q < SLOTS; ++q) {
      int cnt = n[q] - tb;
      cnt = cnt < 0 ? 0 : (cnt > T ? T : cnt);
      bulk[q] = (uint32_t)(cnt * 4) & ~15u;
      mine += bulk[q];
    }
    const uint32_t total = __reduce_add_sync(kFull, mine);
    if (lane == 0) mbar_arrive_expect_tx(bar(st), total);
    const int soff = st * 3 * WORDS;
#pragma unroll
    for (int q = 0; q < SLOTS; ++q) {
      int32_t *d = w + doff[q] + soff;
      if (bulk[q]) bulk_g2s(d, src[q] + tb, bulk[q], bar(st));
      int cnt = n[q] - tb;
      cnt = cnt > T ? T : cnt;
      for (int e = (int)(bulk[q] >> 2); e < cnt; ++e) d[e] = __ldg(src[q] + tb + e);
    }
  }
  __device__ __forceinline__ void skip() const {}
  __device__ __forceinline__ void wait(int st, int t) const {
    mbar_wait_parity(bar(st), (uint32_t)((t >> 1) & 1));
  }
};

// The cp.async ring behind the same interface (vw_sparse < 4: misaligned sub-views,
// small chunks).
template <int L, int VWS>
struct AsyncTiles : SparseTiles<L, VWS> {
  using Base = SparseTiles<L, VWS>;
  int g, l, cnt;
  const int32_t *ri, *ci;
  const float *vi;
  // each lane copies for its own group only: (own_cs, own_n) = its chunk's first nonzero
  // and count, as the kernel already computed them
  template <typename ChunkOf>
  __device__ __forceinline__ void init(int32_t *warp_smem, int lane, const int32_t *ri0,
                                       const int32_t *ci0, const float *vi0, ChunkOf,
                                       int64_t own_cs, int own_n) {
    this->w = warp_smem;
    g = lane / L;
    l = lane & (L - 1);
    cnt = own_n;
    ri = ri0 + own_cs;
    ci = ci0 + own_cs;
    vi = vi0 ? vi0 + own_cs : nullptr;
    if (!vi0) fill_ones(this->vals(0, g) + l * VWS, this->vals(1, g) + l * VWS);
  }
  // val == NULL (v = 1): the value slots of both stages hold 1.0 for good (load() never
  // writes them), so the kernels read s_val unconditionally -- no select per nonzero
  __device__ __forceinline__ static void fill_ones(float *a, float *b) {
#pragma unroll
    for (int v = 0; v < VWS; ++v) a[v] = b[v] = 1.f;
  }
  __device__ __forceinline__ void issue(int st, int tb, int) const {
    Base::load(st, g, l, ri, ci, vi, tb, cnt);
    cp_async_commit();
  }
  __device__ __forceinline__ void skip() const { cp_async_commit(); }  // (empty group)
  __device__ __forceinline__ void wait(int, int) const {
    cp_async_wait<1>();  // all but the most recent group: tile t has landed
  }
};

template <int L, int VWS>
using TilesFor = typename std::conditional<(VWS == 4 && GNN_TMA_TILES), TmaTiles<L, GNN_TILE_MULT>,
                                           AsyncTiles<L, VWS>>::type;

// dynamic shared memory per warp of the tiles of a lane-group width L at vw_sparse vws
inline int tile_bytes_per_warp(int L, int vws) {
  if (vws == 4 && GNN_TMA_TILES) return (4 + 2 * 3 * (32 / L) * (L * 4 * GNN_TILE_MULT + 4)) * 4;
  return 2 * 3 * (32 / L) * (L * vws + 4) * 4;
}
}  // namespace gnn
