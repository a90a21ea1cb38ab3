// sddmm.cu -- hybrid-parallel SDDMM for sm_100a (S_O = (A1 A2) (.) S, P:96;
// Algorithm 2 P:112-131 is the definition, Algorithm 4 P:211-232 the prior-art GPU
// design).
//
// Same plan, chunks and lane groups as SpMM (one hybrid node/edge partition).  A lane
// group owns a whole chunk (all K-slices, so no cross-group reduction is needed).
// Per nonzero i of the chunk: gather the A2T[col_i] slice (U rows in flight per
// lane), multiply with the register-cached A1[row_i] slice -- reloaded only on a row
// switch, the reuse Algorithm 4 lines 8-11 describe -- reduce over the L lanes
// with a transposed butterfly that reduces U nonzeros at once (WarpReduce, line 12),
// scale by val_i after the sum (Algo 2 line 6) and store: the U results of a
// batch land in consecutive lanes, so the store is coalesced; each output is written
// exactly once (plain stores, deterministic).  Tiles whose nonzeros all share one
// row (for every group of the warp) take a fast path with no per-nonzero row or
// bounds logic; the next tile's sparse entries are prefetched into registers.
#include "device.cuh"
#include "internal.cuh"

namespace gnn {

// Lane mapping of SDDMM.  A K-slice holds V = L * R VW-wide vectors (plan rule step 2);
// SDDMM spreads them over Lg = V / Rsd lanes with Rsd vectors per lane, so each dot
// product is reduced over Lg lanes and 32 / Lg nonzeros are in flight per warp step;
// U = nonzeros per batch per group, U * Rsd = 8 feature vectors in flight per lane.
// Measured on the GCR-reordered C4 (profiles/r01_sweep8.txt): Rsd = 2 from V = 8 on
// (K=64: 2.07 -> 1.94 ms, K=128: 4.82 -> 3.61 ms, K=256: 8.85 -> 7.05 ms), 1 below.
#ifndef GNN_SDDMM_R2_FROM
#define GNN_SDDMM_R2_FROM 8  // smallest V that uses Rsd = 2
#endif
#ifndef GNN_SDDMM_UR
#define GNN_SDDMM_UR 8       // U * Rsd: feature vectors in flight per lane
#endif
template <int VW, int V, int SMAX>
struct SddmmShape {
  static constexpr int R = (V >= GNN_SDDMM_R2_FROM && V >= 2) ? 2 : 1;
  static constexpr int Lg = V / R;
  static constexpr int depth = GNN_SDDMM_UR / R > 1 ? GNN_SDDMM_UR / R : 1;
#if defined(GNN_SDDMM_MINB)
  static constexpr int minb = GNN_SDDMM_MINB;
#else
  static constexpr int minb = 1;
#endif
};

// WarpReduce (Algo 4 line 12) of U partial dot products at once over the group's L
// lanes, as a transposed butterfly: each halving step exchanges half of the values
// (U/2 + U/4 + ... shuffles instead of U * log2 L).  Afterwards value u lives in lane
// l with u = l * U / L (U <= L; lanes l % (L/U) == 0 are its owners) or, for U > L, in
// slot i of lane l with u = l * (U/L) + i.  Then S_O = sum * v (Algo 2 line 6) is
// stored for the first `valid` of the U nonzeros at out[0..U).
template <int U, int L>
__device__ __forceinline__ void reduce_scale_store(float (&part)[U], const float (&vj)[U],
                                                   const int l, float *__restrict__ out,
                                                   const int valid) {
  constexpr int P = U > L ? U / L : 1;  // values left per lane after the halving steps
  int cnt = U;
#pragma unroll
  for (int o = L / 2; o >= 1; o >>= 1) {
    if (cnt > 1) {
      const int half = cnt / 2;
      const bool b = (l & o) != 0;
#pragma unroll
      for (int i = 0; i < U / 2; ++i) {
        if (i < half) {
          const float lo = part[i], hi = part[i + half];
          const float send = b ? lo : hi;
          const float keep = b ? hi : lo;
          part[i] = keep + __shfl_xor_sync(kFull, send, o, L);
        }
      }
      cnt = half;
    } else {
      part[0] += __shfl_xor_sync(kFull, part[0], o, L);
    }
  }
  if constexpr (U <= L) {
    constexpr int R = L / U;
    const int u = l / R;
    if (l % R == 0 && u < valid) {
      float v = vj[0];
#pragma unroll
      for (int w = 1; w < U; ++w) v = (w == u) ? vj[w] : v;
      out[u] = part[0] * v;
    }
  } else {
#pragma unroll
    for (int i = 0; i < P; ++i) {
      const int u = l * P + i;
      if (u < valid) {
        float v = vj[0];
#pragma unroll
        for (int w = 1; w < U; ++w) v = (w == u) ? vj[w] : v;
        out[u] = part[i] * v;
      }
    }
  }
}

// L here is V, the number of VW-wide vectors in one K-slice (plan lanes x vecs).
template <int VW, int L, int VWS, int SMAX>
__global__ void __launch_bounds__(kMaxThreads, (SddmmShape<VW, L, SMAX>::minb))
    sddmm_kernel(const SparseArgs a, const float *__restrict__ A1, const int64_t lda1,
                 const float *__restrict__ A2T, const int64_t lda2, float *__restrict__ out) {
  using Sh = SddmmShape<VW, L, SMAX>;
  constexpr int R = Sh::R, Lg = Sh::Lg;
  constexpr int G = 32 / Lg;
  constexpr int T = Lg * VWS;
  constexpr int U0 = Sh::depth > VWS ? Sh::depth : VWS;
  constexpr int U = U0 < T ? U0 : T;
  static_assert(T % U == 0 && U % VWS == 0, "tile / prefetch shape");
  const int lane = threadIdx.x & 31;
  const int g = lane / Lg;
  const int l = lane & (Lg - 1);
  const int64_t c = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * G + g;
  const bool item_ok = c < a.num_chunks;
  if (!__any_sync(kFull, item_ok)) return;
  const int64_t cs = c * a.chunk;
  const int n = item_ok ? (int)(min(cs + (int64_t)a.chunk, a.nnz) - cs) : 0;
  const int S = a.slices;  // <= SMAX (host-checked)
  const uint32_t ld2B = (uint32_t)lda2 * 4u;
  const char *__restrict__ A2b = reinterpret_cast<const char *>(A2T);

  // column of vector r of slice sl owned by lane l: (sl*L + r*Lg + l) * VW
  float a1[SMAX][R][VW];
  int32_t cur[SMAX];  // row whose A1 slice is cached, per slice
#pragma unroll
  for (int sl = 0; sl < SMAX; ++sl) {
    cur[sl] = -1;
#pragma unroll
    for (int r = 0; r < R; ++r)
#pragma unroll
      for (int v = 0; v < VW; ++v) a1[sl][r][v] = 0.f;
  }

  const int32_t *__restrict__ ri = a.row_ind + cs;
  const int32_t *__restrict__ ci = a.col_ind + cs;
  const float *__restrict__ vi = a.val ? a.val + cs : nullptr;
  float *__restrict__ oc = out + cs;
  int32_t rr[VWS], cc[VWS], nr[VWS], nc[VWS];
  float vv[VWS], nv[VWS];
  ld_sparse_i32<VWS>(ri, l * VWS, n, 0, nr);
  ld_sparse_i32<VWS>(ci, l * VWS, n, 0, nc);
  ld_sparse_f32<VWS>(vi, l * VWS, n, nv);

  auto load_a1_slice = [&](int sl, int32_t row) {
    const float *base = A1 + ((int64_t)row - a.row_base) * lda1;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const int k0 = (sl * L + r * Lg + l) * VW;
      if (k0 < a.K) ld_feat<VW>(base + k0, a1[sl][r]);
    }
    cur[sl] = row;
  };

  const int ntiles = (a.chunk + T - 1) / T;
  for (int t = 0; t < ntiles; ++t) {
    const int tb = t * T;
#pragma unroll
    for (int q = 0; q < VWS; ++q) {
      rr[q] = nr[q];
      cc[q] = nc[q];
      vv[q] = nv[q];
    }
    if (t + 1 < ntiles) {
      const int li = tb + T + l * VWS;
      ld_sparse_i32<VWS>(ri, li, n, 0, nr);
      ld_sparse_i32<VWS>(ci, li, n, 0, nc);
      ld_sparse_f32<VWS>(vi, li, n, nv);
    }
    const int32_t r_first = __shfl_sync(kFull, rr[0], 0, Lg);
    const int32_t r_last = __shfl_sync(kFull, rr[VWS - 1], Lg - 1, Lg);
    const bool fast = __all_sync(kFull, ((tb + T <= n) && r_first == r_last) || !item_ok);
    if (fast && item_ok && r_first != cur[0]) {  // row switch at the tile start
#pragma unroll
      for (int sl = 0; sl < SMAX; ++sl)
        if (sl < S) load_a1_slice(sl, r_first);
    }
#pragma unroll 1
    for (int jj = 0; jj < T; jj += U) {
      int32_t rj[U];
      uint32_t cj[U];
      float vj[U], part[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int src = (jj + u) / VWS;
        cj[u] = (uint32_t)__shfl_sync(kFull, cc[u % VWS], src, Lg);
        vj[u] = __shfl_sync(kFull, vv[u % VWS], src, Lg);
        rj[u] = fast ? r_first : __shfl_sync(kFull, rr[u % VWS], src, Lg);
        part[u] = 0.f;
      }
      const int valid = n - (tb + jj);
#pragma unroll
      for (int sl = 0; sl < SMAX; ++sl) {
        if (sl < S) {
          float x[U][R][VW];
#pragma unroll
          for (int u = 0; u < U; ++u) {
            const float *rowp =
                reinterpret_cast<const float *>(A2b + (uint64_t)cj[u] * ld2B);
#pragma unroll
            for (int r = 0; r < R; ++r) {
              const int k0 = (sl * L + r * Lg + l) * VW;
              if (item_ok && k0 < a.K && (fast || u < valid)) {
                ld_feat<VW>(rowp + k0, x[u][r]);
              } else {
#pragma unroll
                for (int v = 0; v < VW; ++v) x[u][r][v] = 0.f;
              }
            }
          }
#pragma unroll
          for (int u = 0; u < U; ++u) {
            if (!fast && item_ok && u < valid && rj[u] != cur[sl]) {
              // row-switch procedure: load the new A1 row (Algo 4 lines 8-11)
              load_a1_slice(sl, rj[u]);
            }
#pragma unroll
            for (int r = 0; r < R; ++r) part[u] = dot_acc<VW>(part[u], a1[sl][r], x[u][r]);
          }
        }
      }
      reduce_scale_store<U, Lg>(part, vj, l, oc + tb + jj, item_ok ? valid : 0);
    }
  }
}

using SddmmFn = void (*)(const SparseArgs, const float *__restrict__, const int64_t,
                         const float *__restrict__, const int64_t, float *__restrict__);

template <int VW, int V, int SMAX>
SddmmFn pick_sddmm_vws(int vws) {
  // a batch must cover whole sparse vectors: narrow the sparse loads when U < vw_sparse
  constexpr int D = SddmmShape<VW, V, SMAX>::depth;
  while (vws > D) vws >>= 1;
  switch (vws) {
    case 1: return sddmm_kernel<VW, V, 1, SMAX>;
    case 2: return sddmm_kernel<VW, V, 2, SMAX>;
    case 4: return sddmm_kernel<VW, V, 4, SMAX>;
  }
  return nullptr;
}
template <int VW>
SddmmFn pick_sddmm_v(int V, int vws, int S) {
  if (S > 1) return V == 64 ? pick_sddmm_vws<VW, 64, 4>(vws) : nullptr;
  switch (V) {
    case 1: return pick_sddmm_vws<VW, 1, 1>(vws);
    case 2: return pick_sddmm_vws<VW, 2, 1>(vws);
    case 4: return pick_sddmm_vws<VW, 4, 1>(vws);
    case 8: return pick_sddmm_vws<VW, 8, 1>(vws);
    case 16: return pick_sddmm_vws<VW, 16, 1>(vws);
    case 32: return pick_sddmm_vws<VW, 32, 1>(vws);
    case 64: return pick_sddmm_vws<VW, 64, 1>(vws);
  }
  return nullptr;
}
// V = L * R vectors per slice; S slices (<= 4)
SddmmFn pick_sddmm(int vw, int V, int vws, int S) {
  if (S > 4) return nullptr;
  switch (vw) {
    case 1: return pick_sddmm_v<1>(V, vws, S);
    case 2: return pick_sddmm_v<2>(V, vws, S);
    case 4: return pick_sddmm_v<4>(V, vws, S);
    case 8: return pick_sddmm_v<8>(V, vws, S);
  }
  return nullptr;
}
// lanes per dot product of the instantiation pick_sddmm returns
template <int VW>
int group_lanes_vw(int V, int S) {
  if (S > 1) return SddmmShape<VW, 64, 4>::Lg;
  switch (V) {
    case 1: return SddmmShape<VW, 1, 1>::Lg;
    case 2: return SddmmShape<VW, 2, 1>::Lg;
    case 4: return SddmmShape<VW, 4, 1>::Lg;
    case 8: return SddmmShape<VW, 8, 1>::Lg;
    case 16: return SddmmShape<VW, 16, 1>::Lg;
    case 32: return SddmmShape<VW, 32, 1>::Lg;
    default: return SddmmShape<VW, 64, 1>::Lg;
  }
}
int sddmm_group_lanes(int vw, int V, int S) {
  switch (vw) {
    case 1: return group_lanes_vw<1>(V, S);
    case 2: return group_lanes_vw<2>(V, S);
    case 4: return group_lanes_vw<4>(V, S);
    default: return group_lanes_vw<8>(V, S);
  }
}

}  // namespace gnn

using namespace gnn;

extern "C" GNN_API gnn_status_t gnn_sddmm(gnn_plan_t plan, const gnn_graph_t *g,
                                          const float *A1, int64_t lda1, const float *A2T,
                                          int64_t lda2, float *out, gnn_stream_t stream) {
  const Plan *p = reinterpret_cast<const Plan *>(plan);
  if (gnn_status_t st = check_common(p, g, "gnn_sddmm")) return st;
  const gnn_plan_info_t &in = p->info;
  const int K = in.K, VW = in.vw_feat;
  if (g->nnz == 0) return GNN_OK;
  if (!A1 || !A2T || !out || lda1 < K || lda2 < K || lda2 >= (int64_t(1) << 30))
    return fail(GNN_ERR_INVALID_ARG, "gnn_sddmm: bad dense operand");
  if (!aligned(A1, 4u * VW) || !aligned(A2T, 4u * VW) || lda1 % VW || lda2 % VW)
    return fail(GNN_ERR_UNSUPPORTED,
                "gnn_sddmm: A1/A2T must be %d-byte aligned with pitches multiple of %d", 4 * VW,
                VW);
  const int vws = effective_vws(in.vw_sparse, g, out);
  const int V = in.lanes * in.vecs;  // vectors per K-slice
  SddmmFn f = pick_sddmm(VW, V, vws, in.slices);
  if (!f)
    return fail(GNN_ERR_UNSUPPORTED, "gnn_sddmm: K=%d needs %d slices (max 4 at vw=%d)", K,
                in.slices, VW);
  const SparseArgs a = make_args(p, g);
  const int threads = in.warps_per_block * 32;
  const int lg = sddmm_group_lanes(VW, V, in.slices);
  const int64_t per_block = (int64_t)(32 / lg) * in.warps_per_block;
  const int64_t blocks = (a.num_chunks + per_block - 1) / per_block;
  f<<<(unsigned)blocks, threads, 0, (cudaStream_t)stream>>>(a, A1, lda1, A2T, lda2, out);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GNN_OK : cuda_fail(e, "gnn_sddmm launch");
}
