// sddmm.cu -- hybrid-parallel SDDMM for sm_100a (S_O = (A1 A2) (.) S, P:96;
// Algorithm 2 P:112-131 is the definition, Algorithm 4 P:211-232 the prior-art GPU
// design).
//
// Same plan, chunks and lane groups as SpMM (one hybrid node/edge partition).  A lane
// group owns a whole chunk (all K-slices, so no cross-group reduction is needed).
// Per nonzero i of the chunk: gather the A2T[col_i] slice (U rows in flight per
// lane), multiply with the register-cached A1[row_i] slice -- reloaded only on a row
// switch, the reuse Algorithm 4 lines 8-11 describe -- reduce over the L lanes
// with an xor-shuffle tree (WarpReduce, line 12), scale by val_i after the sum
// (Algo 2 line 6).  Results are parked in the lane that loaded the nonzero's
// sparse entry and written back as one coalesced vector store per tile (each output
// written exactly once: plain stores, deterministic).
#include "device.cuh"
#include "internal.cuh"

namespace gnn {

template <int VW>
struct SddmmDepth {
  static constexpr int value = VW == 8 ? 4 : 8;
};

template <int VW, int L, int VWS, int SMAX>
__global__ void __launch_bounds__(kMaxThreads)
    sddmm_kernel(const SparseArgs a, const float *__restrict__ A1, const int64_t lda1,
                 const float *__restrict__ A2T, const int64_t lda2, float *__restrict__ out) {
  constexpr int G = 32 / L;
  constexpr int T = L * VWS;
  constexpr int U = SddmmDepth<VW>::value < T ? SddmmDepth<VW>::value : T;
  static_assert(T % U == 0 && U % VWS == 0, "tile / prefetch shape");
  const int lane = threadIdx.x & 31;
  const int g = lane / L;
  const int l = lane & (L - 1);
  const int64_t c = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * G + g;
  const bool item_ok = c < a.num_chunks;
  if (!__any_sync(kFull, item_ok)) return;
  const int64_t cs = c * a.chunk;
  const int64_t ce = item_ok ? min(cs + (int64_t)a.chunk, a.nnz) : cs;
  const int S = a.slices;  // <= SMAX (host-checked)

  float a1[SMAX][VW];
  int32_t cur[SMAX];
#pragma unroll
  for (int sl = 0; sl < SMAX; ++sl) {
    cur[sl] = -1;
#pragma unroll
    for (int v = 0; v < VW; ++v) a1[sl][v] = 0.f;
  }

  const int ntiles = (a.chunk + T - 1) / T;
  for (int t = 0; t < ntiles; ++t) {
    const int64_t tb = cs + (int64_t)t * T;
    const int64_t li = tb + (int64_t)l * VWS;
    int32_t rr[VWS], cc[VWS];
    float vv[VWS];
    ld_sparse_i32<VWS>(a.row_ind, li, ce, 0, rr);
    ld_sparse_i32<VWS>(a.col_ind, li, ce, 0, cc);
    ld_sparse_f32<VWS>(a.val, li, ce, vv);
    float res[VWS];
#pragma unroll
    for (int q = 0; q < VWS; ++q) res[q] = 0.f;
#pragma unroll 1
    for (int jj = 0; jj < T; jj += U) {
      int32_t rj[U], cj[U];
      float vj[U], part[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int src = (jj + u) / VWS;
        rj[u] = __shfl_sync(kFull, rr[u % VWS], src, L);
        cj[u] = __shfl_sync(kFull, cc[u % VWS], src, L);
        vj[u] = __shfl_sync(kFull, vv[u % VWS], src, L);
        part[u] = 0.f;
      }
#pragma unroll
      for (int sl = 0; sl < SMAX; ++sl) {
        if (sl < S) {
          const int k0 = (sl * L + l) * VW;
          const bool col_ok = item_ok && k0 < a.K;
          float x[U][VW];
#pragma unroll
          for (int u = 0; u < U; ++u) {
            if (col_ok && tb + jj + u < ce) {
              ld_feat<VW>(A2T + (int64_t)cj[u] * lda2 + k0, x[u]);
            } else {
#pragma unroll
              for (int v = 0; v < VW; ++v) x[u][v] = 0.f;
            }
          }
#pragma unroll
          for (int u = 0; u < U; ++u) {
            if (col_ok && tb + jj + u < ce) {
              if (rj[u] != cur[sl]) {  // row switch: load the new A1 row (Algo 4 l. 8-11)
                ld_feat<VW>(A1 + ((int64_t)rj[u] - a.row_base) * lda1 + k0, a1[sl]);
                cur[sl] = rj[u];
              }
              float d = part[u];
#pragma unroll
              for (int v = 0; v < VW; ++v) d = fmaf(a1[sl][v], x[u][v], d);
              part[u] = d;
            }
          }
        }
      }
      // WarpReduce over the group's L lanes (Algo 4 line 12), then v scaling.
#pragma unroll
      for (int u = 0; u < U; ++u) {
        float d = part[u];
#pragma unroll
        for (int o = L / 2; o > 0; o >>= 1) d += __shfl_xor_sync(kFull, d, o, L);
        if (l == (jj + u) / VWS) res[u % VWS] = d * vj[u];
      }
    }
    // one coalesced store of the tile's T results
    if (li < ce) {
      if (li + VWS <= ce) {
        if constexpr (VWS == 4) {
          *reinterpret_cast<float4 *>(out + li) = make_float4(res[0], res[1], res[2], res[3]);
        } else if constexpr (VWS == 2) {
          *reinterpret_cast<float2 *>(out + li) = make_float2(res[0], res[1]);
        } else {
          out[li] = res[0];
        }
      } else {
#pragma unroll
        for (int q = 0; q < VWS; ++q)
          if (li + q < ce) out[li + q] = res[q];
      }
    }
  }
}

using SddmmFn = void (*)(const SparseArgs, const float *__restrict__, const int64_t,
                         const float *__restrict__, const int64_t, float *__restrict__);

template <int VW, int L, int SMAX>
SddmmFn pick_sddmm_vws(int vws) {
  switch (vws) {
    case 1: return sddmm_kernel<VW, L, 1, SMAX>;
    case 2: return sddmm_kernel<VW, L, 2, SMAX>;
    case 4: return sddmm_kernel<VW, L, 4, SMAX>;
  }
  return nullptr;
}
template <int VW>
SddmmFn pick_sddmm_l(int L, int vws, int S) {
  if (S > 1) return L == 32 ? pick_sddmm_vws<VW, 32, 4>(vws) : nullptr;
  switch (L) {
    case 1: return pick_sddmm_vws<VW, 1, 1>(vws);
    case 2: return pick_sddmm_vws<VW, 2, 1>(vws);
    case 4: return pick_sddmm_vws<VW, 4, 1>(vws);
    case 8: return pick_sddmm_vws<VW, 8, 1>(vws);
    case 16: return pick_sddmm_vws<VW, 16, 1>(vws);
    case 32: return pick_sddmm_vws<VW, 32, 1>(vws);
  }
  return nullptr;
}
SddmmFn pick_sddmm(int vw, int L, int vws, int S) {
  if (S > 4) return nullptr;
  switch (vw) {
    case 1: return pick_sddmm_l<1>(L, vws, S);
    case 2: return pick_sddmm_l<2>(L, vws, S);
    case 4: return pick_sddmm_l<4>(L, vws, S);
    case 8: return pick_sddmm_l<8>(L, vws, S);
  }
  return nullptr;
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
  if (!A1 || !A2T || !out || lda1 < K || lda2 < K)
    return fail(GNN_ERR_INVALID_ARG, "gnn_sddmm: bad dense operand");
  if (!aligned(A1, 4u * VW) || !aligned(A2T, 4u * VW) || lda1 % VW || lda2 % VW)
    return fail(GNN_ERR_UNSUPPORTED,
                "gnn_sddmm: A1/A2T must be %d-byte aligned with pitches multiple of %d", 4 * VW,
                VW);
  const int vws = effective_vws(in.vw_sparse, g, out);
  SddmmFn f = pick_sddmm(VW, in.lanes, vws, in.slices);
  if (!f)
    return fail(GNN_ERR_UNSUPPORTED, "gnn_sddmm: K=%d needs %d slices (max 4 at vw=%d)", K,
                in.slices, VW);
  const SparseArgs a = make_args(p, g);
  const int threads = in.warps_per_block * 32;
  const int64_t per_block = (int64_t)in.groups * in.warps_per_block;
  const int64_t blocks = (a.num_chunks + per_block - 1) / per_block;
  f<<<(unsigned)blocks, threads, 0, (cudaStream_t)stream>>>(a, A1, lda1, A2T, lda2, out);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GNN_OK : cuda_fail(e, "gnn_sddmm launch");
}
