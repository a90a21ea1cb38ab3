// spmm.cu -- hybrid-parallel SpMM for sm_100a (O = S A; Algorithm 1
// is the definition, Algorithm 3 P:168-195 the prior-art GPU design).
//
// Work decomposition: the plan cuts the nnz into chunks of C*
// consecutive nonzeros (equal work per unit, hybrid node/edge parallelism).
// Each (chunk, K-slice) work item is owned by a lane group of L lanes; every lane
// holds VW consecutive feature columns, so one group gathers L*VW columns of a
// source row per nonzero with one vector load per lane (128-bit, or 256-bit at
// VW = 8).  G = 32/L groups share a warp.  Per tile of T = L*vw_sparse nonzeros the
// group loads (row, col, val) coalesced and vectorised, then broadcasts them
// nonzero by nonzero with width-L shuffles; U feature rows are in flight per lane
// before the FMAs consume them, and the next tile's sparse entries are prefetched into
// registers.  Tiles whose nonzeros all belong to one row (for every group of the warp;
// the common case at high degree) take a fast path with no per-nonzero row or bounds
// logic; the others run the general row-switch loop.  A row switch ("row-switch procedure")
// flushes the accumulator: rows wholly inside the chunk get a plain vector store,
// rows shared with a neighbouring chunk (plan flags) a vector atomic add into a row
// zeroed beforehand by spmm_prezero_kernel.  Empty rows are written as zeros by the
// chunk that precedes them, so O is fully overwritten without a memset.
#include <atomic>
#include <climits>

#include "device.cuh"
#include "internal.cuh"

namespace gnn {

// Feature rows in flight per lane (U) and the register budget, per instantiation.
// Measured on C4 (profiles/r01_sweep4.txt): with 256-bit loads U = 4 is best while
// several chunks share a warp (L <= 8), U = 8 once a group spans >= 16 lanes.
#ifndef GNN_SPMM_MINB
#define GNN_SPMM_MINB 1  // min resident 512-thread blocks/SM the register budget must allow
#endif

// Feature vectors in flight per lane.  Measured on C4 (profiles/r01_sweep4.txt,
// r01_sweep11.txt): 4 while several chunks share a warp (L <= 8, R = 1), 8 for wider
// groups and whenever a lane holds R = 2 vectors per row.
#ifndef GNN_SPMM_DEPTH_R2
#define GNN_SPMM_DEPTH_R2 4
#endif
template <int VW, int L, int R>
struct FeatDepth {
#if defined(GNN_SPMM_DEPTH8)
  static constexpr int value = VW == 8 ? GNN_SPMM_DEPTH8 : 8;
#else
  static constexpr int value = R == 2 ? GNN_SPMM_DEPTH_R2 : (VW == 8 ? (L >= 16 ? 8 : 4) : 8);
#endif
};

// Flush the accumulator of row `cur` (Algo 3 line 15, "AtomicStore"): rows shared
// with a neighbouring chunk are combined with a vector atomic add, rows owned by this
// chunk get a plain vector store.
template <int VW>
__device__ __forceinline__ void flush_row(float *Ok, int64_t ldo, int64_t row_base, int32_t cur,
                                          int32_t rf, int32_t rl, uint32_t fl,
                                          const float (&acc)[VW]) {
  float *o = Ok + ((int64_t)cur - row_base) * ldo;
  const bool shared = (cur == rf && (fl & 1u)) || (cur == rl && (fl & 2u));
  if (shared) red_add<VW>(o, acc);
  else st_vec<VW>(o, acc);
}

// L lanes per (chunk, K-slice) work item, R VW-wide vectors per lane (plan rule step 2).
template <int VW, int L, int R, int VWS>
__global__ void __launch_bounds__(kMaxThreads, GNN_SPMM_MINB)
    spmm_kernel(const SparseArgs a, const float *__restrict__ A, const int64_t lda,
                float *__restrict__ O, const int64_t ldo) {
  constexpr int Lg = L;
  constexpr int G = 32 / Lg;
  constexpr int T = Lg * VWS;  // nonzeros per tile per group
  // U nonzeros per batch: FeatDepth vectors in flight per lane, whole sparse vectors
  constexpr int D = FeatDepth<VW, L, R>::value / R;
  constexpr int U = D > T ? T : (D < VWS ? VWS : D);
  static_assert(T % U == 0 && U % VWS == 0, "tile / prefetch shape");
  const int lane = threadIdx.x & 31;
  const int g = lane / Lg;
  const int l = lane & (Lg - 1);
  const int64_t item = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * G + g;
  const bool item_ok = item < a.num_chunks * a.slices;
  if (!__any_sync(kFull, item_ok)) return;  // warp-uniform exit

  int64_t c = 0;
  int s = 0;
  if (item_ok) {
    c = item / a.slices;
    s = (int)(item - c * a.slices);
  }
  // vector r of this lane covers columns k0 + r * L * VW .. + VW of slice s
  const int k0 = (s * L * R + l) * VW;
  bool col_ok[R];
#pragma unroll
  for (int r = 0; r < R; ++r) col_ok[r] = item_ok && k0 + r * Lg * VW < a.K;
  const int64_t cs = c * a.chunk;
  const int n = item_ok ? (int)(min(cs + (int64_t)a.chunk, a.nnz) - cs) : 0;  // nnz here
  int32_t rf = 0, rl = 0;
  uint32_t fl = 0;
  if (item_ok) {
    rf = a.row_first[c];
    rl = a.row_last[c];
    fl = a.flags[c];
  }
  // feature row c of A starts at Ab + c * ldaB (IMAD.WIDE.U32 per gather)
  const char *__restrict__ Ab = reinterpret_cast<const char *>(A + k0);
  const uint32_t ldaB = (uint32_t)lda * 4u;
  float *__restrict__ Ok = O + k0;  // row r at Ok + (r - row_base) * ldo

  auto zero_row = [&](int64_t row) {
#pragma unroll
    for (int r = 0; r < R; ++r)
      if (col_ok[r]) st_zero<VW>(Ok + (row - a.row_base) * ldo + r * Lg * VW);
  };
  float acc[R][VW];
  auto flush = [&](int32_t row) {
#pragma unroll
    for (int r = 0; r < R; ++r)
      if (col_ok[r])
        flush_row<VW>(Ok + r * Lg * VW, ldo, a.row_base, row, rf, rl, fl, acc[r]);
  };

  // empty rows between the previous chunk's last row and ours are ours to zero
  if (item_ok) {
    const int64_t prev = (c == 0) ? a.row_base - 1 : (int64_t)a.row_last[c - 1];
    for (int64_t r = prev + 1; r < rf; ++r) zero_row(r);
  }

#pragma unroll
  for (int r = 0; r < R; ++r)
#pragma unroll
    for (int v = 0; v < VW; ++v) acc[r][v] = 0.f;
  int32_t cur = -1;

  const int32_t *__restrict__ ri = a.row_ind + cs;
  const int32_t *__restrict__ ci = a.col_ind + cs;
  const float *__restrict__ vi = a.val ? a.val + cs : nullptr;
  // sparse tile registers: current and next (prefetched one tile ahead)
  int32_t rr[VWS], cc[VWS], nr[VWS], nc[VWS];
  float vv[VWS], nv[VWS];
  ld_sparse_i32<VWS>(ri, l * VWS, n, 0, nr);
  ld_sparse_i32<VWS>(ci, l * VWS, n, 0, nc);
  ld_sparse_f32<VWS>(vi, l * VWS, n, nv);

  const int ntiles = (a.chunk + T - 1) / T;  // warp-uniform trip count
  for (int t = 0; t < ntiles; ++t) {
    const int tb = t * T;
#pragma unroll
    for (int q = 0; q < VWS; ++q) {
      rr[q] = nr[q];
      cc[q] = nc[q];
      vv[q] = nv[q];
    }
    if (t + 1 < ntiles) {  // prefetch the next tile's sparse entries
      const int li = tb + T + l * VWS;
      ld_sparse_i32<VWS>(ri, li, n, 0, nr);
      ld_sparse_i32<VWS>(ci, li, n, 0, nc);
      ld_sparse_f32<VWS>(vi, li, n, nv);
    }
    const int32_t r_first = __shfl_sync(kFull, rr[0], 0, Lg);
    const int32_t r_last = __shfl_sync(kFull, rr[VWS - 1], Lg - 1, Lg);
    const bool fast_g = (tb + T <= n) && r_first == r_last;
    if (__all_sync(kFull, fast_g || !item_ok)) {
      // ---- fast path: the whole tile belongs to one row (all groups of the warp)
      if (item_ok && r_first != cur) {
        if (cur >= 0) {
          flush(cur);
          for (int64_t r = (int64_t)cur + 1; r < r_first; ++r) zero_row(r);
        }
        cur = r_first;
#pragma unroll
        for (int r = 0; r < R; ++r)
#pragma unroll
          for (int v = 0; v < VW; ++v) acc[r][v] = 0.f;
      }
#pragma unroll 1
      for (int jj = 0; jj < T; jj += U) {
        uint32_t cj[U];
        float vj[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int src = (jj + u) / VWS;
          cj[u] = (uint32_t)__shfl_sync(kFull, cc[u % VWS], src, Lg);
          vj[u] = __shfl_sync(kFull, vv[u % VWS], src, Lg);
        }
        float x[U][R][VW];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const float *rowp = reinterpret_cast<const float *>(Ab + (uint64_t)cj[u] * ldaB);
#pragma unroll
          for (int r = 0; r < R; ++r) {
            if (col_ok[r]) {
              ld_feat<VW>(rowp + r * Lg * VW, x[u][r]);
            } else {
#pragma unroll
              for (int v = 0; v < VW; ++v) x[u][r][v] = 0.f;
            }
          }
        }
#pragma unroll
        for (int u = 0; u < U; ++u)
#pragma unroll
          for (int r = 0; r < R; ++r) axpy<VW>(acc[r], vj[u], x[u][r]);
      }
    } else {
      // ---- general path: per-nonzero validity and row-switch procedure
#pragma unroll 1
      for (int jj = 0; jj < T; jj += U) {
        int32_t rj[U];
        uint32_t cj[U];
        float vj[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int src = (jj + u) / VWS;
          rj[u] = __shfl_sync(kFull, rr[u % VWS], src, Lg);
          cj[u] = (uint32_t)__shfl_sync(kFull, cc[u % VWS], src, Lg);
          vj[u] = __shfl_sync(kFull, vv[u % VWS], src, Lg);
        }
        float x[U][R][VW];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const float *rowp = reinterpret_cast<const float *>(Ab + (uint64_t)cj[u] * ldaB);
#pragma unroll
          for (int r = 0; r < R; ++r) {
            if (col_ok[r] && tb + jj + u < n) {
              ld_feat<VW>(rowp + r * Lg * VW, x[u][r]);
            } else {
#pragma unroll
              for (int v = 0; v < VW; ++v) x[u][r][v] = 0.f;
            }
          }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
          if (tb + jj + u < n) {
            if (rj[u] != cur) {  // row-switch procedure
              if (cur >= 0) {
                flush(cur);
                for (int64_t r = (int64_t)cur + 1; r < rj[u]; ++r) zero_row(r);
              }
              cur = rj[u];
#pragma unroll
              for (int r = 0; r < R; ++r)
#pragma unroll
                for (int v = 0; v < VW; ++v) acc[r][v] = 0.f;
            }
#pragma unroll
            for (int r = 0; r < R; ++r) axpy<VW>(acc[r], vj[u], x[u][r]);
          }
        }
      }
    }
  }
  if (cur >= 0) flush(cur);
  // trailing empty rows after the last chunk
  if (item_ok && c == a.num_chunks - 1) {
    for (int64_t r = (int64_t)rl + 1; r < a.row_base + a.M; ++r) zero_row(r);
  }
}

// Zero every row shared by several chunks before the atomics land on it: the row
// is zeroed by the chunk in which it starts (tail flag set, and not a pure
// continuation of an earlier chunk's row).  One warp per chunk.
template <int VW>
__global__ void spmm_prezero_kernel(const SparseArgs a, float *__restrict__ O,
                                    const int64_t ldo) {
  const int64_t c = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (c >= a.num_chunks) return;
  const uint32_t fl = a.flags[c];
  if (!(fl & 2u)) return;
  const int32_t rf = a.row_first[c], rl = a.row_last[c];
  if ((fl & 1u) && rf == rl) return;
  float *o = O + ((int64_t)rl - a.row_base) * ldo;
  for (int k = lane * VW; k < a.K; k += 32 * VW) st_zero<VW>(o + k);
}

// ------------------------------------------------------------ dispatch ----
using SpmmFn = void (*)(const SparseArgs, const float *__restrict__, const int64_t,
                        float *__restrict__, const int64_t);

template <int VW, int L, int R>
SpmmFn pick_vws(int vws) {
  switch (vws) {
    case 1: return spmm_kernel<VW, L, R, 1>;
    case 2: return spmm_kernel<VW, L, R, 2>;
    case 4: return spmm_kernel<VW, L, R, 4>;
  }
  return nullptr;
}
template <int VW>
SpmmFn pick_l(int L, int R, int vws) {
  if (R == 2) {  // the plan uses R = 2 only for rows of >= 16 vectors, i.e. L >= 8
    switch (L) {
      case 8: return pick_vws<VW, 8, 2>(vws);
      case 16: return pick_vws<VW, 16, 2>(vws);
      case 32: return pick_vws<VW, 32, 2>(vws);
    }
    return nullptr;
  }
  switch (L) {
    case 1: return pick_vws<VW, 1, 1>(vws);
    case 2: return pick_vws<VW, 2, 1>(vws);
    case 4: return pick_vws<VW, 4, 1>(vws);
    case 8: return pick_vws<VW, 8, 1>(vws);
    case 16: return pick_vws<VW, 16, 1>(vws);
    case 32: return pick_vws<VW, 32, 1>(vws);
  }
  return nullptr;
}
SpmmFn pick_spmm(int vw, int L, int R, int vws) {
  switch (vw) {
    case 1: return pick_l<1>(L, R, vws);
    case 2: return pick_l<2>(L, R, vws);
    case 4: return pick_l<4>(L, R, vws);
    case 8: return pick_l<8>(L, R, vws);
  }
  return nullptr;
}

// Cached per (device, vw, lanes, vecs, wpb): the occupancy API is a host-side query but
// not free, and plans are rebuilt every step in graph-sampling training (C3).
int spmm_active_blocks_per_sm(int vw, int lanes, int vecs, int wpb) {
  static std::atomic<int> cache[64][4][6][2][17];
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64 || wpb < 1 || wpb > 16 ||
      vecs < 1 || vecs > 2)
    return 0;
  const int iv = vw == 1 ? 0 : vw == 2 ? 1 : vw == 4 ? 2 : 3;
  int il = 0;
  while ((1 << il) < lanes && il < 5) ++il;
  std::atomic<int> &slot = cache[dev][iv][il][vecs - 1][wpb];
  int n = slot.load(std::memory_order_relaxed);
  if (n > 0) return n;
  SpmmFn f = pick_spmm(vw, lanes, vecs, 1);
  if (!f) return 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, f, wpb * 32, 0) != cudaSuccess) return 0;
  slot.store(n, std::memory_order_relaxed);
  return n;
}

// Common argument checks for gnn_spmm / gnn_sddmm.
gnn_status_t check_common(const Plan *p, const gnn_graph_t *g, const char *who) {
  if (!p || !g) return fail(GNN_ERR_INVALID_ARG, "%s: NULL plan or graph", who);
  if (g->nnz != p->info.nnz || g->row_ind != p->row_ind || g->M != p->M ||
      g->row_base != p->row_base)
    return fail(GNN_ERR_INVALID_ARG, "%s: graph does not match the plan", who);
  if (g->nnz > 0 && (!g->row_ind || !g->col_ind))
    return fail(GNN_ERR_INVALID_ARG, "%s: NULL sparse arrays", who);
  int dev = -1;
  cudaGetDevice(&dev);
  if (dev != p->device)
    return fail(GNN_ERR_INVALID_ARG, "%s: plan built for device %d, current %d", who, p->device,
                dev);
  return GNN_OK;
}

// Sparse vector width actually usable for these pointers (HVMA needs aligned bases).
int effective_vws(int vws, const gnn_graph_t *g, const void *extra) {
  while (vws > 1) {
    const size_t al = 4u * vws;
    if (aligned(g->row_ind, al) && aligned(g->col_ind, al) && (!g->val || aligned(g->val, al)) &&
        (!extra || aligned(extra, al)))
      break;
    vws >>= 1;
  }
  return vws;
}

SparseArgs make_args(const Plan *p, const gnn_graph_t *g) {
  SparseArgs a;
  a.row_ind = g->row_ind;
  a.col_ind = g->col_ind;
  a.val = g->val;
  a.row_first = p->row_first;
  a.row_last = p->row_last;
  a.flags = p->flags;
  a.nnz = g->nnz;
  a.num_chunks = p->info.num_chunks;
  a.row_base = g->row_base;
  a.M = g->M;
  a.chunk = p->info.chunk;
  a.K = p->info.K;
  a.slices = p->info.slices;
  a.vecs = p->info.vecs;
  return a;
}

}  // namespace gnn

using namespace gnn;

extern "C" GNN_API gnn_status_t gnn_spmm(gnn_plan_t plan, const gnn_graph_t *g, const float *A,
                                         int64_t lda, float *O, int64_t ldo,
                                         gnn_stream_t stream) {
  const Plan *p = reinterpret_cast<const Plan *>(plan);
  if (gnn_status_t st = check_common(p, g, "gnn_spmm")) return st;
  const gnn_plan_info_t &in = p->info;
  const int K = in.K, VW = in.vw_feat;
  if (g->M == 0) return GNN_OK;
  if (!O || ldo < K || (g->nnz > 0 && (!A || lda < K || lda >= (int64_t(1) << 30))))
    return fail(GNN_ERR_INVALID_ARG, "gnn_spmm: bad dense operand (lda=%lld ldo=%lld K=%d)",
                (long long)lda, (long long)ldo, K);
  if (!aligned(O, 4u * VW) || ldo % VW || (g->nnz > 0 && (!aligned(A, 4u * VW) || lda % VW)))
    return fail(GNN_ERR_UNSUPPORTED,
                "gnn_spmm: A/O must be %d-byte aligned with pitches multiple of %d "
                "(re-plan with force_vw)", 4 * VW, VW);
  cudaStream_t s = (cudaStream_t)stream;
  if (g->nnz == 0) {  // no chunks: O := 0
    cudaError_t e = cudaMemset2DAsync(O, ldo * sizeof(float), 0, K * sizeof(float), g->M, s);
    return e == cudaSuccess ? GNN_OK : cuda_fail(e, "gnn_spmm memset");
  }
  const int vws = effective_vws(in.vw_sparse, g, nullptr);
  SpmmFn f = pick_spmm(VW, in.lanes, in.vecs, vws);
  if (!f) return fail(GNN_ERR_UNSUPPORTED, "gnn_spmm: no kernel for vw=%d L=%d", VW, in.lanes);
  const SparseArgs a = make_args(p, g);
  const int threads = in.warps_per_block * 32;
  {
    const int64_t blocks = (a.num_chunks * 32 + 255) / 256;
    switch (VW) {
      case 1: spmm_prezero_kernel<1><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo); break;
      case 2: spmm_prezero_kernel<2><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo); break;
      case 4: spmm_prezero_kernel<4><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo); break;
      default: spmm_prezero_kernel<8><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo); break;
    }
  }
  f<<<(unsigned)in.num_blocks, threads, 0, s>>>(a, A, lda, O, ldo);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GNN_OK : cuda_fail(e, "gnn_spmm launch");
}
