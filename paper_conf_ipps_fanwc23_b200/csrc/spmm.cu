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

#include "spmm_kernel.cuh"

namespace gnn {

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

SpmmFn pick_spmm(int dtype, int vw, int L, int R, int vws) {
  return dtype == GNN_BF16 ? pick_spmm_bf16(vw, L, R, vws) : pick_spmm_f32(vw, L, R, vws);
}

// Cached per (device, dtype, vw, lanes, vecs, wpb): the occupancy API is a host-side
// query but not free, and plans are rebuilt every step in graph-sampling training (C3).
int spmm_active_blocks_per_sm(int dtype, int vw, int lanes, int vecs, int wpb) {
  static std::atomic<int> cache[64][2][5][6][2][17];
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64 || wpb < 1 || wpb > 16 ||
      vecs < 1 || vecs > 2 || dtype < 0 || dtype > 1)
    return 0;
  int iv = 0;
  while ((1 << iv) < vw && iv < 4) ++iv;
  int il = 0;
  while ((1 << il) < lanes && il < 5) ++il;
  std::atomic<int> &slot = cache[dev][dtype][iv][il][vecs - 1][wpb];
  int n = slot.load(std::memory_order_relaxed);
  if (n > 0) return n;
  SpmmFn f = pick_spmm(dtype, vw, lanes, vecs, 1);
  if (!f) return 0;
  // the plan's vw_sparse is not known yet: size the tiles for the widest (4)
  const size_t smem = (size_t)wpb * spmm_tile_bytes_per_warp(lanes, 4);
  if (cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) !=
      cudaSuccess)
    return 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, f, wpb * 32, smem) != cudaSuccess)
    return 0;
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
#ifndef GNN_VWS_MAX
#define GNN_VWS_MAX 4  // widest sparse vector the kernels use (tuning knob)
#endif
int effective_vws(int vws, const gnn_graph_t *g, const void *extra) {
  while (vws > GNN_VWS_MAX) vws >>= 1;
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

namespace gnn {
static gnn_status_t launch_spmm(const Plan *p, const gnn_graph_t *g, const void *A, int64_t lda,
                                float *O, int64_t ldo, gnn_stream_t stream, int dtype,
                                const char *who) {
  if (gnn_status_t st = check_common(p, g, who)) return st;
  const gnn_plan_info_t &in = p->info;
  if (in.feature_dtype != dtype)
    return fail(GNN_ERR_INVALID_ARG, "%s: plan was built for feature_dtype %d", who,
                in.feature_dtype);
  const int K = in.K, VW = in.vw_feat;
  const int ES = dtype == GNN_BF16 ? 2 : 4;
  const int VO = VW < 8 ? VW : 8;  // fp32 output vector granule
  if (g->M == 0) return GNN_OK;
  if (!O || ldo < K || (g->nnz > 0 && (!A || lda < K || lda >= (int64_t(1) << 29))))
    return fail(GNN_ERR_INVALID_ARG, "%s: bad dense operand (lda=%lld ldo=%lld K=%d)", who,
                (long long)lda, (long long)ldo, K);
  if (!aligned(O, 4u * VO) || ldo % VO ||
      (g->nnz > 0 && (!aligned(A, (size_t)ES * VW) || lda % VW)))
    return fail(GNN_ERR_UNSUPPORTED,
                "%s: A must be %d-byte aligned with a pitch multiple of %d, O %d-byte aligned "
                "with a pitch multiple of %d (re-plan with force_vw)",
                who, ES * VW, VW, 4 * VO, VO);
  cudaStream_t s = (cudaStream_t)stream;
  if (g->nnz == 0) {  // no chunks: O := 0
    cudaError_t e = cudaMemset2DAsync(O, ldo * sizeof(float), 0, K * sizeof(float), g->M, s);
    return e == cudaSuccess ? GNN_OK : cuda_fail(e, "gnn_spmm memset");
  }
  const int vws = effective_vws(in.vw_sparse, g, nullptr);
  SpmmFn f = pick_spmm(dtype, VW, in.lanes, in.vecs, vws);
  if (!f) return fail(GNN_ERR_UNSUPPORTED, "%s: no kernel for vw=%d L=%d", who, VW, in.lanes);
  const SparseArgs a = make_args(p, g);
  const int threads = in.warps_per_block * 32;
  {
    const int64_t blocks = (a.num_chunks * 32 + 255) / 256;
    switch (VO) {
      case 1: spmm_prezero_kernel<1><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo); break;
      case 2: spmm_prezero_kernel<2><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo); break;
      case 4: spmm_prezero_kernel<4><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo); break;
      default: spmm_prezero_kernel<8><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo); break;
    }
  }
  const size_t smem = (size_t)in.warps_per_block * spmm_tile_bytes_per_warp(in.lanes, vws);
  if (smem > 48 * 1024) {
    cudaError_t e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return cuda_fail(e, "gnn_spmm smem attribute");
  }
  f<<<(unsigned)in.num_blocks, threads, smem, s>>>(a, A, lda, O, ldo);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GNN_OK : cuda_fail(e, "gnn_spmm launch");
}
}  // namespace gnn

extern "C" GNN_API gnn_status_t gnn_spmm(gnn_plan_t plan, const gnn_graph_t *g, const float *A,
                                         int64_t lda, float *O, int64_t ldo,
                                         gnn_stream_t stream) {
  return launch_spmm(reinterpret_cast<const Plan *>(plan), g, A, lda, O, ldo, stream, GNN_F32,
                     "gnn_spmm");
}

extern "C" GNN_API gnn_status_t gnn_spmm_bf16(gnn_plan_t plan, const gnn_graph_t *g,
                                              const uint16_t *A, int64_t lda, float *O,
                                              int64_t ldo, gnn_stream_t stream) {
  return launch_spmm(reinterpret_cast<const Plan *>(plan), g, A, lda, O, ldo, stream, GNN_BF16,
                     "gnn_spmm_bf16");
}
