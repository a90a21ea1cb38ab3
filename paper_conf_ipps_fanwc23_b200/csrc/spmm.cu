// spmm.cu -- hybrid-parallel SpMM for sm_100a (O = S A; Algorithm 1
// is the definition, Algorithm 3 P:168-195 the prior-art GPU design).
//
// Work decomposition: the plan cuts the nnz into chunks of C* consecutive
// nonzeros (equal work per unit, hybrid node/edge parallelism).  Each (chunk,
// K-slice) work item is owned by a lane group of L lanes; every lane holds VW consecutive
// feature columns, so one group gathers L*VW columns of a source row per nonzero with one
// vector load per lane (256-bit at VW = 8 fp32 / 16 bf16).  G = 32/L groups share a warp.
// The chunk's (row, col, val) entries are staged through a per-warp, double-buffered
// shared-memory ring filled by cp.async one tile ahead of use, and read back as
// warp-broadcast shared loads; U feature rows are in flight per lane before the FMAs
// consume them.  Tiles whose nonzeros all belong to one row (for every group of the warp;
// the common case at high degree) take a fast path with no per-nonzero row or bounds
// logic; the others run the general row-switch loop.  A row switch ("row-switch
// procedure") flushes the accumulator: rows wholly inside the chunk get a plain vector
// store, rows shared with a neighbouring chunk (plan flags) a vector atomic add into a row
// zeroed beforehand by spmm_prezero_kernel.  Empty rows are written as zeros by the chunk
// that precedes them, so O is fully overwritten without a memset.
#include <atomic>
#include <climits>

#include <math.h>

#include "spmm_kernel.cuh"

namespace gnn {

// Initialise every row shared by several chunks before the atomics land on it (0 for
// sum, -inf / +inf for max / min): the row is initialised by the chunk in which it starts
// (tail flag set, and not a pure continuation of an earlier chunk's row).  One warp per
// chunk.
template <int VW>
__global__ void spmm_prezero_kernel(const SparseArgs a, float *__restrict__ O,
                                    const int64_t ldo, const float init) {
  // let a programmatic dependent (the SpMM of gnn_plan_spmm_sddmm) launch right away
  asm volatile("griddepcontrol.launch_dependents;");
  const int64_t c = a.c_begin + (((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5);
  const int lane = threadIdx.x & 31;
  if (c >= a.c_end) return;
  int32_t rf, rl;
  uint32_t fl;
  chunk_rows(a, c, rf, rl, fl);
  if (!(fl & 2u)) return;
  if ((fl & 1u) && rf == rl) return;
  float *o = O + ((int64_t)rl - a.row_base) * ldo;
  float z[VW];
#pragma unroll
  for (int v = 0; v < VW; ++v) z[v] = init;
  for (int k = lane * VW; k < a.K; k += 32 * VW) st_vec<VW>(o + k, z);
}

// Deterministic plans: every row split across chunks is combined from the per-chunk
// partials in chunk order (no atomics): one warp per chunk in which such a row starts,
// lanes over the K columns.  AGG: 0 sum, 1 max, 2 min.
template <int AGG>
__global__ void spmm_fixup_kernel(const SparseArgs a, float *__restrict__ O, const int64_t ldo) {
  const int64_t c0 = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (c0 >= a.num_chunks) return;
  const uint32_t f0 = a.flags[c0];
  if (!(f0 & 2u)) return;
  const int32_t rf0 = a.row_first[c0], r = a.row_last[c0];
  if ((f0 & 1u) && rf0 == r) return;  // the row started in an earlier chunk
  const int K = a.K;
  float *o = O + ((int64_t)r - a.row_base) * ldo;
  for (int k = lane; k < K; k += 32) {
    float acc = a.carry[(c0 * 2 + (r == rf0 ? 0 : 1)) * (int64_t)K + k];
    for (int64_t c = c0 + 1; c < a.num_chunks; ++c) {  // chunk c starts with row r
      const float v = a.carry[(c * 2) * (int64_t)K + k];
      acc = AGG == 0 ? acc + v : (AGG == 1 ? fmaxf(acc, v) : fminf(acc, v));
      if (!((a.flags[c] & 2u) && a.row_last[c] == r)) break;
    }
    o[k] = (AGG == 0 && a.accum) ? o[k] + acc : acc;
  }
}

// Mean aggregator: O[r] *= 1 / (nonzeros of row r) for rows with nonzeros (row_ptr read
// relative to row_ptr[0]).  One warp per row.
__global__ void spmm_row_mean_kernel(const int32_t *__restrict__ row_ptr, int64_t M, int32_t K,
                                     float *__restrict__ O, int64_t ldo) {
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t r = warp; r < M; r += nwarps) {
    const int32_t cnt = row_ptr[r + 1] - row_ptr[r];
    if (cnt <= 0) continue;
    const float s = 1.0f / (float)cnt;
    float *o = O + r * ldo;
    for (int k = lane; k < K; k += 32) o[k] *= s;
  }
}

SpmmFn pick_spmm(int dtype, int vw, int L, int R, int vws, int agg = kAggSum) {
  if (dtype == GNN_BF16) return agg == kAggSum ? pick_spmm_bf16(vw, L, R, vws) : nullptr;
  if (agg == kAggMax) return pick_spmm_f32_max(vw, L, R, vws);
  if (agg == kAggMin) return pick_spmm_f32_min(vw, L, R, vws);
  return pick_spmm_f32(vw, L, R, vws);
}

#ifndef GNN_SPMM_BF16_R2_WIDEN
#define GNN_SPMM_BF16_R2_WIDEN 1  // measured: bf16 K=256 SpMM 4.30 -> 3.96 ms (r01_sweep43)
#endif
#ifndef GNN_SPMM_F32_R2_WIDEN
#define GNN_SPMM_F32_R2_WIDEN 1  // measured at 80 registers: C4 K=256 5.94 -> 5.87 ms, C5
                                 // 8.74 -> 8.61 (r02_s1; at 128 registers C5 lost 16%)
#endif
// The lane shape the sum kernel is launched with: rows of two vectors per lane (R = 2)
// run as one vector per lane on twice the lanes -- half the accumulators per lane, each
// output element summed in the same order (identical results).
bool spmm_widen(int dtype, int agg, int lanes, int vecs) {
  return agg == kAggSum && vecs == 2 && lanes <= 16 &&
         ((dtype == GNN_BF16 && GNN_SPMM_BF16_R2_WIDEN) ||
          (dtype == GNN_F32 && GNN_SPMM_F32_R2_WIDEN));
}

// Cached per (device, dtype, vw, lanes, vecs, wpb): the occupancy API is a host-side
// query but not free, and plans are rebuilt every step in graph-sampling training (C3).
// The query is for the kernel the sum launcher actually runs (after the widen remap).
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
  if (spmm_widen(dtype, kAggSum, lanes, vecs)) {
    lanes *= 2;
    vecs = 1;
  }
  SpmmFn f = pick_spmm(dtype, vw, lanes, vecs, 1);
  if (!f) return 0;
  // the plan's vw_sparse is not known yet: size the tiles for the widest (4)
  const size_t smem = (size_t)wpb * spmm_tile_bytes_per_warp(lanes, 4);
  // only ever raise the per-function limit above the 48 KB default (a smaller value would
  // make later launches with more warps per block fail); launches re-raise it as needed
  if (smem > 48 * 1024 &&
      cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) !=
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
  a.accum = 0;
  a.carry = nullptr;
  a.c_begin = 0;
  a.c_end = a.num_chunks;
  a.inline_plan = p->inline_plan ? 1 : 0;
  return a;
}

}  // namespace gnn

using namespace gnn;

namespace gnn {
// c0 < 0: the whole plan; else chunks [c0, c1) only (sum, overwrite, atomic plans: the
// pipelined host path), without the pre-zero pass: the caller runs launch_spmm_prezero
// over the whole plan first, so ranges may then run concurrently.
gnn_status_t launch_spmm(const Plan *p, const gnn_graph_t *g, const void *A, int64_t lda,
                         float *O, int64_t ldo, gnn_stream_t stream, int dtype, int agg_api,
                         int accumulate, const char *who, int64_t c0, int64_t c1) {
  if (gnn_status_t st = check_common(p, g, who)) return st;
  const gnn_plan_info_t &in = p->info;
  if (in.feature_dtype != dtype)
    return fail(GNN_ERR_INVALID_ARG, "%s: plan was built for feature_dtype %d", who,
                in.feature_dtype);
  if (agg_api < GNN_AGG_SUM || agg_api > GNN_AGG_MIN || (accumulate != 0 && accumulate != 1))
    return fail(GNN_ERR_INVALID_ARG, "%s: bad aggregator %d / accumulate %d", who, agg_api,
                accumulate);
  if (accumulate && agg_api != GNN_AGG_SUM)
    return fail(GNN_ERR_UNSUPPORTED, "%s: accumulate (beta = 1) is defined for sum only", who);
  if (agg_api == GNN_AGG_MEAN && g->M > 0 && !g->row_ptr)
    return fail(GNN_ERR_INVALID_ARG, "%s: the mean aggregator needs graph->row_ptr", who);
  const int agg = agg_api == GNN_AGG_MAX ? kAggMax : agg_api == GNN_AGG_MIN ? kAggMin : kAggSum;
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
  if (g->nnz == 0) {  // no chunks: O := 0 (beta = 1: unchanged)
    if (accumulate) return GNN_OK;
    cudaError_t e = cudaMemset2DAsync(O, ldo * sizeof(float), 0, K * sizeof(float), g->M, s);
    return e == cudaSuccess ? GNN_OK : cuda_fail(e, "gnn_spmm memset");
  }
  int vws = effective_vws(in.vw_sparse, g, nullptr);
#ifndef GNN_SPMM_BF16_R2_VWS2
#define GNN_SPMM_BF16_R2_VWS2 1  // measured: bf16 K=256 SpMM 4.43 -> 4.30 ms (r01_sweep39)
#endif
#if GNN_SPMM_BF16_R2_VWS2
  // bf16 rows of two 32-byte vectors per lane (R = 2): with 4-wide sparse vectors the
  // batch holds 4 nonzeros x 2 vectors of 16 bf16 in flight, which spills at the 128-register
  // budget (ptxas: 308 B); 2-wide sparse copies halve the batch and remove the spill
  if (dtype == GNN_BF16 && in.vecs == 2 && vws > 2) vws = 2;
#endif
  int lanes = in.lanes, vecs = in.vecs;
  if (spmm_widen(dtype, agg, lanes, vecs)) {
    lanes *= 2;
    vecs = 1;
    vws = effective_vws(in.vw_sparse, g, nullptr);
    if (vws > 2) vws = 2;
  }
  SpmmFn f = pick_spmm(dtype, VW, lanes, vecs, vws, agg);
  if (!f)
    return fail(GNN_ERR_UNSUPPORTED, "%s: no kernel for vw=%d L=%d agg=%d dtype=%d", who, VW,
                lanes, agg_api, dtype);
  SparseArgs a = make_args(p, g);
  a.accum = accumulate;
  a.carry = p->carry;
  if (c0 >= 0) {
    if (c1 < c0 || c1 > a.num_chunks || a.carry || agg_api != GNN_AGG_SUM)
      return fail(GNN_ERR_INVALID_ARG, "%s: bad chunk range [%lld, %lld)", who, (long long)c0,
                  (long long)c1);
    if (c1 == c0) return GNN_OK;
    a.c_begin = c0;
    a.c_end = c1;
  }
  const int64_t nch = a.c_end - a.c_begin;
  const int threads = in.warps_per_block * 32;
  if (!accumulate && !a.carry && c0 < 0) {
    const int64_t blocks = (nch * 32 + 255) / 256;
    const float init = agg == kAggMax ? -INFINITY : agg == kAggMin ? INFINITY : 0.f;
    switch (VO) {
      case 1: spmm_prezero_kernel<1><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo, init); break;
      case 2: spmm_prezero_kernel<2><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo, init); break;
      case 4: spmm_prezero_kernel<4><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo, init); break;
      default: spmm_prezero_kernel<8><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo, init); break;
    }
  }
  const size_t smem = (size_t)in.warps_per_block * spmm_tile_bytes_per_warp(lanes, vws);
  if (smem > 48 * 1024) {
    cudaError_t e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return cuda_fail(e, "gnn_spmm smem attribute");
  }
  const int64_t per_block = (int64_t)(32 / lanes) * in.warps_per_block;  // items / block
  const int64_t grid = (nch * in.slices + per_block - 1) / per_block;
  if (p->inline_plan) {
    // programmatic dependent launch: the SpMM starts while the pre-zero drains and waits
    // for it only before its first atomic flush (spmm_kernel, griddepcontrol.wait)
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3((unsigned)grid);
    cfg.blockDim = dim3(threads);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    cudaError_t e = cudaLaunchKernelEx(&cfg, f, a, A, lda, O, ldo);
    if (e != cudaSuccess) return cuda_fail(e, "gnn_spmm launch (PDL)");
  } else {
    f<<<(unsigned)grid, threads, smem, s>>>(a, A, lda, O, ldo);
  }
  if (a.carry) {
    const int64_t blocks = (a.num_chunks * 32 + 255) / 256;
    if (agg == kAggMax) spmm_fixup_kernel<1><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo);
    else if (agg == kAggMin) spmm_fixup_kernel<2><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo);
    else spmm_fixup_kernel<0><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo);
  }
  if (agg_api == GNN_AGG_MEAN) {
    DeviceInfo d;
    device_info(&d);
    int64_t blocks = (g->M * 32 + 255) / 256;
    if (blocks > (int64_t)d.num_sms * 16) blocks = (int64_t)d.num_sms * 16;
    spmm_row_mean_kernel<<<(unsigned)blocks, 256, 0, s>>>(g->row_ptr, g->M, K, O, ldo);
  }
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GNN_OK : cuda_fail(e, "gnn_spmm launch");
}
}  // namespace gnn

namespace gnn {
gnn_status_t launch_spmm_prezero(const Plan *p, const gnn_graph_t *g, float *O, int64_t ldo,
                                 gnn_stream_t stream, int64_t c0, int64_t c1) {
  if (gnn_status_t st = check_common(p, g, "spmm prezero")) return st;
  if (p->info.num_chunks == 0) return GNN_OK;
  SparseArgs a = make_args(p, g);
  if (c0 >= 0) {
    if (c1 < c0 || c1 > a.num_chunks)
      return fail(GNN_ERR_INVALID_ARG, "spmm prezero: bad chunk range [%lld, %lld)",
                  (long long)c0, (long long)c1);
    if (c1 == c0) return GNN_OK;
    a.c_begin = c0;
    a.c_end = c1;
  }
  const int VW = p->info.vw_feat, VO = VW < 8 ? VW : 8;
  const int64_t blocks = ((a.c_end - a.c_begin) * 32 + 255) / 256;
  cudaStream_t s = (cudaStream_t)stream;
  switch (VO) {
    case 1: spmm_prezero_kernel<1><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo, 0.f); break;
    case 2: spmm_prezero_kernel<2><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo, 0.f); break;
    case 4: spmm_prezero_kernel<4><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo, 0.f); break;
    default: spmm_prezero_kernel<8><<<(unsigned)blocks, 256, 0, s>>>(a, O, ldo, 0.f); break;
  }
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GNN_OK : cuda_fail(e, "spmm prezero launch");
}
}  // namespace gnn

extern "C" GNN_API gnn_status_t gnn_spmm(gnn_plan_t plan, const gnn_graph_t *g, const float *A,
                                         int64_t lda, float *O, int64_t ldo,
                                         gnn_stream_t stream) {
  return launch_spmm(reinterpret_cast<const Plan *>(plan), g, A, lda, O, ldo, stream, GNN_F32,
                     GNN_AGG_SUM, 0, "gnn_spmm", -1, 0);
}

extern "C" GNN_API gnn_status_t gnn_spmm_bf16(gnn_plan_t plan, const gnn_graph_t *g,
                                              const uint16_t *A, int64_t lda, float *O,
                                              int64_t ldo, gnn_stream_t stream) {
  return launch_spmm(reinterpret_cast<const Plan *>(plan), g, A, lda, O, ldo, stream, GNN_BF16,
                     GNN_AGG_SUM, 0, "gnn_spmm_bf16", -1, 0);
}

extern "C" GNN_API gnn_status_t gnn_spmm_ex(gnn_plan_t plan, const gnn_graph_t *g, const void *A,
                                            int64_t lda, float *O, int64_t ldo, int32_t agg,
                                            int32_t accumulate, gnn_stream_t stream) {
  const Plan *p = reinterpret_cast<const Plan *>(plan);
  const int dtype = p ? p->info.feature_dtype : GNN_F32;
  return launch_spmm(p, g, A, lda, O, ldo, stream, dtype, agg, accumulate, "gnn_spmm_ex", -1, 0);
}
