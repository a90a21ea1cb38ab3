// plan.cu -- Dynamic Task Partition + HVMA candidate set:
// host-side choice of the chunk size C* (scalar integer arithmetic, no device
// reads, no sync) and the device plan kernel that tabulates, per chunk, its first
// and last row and whether those rows continue into the neighbouring chunks (the
// node boundaries the hybrid-parallel kernels must respect).
#include <cuda_runtime.h>
#include <stdlib.h>
#include <string.h>

#include <new>

#include "internal.cuh"

namespace gnn {

namespace {

// NnzPerWarp candidate set.
constexpr int32_t kCand[6] = {8, 32, 64, 128, 256, 512};

inline int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }
inline size_t align256(size_t b) { return (b + 255) & ~size_t(255); }

// InEq. (5) RHS in integer form (DESIGN.md "Plan rule" step 4).
inline int64_t blocks_for(int64_t nnz, int64_t C, int64_t S, int64_t G, int64_t WPB) {
  return cdiv(cdiv(cdiv(nnz, C) * S, G), WPB);
}

gnn_status_t make_info(int64_t M, int64_t nnz, int32_t K, const gnn_plan_opts_t *opts,
                       gnn_plan_info_t *info) {
  gnn_plan_opts_t o{};
  if (opts) o = *opts;
  const int32_t alpha = o.alpha ? o.alpha : 2;
  // WarpsPerBlock (no value given; DESIGN reading 13): 2 -- at the same resident
  // warps per SM, 4-warp blocks measured 1-3% faster than 8 (profiles/r02_s1) and 2-warp
  // blocks 0-1.6% faster than 4 (C4 fp32 / bf16, C5 bf16; C5 fp32 equal; r02_s22/s23)
  const int32_t wpb = o.warps_per_block ? o.warps_per_block : 2;
  if (M < 0 || nnz < 0 || nnz >= (int64_t(1) << 31) || K < 1 || alpha < 1 || wpb < 1 ||
      wpb * 32 > kMaxThreads || o.force_chunk < 0 || o.deterministic < 0 ||
      o.deterministic > 1 || o.no_locality < 0 || o.no_locality > 1)
    return fail(GNN_ERR_INVALID_ARG,
                "plan: bad arguments (nnz=%lld K=%d alpha=%d wpb=%d force_chunk=%d det=%d)",
                (long long)nnz, K, alpha, wpb, o.force_chunk, o.deterministic);
  // step 1: feature vector width (elements of the feature dtype) from K alone, or forced;
  // the widest of 256/128/64/32-bit that divides the row
  const int32_t dt = o.feature_dtype;
  if (dt != GNN_F32 && dt != GNN_BF16)
    return fail(GNN_ERR_INVALID_ARG, "plan: feature_dtype %d unknown", dt);
  const int32_t vmax = dt == GNN_BF16 ? 16 : 8, vmin = dt == GNN_BF16 ? 2 : 1;
  int32_t vw;
  if (o.force_vw) {
    bool ok = false;
    for (int32_t v = vmin; v <= vmax; v *= 2) ok |= (o.force_vw == v);
    if (!ok || K % o.force_vw)
      return fail(GNN_ERR_INVALID_ARG, "plan: force_vw=%d invalid for K=%d (dtype %d)",
                  o.force_vw, K, dt);
    vw = o.force_vw;
  } else {
    vw = 0;
    for (int32_t v = vmax; v >= vmin && !vw; v /= 2)
      if (K % v == 0) vw = v;
    if (!vw) return fail(GNN_ERR_INVALID_ARG, "plan: bf16 features need an even K (K=%d)", K);
  }
  // step 2: vectors per lane, lanes per chunk-slice, slices, chunk-slices per warp
  const int64_t need = cdiv(K, vw);  // VW-wide vectors in a feature row
  const int32_t R = need >= 16 ? 2 : 1;
  int32_t L = 1;
  while (L < cdiv(need, R) && L < 32) L *= 2;
  const int32_t S = (int32_t)cdiv(K, (int64_t)L * R * vw);
  const int32_t G = 32 / L;
  // step 3: FullWaveSize (Eqs. 3-4) from the occupancy of the SpMM kernel, unless the
  // caller overrides the device parameters (tests feed the same values to the oracle)
  if (o.num_sms < 0 || o.active_blocks_per_sm < 0 || o.l2_bytes < 0)
    return fail(GNN_ERR_INVALID_ARG, "plan: negative device-parameter override");
  DeviceInfo d;
  if (gnn_status_t st = device_info(&d)) return st;
  const int32_t nsm = o.num_sms ? o.num_sms : d.num_sms;
  const int32_t abs = o.active_blocks_per_sm ? o.active_blocks_per_sm
                                             : spmm_active_blocks_per_sm(dt, vw, L, R, wpb);
  if (abs < 1) return fail(GNN_ERR_CUDA, "plan: occupancy query failed (vw=%d L=%d)", vw, L);
  const int64_t FW = (int64_t)nsm * abs;
  // steps 4-5: the largest candidate satisfying InEq. (5); none -> 8
  int32_t C = 8;
  for (int32_t c : kCand)
    if (blocks_for(nnz, c, S, G, wpb) >= alpha * FW) C = c;
  const int32_t C_dtp = C;
  // step 5b (B200 addition): locality cap.  A full wave holds FW*WPB*G/S chunks, i.e.
  // about that many * C / (nnz / M) rows in flight; after a clustering reorder their
  // feature rows are the L2 working set, so C* is the largest candidate <= C_dtp whose
  // rows in flight fit a quarter of L2 (else 8).
  const int64_t l2 = o.no_locality ? 0 : (o.l2_bytes ? o.l2_bytes : d.l2_bytes);  // 0: cap off
  if (l2 > 0 && nnz > 0 && M > 0) {
    const int64_t eb = dt == GNN_BF16 ? 2 : 4;
    const int64_t rows_fit = (l2 / 4) / ((int64_t)K * eb);
    int32_t Cl = kCand[0];
    for (int32_t c : kCand) {
      if (c > C_dtp) break;
      int64_t rows = ((FW * wpb * G * c) / S) * M / nnz;
      if (rows > M) rows = M;
      if (rows <= rows_fit) Cl = c;
    }
    C = Cl;
    // step 5c (B200 addition, on with the cap): chunk floor 64 where Eq. 5 itself fell
    // below 64.  On graphs that fill fewer than alpha waves (sampled subgraphs) Eq. 5 gives
    // 8 or 32, where the sparse loads are scalar and each chunk's fixed cost dominates;
    // C* = 64 measured faster on every C3 subgraph mix (K=32 0.053 -> 0.044 ms, K=128
    // 0.080 -> 0.073 ms; profiles/r01_sweep45).  A cap below 64 on a graph where Eq. 5
    // was feasible at >= 64 stands (locality, not parallelism, decided it).
    if (C_dtp < 64) C = 64;
  }
  if (o.force_chunk > 0) C = o.force_chunk;
  // step 6: sparse vector width (HVMA)
  int32_t vws = 1;
  if (C >= 128 && C % 4 == 0) vws = 4;
  else if (C >= 64 && C % 2 == 0) vws = 2;
  // step 7
  info->chunk = C;
  info->vw_feat = vw;
  info->vw_sparse = vws;
  info->lanes = L;
  info->vecs = R;
  info->slices = S;
  info->groups = G;
  info->warps_per_block = wpb;
  info->active_blocks_per_sm = abs;
  info->num_sms = nsm;
  info->alpha = alpha;
  info->K = K;
  info->feature_dtype = dt;
  info->chunk_dtp = C_dtp;
  info->M = M;
  info->l2_bytes = l2;
  info->nnz = nnz;
  info->num_chunks = nnz > 0 ? cdiv(nnz, C) : 0;
  info->num_blocks = nnz > 0 ? blocks_for(nnz, C, S, G, wpb) : 0;
  return GNN_OK;
}

// row_first | row_last | flags [| carry: 2 partial rows of K fp32 per chunk when the
// plan is deterministic (split rows are summed in chunk order by a fix-up pass instead of
// with atomics)]
size_t ws_bytes_for(int64_t nch, int32_t K, int32_t deterministic) {
  if (nch == 0) return 0;
  size_t b = 2 * align256(sizeof(int32_t) * nch) + align256(nch);
  if (deterministic) b += align256(sizeof(float) * 2 * (size_t)nch * K);
  return b;
}

// One thread per chunk: Algo 3 lines 2-3 (warp_start = id * NnzPerWarp, end
// clamped to NNZ) and the node-boundary flags of the hybrid strategy.
// Chunks [c0, c1) (the pipelined host path plans piece by piece as the row array lands).
__global__ void plan_kernel(const int32_t *__restrict__ row_ind, int64_t nnz, int32_t C,
                            int64_t c0, int64_t c1, int32_t *__restrict__ row_first,
                            int32_t *__restrict__ row_last, uint8_t *__restrict__ flags) {
  const int64_t c = c0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= c1) return;
  const int64_t s = c * C;
  const int64_t e = s + C < nnz ? s + C : nnz;
  const int32_t rf = row_ind[s], rl = row_ind[e - 1];
  uint8_t f = 0;
  if (s > 0 && row_ind[s - 1] == rf) f |= 1;
  if (e < nnz && row_ind[e] == rl) f |= 2;
  row_first[c] = rf;
  row_last[c] = rl;
  flags[c] = f;
}

}  // namespace
}  // namespace gnn

using namespace gnn;

namespace gnn {
// gnn_plan_create; launch = false leaves the plan arrays to launch_plan_range calls.
gnn_status_t plan_create(const gnn_graph_t *g, int32_t K, const gnn_plan_opts_t *opts,
                         void *workspace, size_t ws_bytes, gnn_stream_t stream, gnn_plan_t *out,
                         bool launch) {
  if (!out) return fail(GNN_ERR_INVALID_ARG, "gnn_plan_create: out is NULL");
  *out = nullptr;
  if (!g || g->M < 0 || g->N < 0 || g->nnz < 0 || g->row_base < 0 ||
      (g->nnz > 0 && (!g->row_ind || !g->col_ind)))
    return fail(GNN_ERR_INVALID_ARG, "gnn_plan_create: bad graph descriptor");
  gnn_plan_info_t info;
  if (gnn_status_t st = make_info(g->M, g->nnz, K, opts, &info)) return st;
  // GNN_VALIDATE=1: check the graph's contents (sortedness, index ranges) before planning
  // -- a debug switch: gnn_validate synchronises the stream
  const char *v = getenv("GNN_VALIDATE");
  if (v && v[0] == '1' && g->nnz > 0)
    if (gnn_status_t st = gnn_validate(g, stream)) return st;
  const int64_t nch = info.num_chunks;
  const int32_t det = opts ? opts->deterministic : 0;
  const size_t need = ws_bytes_for(nch, K, det);
  if (ws_bytes < need || (need > 0 && (!workspace || !aligned(workspace, 256))))
    return fail(GNN_ERR_WORKSPACE, "gnn_plan_create: workspace %zu B (need %zu B, 256-B aligned)",
                ws_bytes, need);
  Plan *p = new (std::nothrow) Plan();
  if (!p) return fail(GNN_ERR_INVALID_ARG, "gnn_plan_create: out of host memory");
  p->info = info;
  p->row_ind = g->row_ind;
  p->M = g->M;
  p->row_base = g->row_base;
  char *w = (char *)workspace;
  p->row_first = (int32_t *)w;
  p->row_last = (int32_t *)(w + align256(sizeof(int32_t) * nch));
  p->flags = (uint8_t *)(w + 2 * align256(sizeof(int32_t) * nch));
  p->carry = det && nch > 0 ? (float *)(w + 2 * align256(sizeof(int32_t) * nch) + align256(nch))
                            : nullptr;
  DeviceInfo d;
  device_info(&d);
  p->device = d.device;
  if (launch && nch > 0) {
    if (gnn_status_t st = launch_plan_range(p, stream, 0, nch)) {
      delete p;
      return st;
    }
  }
  *out = reinterpret_cast<gnn_plan_t>(p);
  return GNN_OK;
}

// Plan kernel over chunks [c0, c1): reads RowInd[c0*C* - 1 .. min(c1*C*, nnz)] only.
gnn_status_t launch_plan_range(const Plan *p, gnn_stream_t stream, int64_t c0, int64_t c1) {
  if (c0 < 0 || c1 > p->info.num_chunks || c1 < c0)
    return fail(GNN_ERR_INVALID_ARG, "plan: bad chunk range [%lld, %lld)", (long long)c0,
                (long long)c1);
  if (c1 == c0) return GNN_OK;
  const int threads = 256;
  plan_kernel<<<(unsigned)cdiv(c1 - c0, threads), threads, 0, (cudaStream_t)stream>>>(
      p->row_ind, p->info.nnz, p->info.chunk, c0, c1, p->row_first, p->row_last, p->flags);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GNN_OK : cuda_fail(e, "plan kernel launch");
}

}  // namespace gnn

extern "C" {

GNN_API size_t gnn_plan_workspace_bytes(int64_t M, int64_t nnz, int32_t K,
                                        const gnn_plan_opts_t *opts) {
  gnn_plan_info_t info;
  if (make_info(M, nnz, K, opts, &info) != GNN_OK) return (size_t)-1;
  return ws_bytes_for(info.num_chunks, K, opts ? opts->deterministic : 0);
}

GNN_API gnn_status_t gnn_plan_create(const gnn_graph_t *g, int32_t K,
                                     const gnn_plan_opts_t *opts, void *workspace,
                                     size_t ws_bytes, gnn_stream_t stream, gnn_plan_t *out) {
  return plan_create(g, K, opts, workspace, ws_bytes, stream, out, true);
}

GNN_API gnn_status_t gnn_plan_info(gnn_plan_t plan, gnn_plan_info_t *info) {
  if (!plan || !info) return fail(GNN_ERR_INVALID_ARG, "gnn_plan_info: NULL argument");
  *info = reinterpret_cast<Plan *>(plan)->info;
  return GNN_OK;
}

GNN_API gnn_status_t gnn_plan_arrays(gnn_plan_t plan, const int32_t **row_first,
                                     const int32_t **row_last, const uint8_t **flags) {
  if (!plan) return fail(GNN_ERR_INVALID_ARG, "gnn_plan_arrays: NULL plan");
  Plan *p = reinterpret_cast<Plan *>(plan);
  if (row_first) *row_first = p->row_first;
  if (row_last) *row_last = p->row_last;
  if (flags) *flags = p->flags;
  return GNN_OK;
}

GNN_API void gnn_plan_destroy(gnn_plan_t plan) { delete reinterpret_cast<Plan *>(plan); }

}  // extern "C"
