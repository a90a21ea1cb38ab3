// host_api.cu -- the end-to-end entry point on HOST buffers (bench.py's e2e path): the
// caller hands host arrays and one device workspace; the library copies the graph and X
// in, plans (GPU plan kernel), runs SpMM and SDDMM, and copies O and S_O out.
// Pipelined over pieces of the plan's chunks on three streams: ColInd/Value of piece p+1
// upload (copy-in stream) while piece p computes (caller's stream) while the finished
// rows / edge values of piece p-1 download (copy-out stream); PCIe is full duplex, so
// the call costs about max(upload, compute, download) instead of their sum.
#include <cuda_runtime.h>
#include <stdlib.h>

#include "internal.cuh"

namespace gnn {
namespace {
constexpr int kMaxPieces = 32;
inline size_t a256(size_t b) { return (b + 255) & ~size_t(255); }

struct HostLayout {  // offsets inside the workspace; the graph part does not depend on K
  size_t row_ind, col_ind, val, X, O, out, plan, total;
};

HostLayout layout(int64_t M, int64_t N, int64_t nnz, int32_t K, size_t plan_bytes) {
  HostLayout l{};
  size_t o = 0;
  l.row_ind = o; o += a256(4 * (size_t)nnz);
  l.col_ind = o; o += a256(4 * (size_t)nnz);
  l.val = o;     o += a256(4 * (size_t)nnz);
  l.X = o;       o += a256(4 * (size_t)N * K);
  l.O = o;       o += a256(4 * (size_t)M * K);
  l.out = o;     o += a256(4 * (size_t)nnz);
  l.plan = o;    o += a256(plan_bytes);
  l.total = o;
  return l;
}
// Internal streams + events of one gnn_run_host call, released on every return path
// (cudaStreamDestroy / cudaEventDestroy defer the release until pending work is done).
struct CallResources {
  cudaStream_t sin = nullptr, sout = nullptr, s2 = nullptr;
  cudaEvent_t ev[3 * kMaxPieces + 5] = {};
  int nev = 0;
  ~CallResources() {
    for (int i = 0; i < nev; ++i) cudaEventDestroy(ev[i]);
    if (s2) cudaStreamDestroy(s2);
    if (sin) cudaStreamDestroy(sin);
    if (sout) cudaStreamDestroy(sout);
  }
  cudaError_t event(cudaEvent_t *e) {
    cudaError_t r = cudaEventCreateWithFlags(&ev[nev], cudaEventDisableTiming);
    if (r == cudaSuccess) *e = ev[nev++];
    return r;
  }
};

// Pieces of the copy/compute pipeline: GNN_HOST_PIECES (tuning knob) or one per 4M
// nonzeros, at most kMaxPieces.
int host_pieces(int64_t nnz) {
  if (const char *e = getenv("GNN_HOST_PIECES")) {
    const int v = atoi(e);
    if (v >= 1) return v < kMaxPieces ? v : kMaxPieces;
  }
  const int64_t p = nnz / (int64_t(4) << 20);
  return p < 1 ? 1 : (p > kMaxPieces ? kMaxPieces : (int)p);
}
}  // namespace
}  // namespace gnn

using namespace gnn;

extern "C" {

GNN_API size_t gnn_run_host_workspace_bytes(int64_t M, int64_t N, int64_t nnz, int32_t K,
                                            const gnn_plan_opts_t *opts) {
  if (M < 0 || N < 0 || nnz < 0 || K < 1) return (size_t)-1;
  const size_t pb = gnn_plan_workspace_bytes(nnz, K, opts);
  if (pb == (size_t)-1) return (size_t)-1;
  return layout(M, N, nnz, K, pb).total;
}

GNN_API gnn_status_t gnn_run_host(const gnn_graph_t *gh, int32_t upload_graph, const float *X_host,
                                  int32_t K, float *O_host, float *out_host,
                                  const gnn_plan_opts_t *opts, void *workspace, size_t ws_bytes,
                                  gnn_stream_t stream) {
  if (!gh || gh->M < 0 || gh->N < 0 || gh->nnz < 0 || K < 1 || !X_host || gh->M != gh->N ||
      gh->row_base != 0 || (gh->nnz > 0 && (!gh->row_ind || !gh->col_ind)))
    return fail(GNN_ERR_INVALID_ARG,
                "gnn_run_host: bad arguments (square graph with host arrays, K >= 1)");
  if (opts && opts->feature_dtype != GNN_F32)
    return fail(GNN_ERR_UNSUPPORTED, "gnn_run_host: fp32 features only");
  const size_t pb = gnn_plan_workspace_bytes(gh->nnz, K, opts);
  if (pb == (size_t)-1) return fail(GNN_ERR_INVALID_ARG, "gnn_run_host: %s", gnn_last_error());
  const HostLayout l = layout(gh->M, gh->N, gh->nnz, K, pb);
  if (!workspace || ws_bytes < l.total || !aligned(workspace, 256))
    return fail(GNN_ERR_WORKSPACE, "gnn_run_host: workspace %zu B (need %zu B, 256-B aligned)",
                ws_bytes, l.total);
  char *w = (char *)workspace;
  cudaStream_t s = (cudaStream_t)stream;  // compute runs on the caller's stream
  const int64_t nnz = gh->nnz, M = gh->M, N = gh->N;
  const bool up = upload_graph && nnz > 0;
  CallResources res;
  cudaEvent_t ev_entry, ev_ri = nullptr, ev_x, ev_done;
  cudaError_t e = cudaStreamCreateWithFlags(&res.sin, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&res.sout, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = res.event(&ev_entry);
  if (e == cudaSuccess) e = res.event(&ev_x);
  if (e == cudaSuccess) e = res.event(&ev_done);
  if (e == cudaSuccess && up) e = res.event(&ev_ri);
  // everything earlier on the caller's stream (e.g. the previous call still reading this
  // workspace) happens before this call's copies
  if (e == cudaSuccess) e = cudaEventRecord(ev_entry, s);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(res.sin, ev_entry, 0);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(res.sout, ev_entry, 0);
  if (e != cudaSuccess) return cuda_fail(e, "gnn_run_host streams/events");
  // copy-in stream: RowInd (the plan kernel reads all of it), X, then ColInd/Value piece
  // by piece so that piece p computes while piece p+1 is in flight
  if (up) {
    e = cudaMemcpyAsync(w + l.row_ind, gh->row_ind, 4 * nnz, cudaMemcpyHostToDevice, res.sin);
    if (e == cudaSuccess) e = cudaEventRecord(ev_ri, res.sin);
    if (e != cudaSuccess) return cuda_fail(e, "gnn_run_host graph upload");
  }
  if (N > 0) {
    e = cudaMemcpyAsync(w + l.X, X_host, 4 * (size_t)N * K, cudaMemcpyHostToDevice, res.sin);
    if (e != cudaSuccess) return cuda_fail(e, "gnn_run_host X upload");
  }
  if ((e = cudaEventRecord(ev_x, res.sin)) != cudaSuccess)
    return cuda_fail(e, "gnn_run_host event");
  gnn_graph_t gd = *gh;
  gd.row_ptr = nullptr;
  gd.row_ind = (const int32_t *)(w + l.row_ind);
  gd.col_ind = (const int32_t *)(w + l.col_ind);
  gd.val = gh->val ? (const float *)(w + l.val) : nullptr;
  if (up && (e = cudaStreamWaitEvent(s, ev_ri, 0)) != cudaSuccess)
    return cuda_fail(e, "gnn_run_host wait");
  gnn_plan_t plan = nullptr;
  if (gnn_status_t st = gnn_plan_create(&gd, K, opts, w + l.plan, pb, stream, &plan)) return st;
  gnn_plan_info_t info;
  gnn_plan_info(plan, &info);
  const float *X = (const float *)(w + l.X);
  float *O = (float *)(w + l.O), *out = (float *)(w + l.out);
  const int64_t nch = info.num_chunks, C = info.chunk;
  // deterministic plans combine split rows after the whole SpMM: one piece
  const int P = (nnz == 0 || (opts && opts->deterministic)) ? 1
                : (int)(host_pieces(nnz) < nch ? host_pieces(nnz) : nch);
  gnn_status_t st = GNN_OK;
  cudaEvent_t ev_pz;
  if ((e = res.event(&ev_pz)) != cudaSuccess) st = cuda_fail(e, "gnn_run_host event");
  const int64_t r0 = P == 1 ? -1 : 0;  // whole-plan launches when unpipelined
  if (st == GNN_OK && O_host && P > 1) {
    // rows shared by chunks are zeroed once for the whole plan, so the pieces are
    // independent and alternate between two compute streams (one piece's tail wave
    // overlaps the next piece)
    st = launch_spmm_prezero(reinterpret_cast<const Plan *>(plan), &gd, O, K, stream);
  }
  if (st == GNN_OK && P > 1) {
    e = cudaStreamCreateWithFlags(&res.s2, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaEventRecord(ev_pz, s);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(res.s2, ev_pz, 0);
    if (e != cudaSuccess) st = cuda_fail(e, "gnn_run_host compute stream");
  }
  int64_t rows_done = 0;
  for (int p = 0; p < P && st == GNN_OK; ++p) {
    const int64_t c0 = nch * p / P, c1 = nch * (p + 1) / P;
    const int64_t b = c0 * C, en = c1 * C < nnz ? c1 * C : nnz;  // this piece's nonzeros
    cudaStream_t sc = (p & 1) ? res.s2 : s;
    cudaEvent_t ev_in, ev_o, ev_e;
    e = res.event(&ev_in);
    if (e == cudaSuccess) e = res.event(&ev_o);
    if (e == cudaSuccess) e = res.event(&ev_e);
    if (e == cudaSuccess && up && en > b) {
      e = cudaMemcpyAsync(w + l.col_ind + 4 * b, gh->col_ind + b, 4 * (en - b),
                          cudaMemcpyHostToDevice, res.sin);
      if (e == cudaSuccess && gh->val)
        e = cudaMemcpyAsync(w + l.val + 4 * b, gh->val + b, 4 * (en - b), cudaMemcpyHostToDevice,
                            res.sin);
    }
    if (e == cudaSuccess) e = cudaEventRecord(ev_in, res.sin);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(sc, ev_in, 0);  // (after X: same stream)
    if (e != cudaSuccess) { st = cuda_fail(e, "gnn_run_host piece upload"); break; }
    if (O_host) {
      st = launch_spmm(reinterpret_cast<const Plan *>(plan), &gd, X, K, O, K, sc, GNN_F32,
                       GNN_AGG_SUM, 0, "gnn_run_host spmm", r0 < 0 ? -1 : c0, c1);
      if (st != GNN_OK) break;
      // rows final once pieces 0..p are done: up to this piece's last row, minus that row
      // if it continues into the next piece (whose first chunk also zeroes the empty rows
      // before it).  The copy-out stream waits for every piece in order.
      int64_t done = M;
      if (p + 1 < P) {
        const int32_t rl = gh->row_ind[en - 1];
        done = gh->row_ind[en] == rl ? rl : (int64_t)rl + 1;
      }
      e = cudaEventRecord(ev_o, sc);
      if (e == cudaSuccess) e = cudaStreamWaitEvent(res.sout, ev_o, 0);
      if (e == cudaSuccess && done > rows_done)
        e = cudaMemcpyAsync(O_host + rows_done * K, O + rows_done * K,
                            4 * (size_t)(done - rows_done) * K, cudaMemcpyDeviceToHost, res.sout);
      if (e != cudaSuccess) { st = cuda_fail(e, "gnn_run_host O download"); break; }
      if (done > rows_done) rows_done = done;
    }
    if (out_host && en > b) {
      st = launch_sddmm(reinterpret_cast<const Plan *>(plan), &gd, X, K, X, K, out, sc, GNN_F32,
                        "gnn_run_host sddmm", r0 < 0 ? -1 : c0, c1);
      if (st != GNN_OK) break;
      e = cudaEventRecord(ev_e, sc);
      if (e == cudaSuccess) e = cudaStreamWaitEvent(res.sout, ev_e, 0);
      if (e == cudaSuccess)
        e = cudaMemcpyAsync(out_host + b, out + b, 4 * (size_t)(en - b), cudaMemcpyDeviceToHost,
                            res.sout);
      if (e != cudaSuccess) { st = cuda_fail(e, "gnn_run_host S_O download"); break; }
    }
  }
  // the caller's stream covers every copy of this call
  if ((e = cudaEventRecord(ev_done, res.sout)) == cudaSuccess) e = cudaStreamWaitEvent(s, ev_done, 0);
  if (e != cudaSuccess && st == GNN_OK) st = cuda_fail(e, "gnn_run_host join");
  gnn_plan_destroy(plan);
  return st;
}

}  // extern "C"
