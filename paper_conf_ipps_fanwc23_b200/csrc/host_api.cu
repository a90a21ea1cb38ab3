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
constexpr int kMaxK = 16;  // feature widths per gnn_run_host_multi call
inline size_t a256(size_t b) { return (b + 255) & ~size_t(255); }

struct HostLayout {  // offsets inside the workspace; the graph part does not depend on K
  size_t row_ind, col_ind, val, total;
  size_t X[kMaxK], O[kMaxK], out[kMaxK], plan[kMaxK];
};

// graph arrays, then per feature width k: X_k, O_k, S_O_k, plan workspace k (nk = 1 is
// gnn_run_host's layout)
bool layout(int64_t M, int64_t N, int64_t nnz, int32_t nk, const int32_t *K,
            const gnn_plan_opts_t *opts, HostLayout *l) {
  size_t o = 0;
  l->row_ind = o; o += a256(4 * (size_t)nnz);
  l->col_ind = o; o += a256(4 * (size_t)nnz);
  l->val = o;     o += a256(4 * (size_t)nnz);
  for (int k = 0; k < nk; ++k) {
    const size_t pb = gnn_plan_workspace_bytes(M, nnz, K[k], opts);
    if (pb == (size_t)-1) return false;
    l->X[k] = o;    o += a256(4 * (size_t)N * K[k]);
    l->O[k] = o;    o += a256(4 * (size_t)M * K[k]);
    l->out[k] = o;  o += a256(4 * (size_t)nnz);
    l->plan[k] = o; o += a256(pb);
  }
  l->total = o;
  return true;
}
// Internal streams + events of one gnn_run_host call, released on every return path
// (cudaStreamDestroy / cudaEventDestroy defer the release until pending work is done).
struct CallResources {
  cudaStream_t sin = nullptr, sout = nullptr, s2 = nullptr;
  cudaEvent_t ev[8] = {};
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

GNN_API size_t gnn_run_host_multi_workspace_bytes(int64_t M, int64_t N, int64_t nnz,
                                                  int32_t nk, const int32_t *K,
                                                  const gnn_plan_opts_t *opts) {
  if (M < 0 || N < 0 || nnz < 0 || nk < 1 || nk > kMaxK || !K) return (size_t)-1;
  for (int k = 0; k < nk; ++k)
    if (K[k] < 1) return (size_t)-1;
  HostLayout l;
  return layout(M, N, nnz, nk, K, opts, &l) ? l.total : (size_t)-1;
}

GNN_API size_t gnn_run_host_workspace_bytes(int64_t M, int64_t N, int64_t nnz, int32_t K,
                                            const gnn_plan_opts_t *opts) {
  return gnn_run_host_multi_workspace_bytes(M, N, nnz, 1, &K, opts);
}

GNN_API gnn_status_t gnn_run_host_multi(const gnn_graph_t *gh, int32_t upload_graph, int32_t nk,
                                        const int32_t *Ks, const float *const *X_host,
                                        float *const *O_host, float *const *out_host,
                                        const gnn_plan_opts_t *opts, void *workspace,
                                        size_t ws_bytes, gnn_stream_t stream) {
  if (!gh || gh->M < 0 || gh->N < 0 || gh->nnz < 0 || nk < 1 || nk > kMaxK || !Ks || !X_host ||
      gh->row_base < 0 || gh->row_base + gh->M > gh->N ||
      (gh->nnz > 0 && (!gh->row_ind || !gh->col_ind)))
    return fail(GNN_ERR_INVALID_ARG,
                "gnn_run_host: bad arguments (host arrays, rows [row_base, row_base + M) of an "
                "N-node graph, 1 <= nk <= %d)",
                kMaxK);
  for (int k = 0; k < nk; ++k)
    if (Ks[k] < 1 || !X_host[k])
      return fail(GNN_ERR_INVALID_ARG, "gnn_run_host: K[%d] = %d / X_host[%d] missing", k, Ks[k],
                  k);
  if (opts && opts->feature_dtype != GNN_F32)
    return fail(GNN_ERR_UNSUPPORTED, "gnn_run_host: fp32 features only");
  HostLayout l;
  if (!layout(gh->M, gh->N, gh->nnz, nk, Ks, opts, &l))
    return fail(GNN_ERR_INVALID_ARG, "gnn_run_host: %s", gnn_last_error());
  if (!workspace || ws_bytes < l.total || !aligned(workspace, 256))
    return fail(GNN_ERR_WORKSPACE, "gnn_run_host: workspace %zu B (need %zu B, 256-B aligned)",
                ws_bytes, l.total);
  char *w = (char *)workspace;
  cudaStream_t s = (cudaStream_t)stream;  // compute runs on the caller's stream (+ s2)
  const int64_t nnz = gh->nnz, M = gh->M, N = gh->N, r0 = gh->row_base;
  const bool up = upload_graph && nnz > 0;
  // Events are re-recorded for every piece: a stream wait captures the event's most recent
  // record at the time it is enqueued, so a fixed set of 8 serves the whole call.
  CallResources res;
  cudaEvent_t ev_entry, ev_ri, ev_x, ev_done, ev_pz, ev_in, ev_o, ev_e;
  cudaError_t e = cudaStreamCreateWithFlags(&res.sin, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&res.sout, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&res.s2, cudaStreamNonBlocking);
  cudaEvent_t *evs[8] = {&ev_entry, &ev_ri, &ev_x, &ev_done, &ev_pz, &ev_in, &ev_o, &ev_e};
  for (int i = 0; i < 8 && e == cudaSuccess; ++i) e = res.event(evs[i]);
  // everything earlier on the caller's stream (e.g. the previous call still reading this
  // workspace) happens before this call's copies
  if (e == cudaSuccess) e = cudaEventRecord(ev_entry, s);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(res.sin, ev_entry, 0);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(res.sout, ev_entry, 0);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(res.s2, ev_entry, 0);
  if (e != cudaSuccess) return cuda_fail(e, "gnn_run_host streams/events");
  // copy-in stream: RowInd (the plan kernels read all of it), X_0, ColInd/Value piece by
  // piece (piece p computes while piece p+1 is in flight), then X_1, X_2, ...
  if (up) {
    e = cudaMemcpyAsync(w + l.row_ind, gh->row_ind, 4 * nnz, cudaMemcpyHostToDevice, res.sin);
    if (e == cudaSuccess) e = cudaEventRecord(ev_ri, res.sin);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(s, ev_ri, 0);
    if (e != cudaSuccess) return cuda_fail(e, "gnn_run_host graph upload");
  }
  gnn_graph_t gd = *gh;
  gd.row_ptr = nullptr;
  gd.row_ind = (const int32_t *)(w + l.row_ind);
  gd.col_ind = (const int32_t *)(w + l.col_ind);
  gd.val = gh->val ? (const float *)(w + l.val) : nullptr;
  struct PlanGuard {
    gnn_plan_t p[kMaxK] = {};
    ~PlanGuard() {
      for (gnn_plan_t q : p)
        if (q) gnn_plan_destroy(q);
    }
  } plans;
  // every plan (GPU plan kernel) and every pre-zero pass up front on the caller's stream:
  // afterwards the pieces are independent and alternate between the two compute streams
  // (one piece's tail wave overlaps the next piece)
  const bool det = opts && opts->deterministic;
  for (int k = 0; k < nk; ++k) {
    if (gnn_status_t st = gnn_plan_create(&gd, Ks[k], opts, w + l.plan[k],
                                          gnn_plan_workspace_bytes(M, nnz, Ks[k], opts), stream,
                                          &plans.p[k]))
      return st;
    if (O_host && O_host[k] && !det && nnz > 0)
      if (gnn_status_t st = launch_spmm_prezero(reinterpret_cast<const Plan *>(plans.p[k]), &gd,
                                                (float *)(w + l.O[k]), Ks[k], stream))
        return st;
  }
  if ((e = cudaEventRecord(ev_pz, s)) == cudaSuccess) e = cudaStreamWaitEvent(res.s2, ev_pz, 0);
  if (e != cudaSuccess) return cuda_fail(e, "gnn_run_host compute stream");
  gnn_status_t st = GNN_OK;
  int64_t piece_no = 0;
  for (int k = 0; k < nk && st == GNN_OK; ++k) {
    const int32_t K = Ks[k];
    const Plan *plan = reinterpret_cast<const Plan *>(plans.p[k]);
    const float *X = (const float *)(w + l.X[k]);
    float *O = (float *)(w + l.O[k]), *out = (float *)(w + l.out[k]);
    float *Oh = O_host ? O_host[k] : nullptr, *Eh = out_host ? out_host[k] : nullptr;
    if (N > 0) {
      e = cudaMemcpyAsync(w + l.X[k], X_host[k], 4 * (size_t)N * K, cudaMemcpyHostToDevice,
                          res.sin);
      if (e != cudaSuccess) { st = cuda_fail(e, "gnn_run_host X upload"); break; }
    }
    if ((e = cudaEventRecord(ev_x, res.sin)) == cudaSuccess) e = cudaStreamWaitEvent(s, ev_x, 0);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(res.s2, ev_x, 0);
    if (e != cudaSuccess) { st = cuda_fail(e, "gnn_run_host event"); break; }
    const int64_t nch = plan->info.num_chunks, C = plan->info.chunk;
    // deterministic plans combine split rows after the whole SpMM: one piece
    const int P = (nnz == 0 || det) ? 1 : (int)(host_pieces(nnz) < nch ? host_pieces(nnz) : nch);
    const bool whole = P == 1;  // whole-plan launches (pre-zero / fix-up inside) when unpipelined
    int64_t rows_done = 0;
    for (int p = 0; p < P && st == GNN_OK; ++p, ++piece_no) {
      const int64_t c0 = nch * p / P, c1 = nch * (p + 1) / P;
      const int64_t b = c0 * C, en = c1 * C < nnz ? c1 * C : nnz;  // this piece's nonzeros
      cudaStream_t sc = (piece_no & 1) ? res.s2 : s;
      if (k == 0 && up && en > b) {  // the graph arrives with the first feature width
        e = cudaMemcpyAsync(w + l.col_ind + 4 * b, gh->col_ind + b, 4 * (en - b),
                            cudaMemcpyHostToDevice, res.sin);
        if (e == cudaSuccess && gh->val)
          e = cudaMemcpyAsync(w + l.val + 4 * b, gh->val + b, 4 * (en - b),
                              cudaMemcpyHostToDevice, res.sin);
        if (e == cudaSuccess) e = cudaEventRecord(ev_in, res.sin);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(sc, ev_in, 0);  // (after X_0: in order)
        if (e != cudaSuccess) { st = cuda_fail(e, "gnn_run_host piece upload"); break; }
      }
      if (Oh) {
        st = launch_spmm(plan, &gd, X, K, O, K, sc, GNN_F32, GNN_AGG_SUM, 0, "gnn_run_host spmm",
                         whole ? -1 : c0, c1);
        if (st != GNN_OK) break;
        // rows final once pieces 0..p are done: up to this piece's last row, minus that
        // row if it continues into the next piece (whose first chunk also zeroes the empty
        // rows before it).  The copy-out stream waits for every piece in order.
        int64_t done = M;  // (local rows: global row id - row_base)
        if (p + 1 < P) {
          const int32_t rl = gh->row_ind[en - 1];
          done = (gh->row_ind[en] == rl ? rl : (int64_t)rl + 1) - r0;
        }
        e = cudaEventRecord(ev_o, sc);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(res.sout, ev_o, 0);
        if (e == cudaSuccess && done > rows_done)
          e = cudaMemcpyAsync(Oh + rows_done * K, O + rows_done * K,
                              4 * (size_t)(done - rows_done) * K, cudaMemcpyDeviceToHost,
                              res.sout);
        if (e != cudaSuccess) { st = cuda_fail(e, "gnn_run_host O download"); break; }
        if (done > rows_done) rows_done = done;
      }
      if (Eh && en > b) {
        // A1 = the shard's own rows of X (destination rows), A2T = all of X
        st = launch_sddmm(plan, &gd, X + r0 * K, K, X, K, out, sc, GNN_F32,
                          "gnn_run_host sddmm", whole ? -1 : c0, c1);
        if (st != GNN_OK) break;
        e = cudaEventRecord(ev_e, sc);
        if (e == cudaSuccess) e = cudaStreamWaitEvent(res.sout, ev_e, 0);
        if (e == cudaSuccess)
          e = cudaMemcpyAsync(Eh + b, out + b, 4 * (size_t)(en - b), cudaMemcpyDeviceToHost,
                              res.sout);
        if (e != cudaSuccess) { st = cuda_fail(e, "gnn_run_host S_O download"); break; }
      }
    }
  }
  // the caller's stream covers every copy and kernel of this call (the copy-out stream
  // waited for every piece; s2 is joined explicitly for calls without outputs)
  cudaError_t e2 = cudaEventRecord(ev_done, res.sout);
  if (e2 == cudaSuccess) e2 = cudaStreamWaitEvent(s, ev_done, 0);
  if (e2 == cudaSuccess) e2 = cudaEventRecord(ev_done, res.s2);
  if (e2 == cudaSuccess) e2 = cudaStreamWaitEvent(s, ev_done, 0);
  if (e2 == cudaSuccess) e2 = cudaEventRecord(ev_done, res.sin);
  if (e2 == cudaSuccess) e2 = cudaStreamWaitEvent(s, ev_done, 0);
  if (e2 != cudaSuccess && st == GNN_OK) st = cuda_fail(e2, "gnn_run_host join");
  return st;
}

GNN_API gnn_status_t gnn_run_host(const gnn_graph_t *gh, int32_t upload_graph, const float *X_host,
                                  int32_t K, float *O_host, float *out_host,
                                  const gnn_plan_opts_t *opts, void *workspace, size_t ws_bytes,
                                  gnn_stream_t stream) {
  return gnn_run_host_multi(gh, upload_graph, 1, &K, &X_host, O_host ? &O_host : nullptr,
                            out_host ? &out_host : nullptr, opts, workspace, ws_bytes, stream);
}

}  // extern "C"
