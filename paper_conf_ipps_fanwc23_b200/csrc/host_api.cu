// host_api.cu -- the end-to-end entry point on HOST buffers (bench.py's e2e path): the
// caller hands host arrays and one device workspace; the library copies the graph and X
// in, plans (GPU plan kernel), runs SpMM and SDDMM, and copies O and S_O out.
// Pipelined over pieces of the nonzeros.  Copy-in stream: the narrow widths' X
// interleaved with the first pieces, the widest X near the end (a piece =
// RowInd/ColInd/Value of a range of nonzeros common to every width); prep
// stream: each piece is planned (plan kernel over the chunks that end inside it) and its
// split rows pre-zeroed, in piece order; two alternating compute streams: SpMM + SDDMM of
// every width whose X has landed (a width catches up on earlier pieces when its X lands);
// copy-out stream: each unit's S_O entries and the O rows that became final.  PCIe is
// full duplex, so the call costs about max(upload, compute, download) instead of their sum.
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>

#include "internal.cuh"

namespace gnn {
namespace {
constexpr int kMaxPieces = 32;
constexpr int kMaxK = 16;  // feature widths per gnn_run_host_multi call
inline size_t a256(size_t b) { return (b + 255) & ~size_t(255); }

// RowInd of nonzeros [b, er) decoded on the device from the CSR offsets of the rows they
// span (the hybrid format's two row encodings): local rows [ra, ra + nr) with device
// offsets rp[0..nr] (read relative to base = row_ptr[0]); one warp per row.
__global__ void csr_range_to_coo_kernel(const int32_t *__restrict__ rp, int64_t nr, int64_t ra,
                                        int64_t base, int64_t b, int64_t er, int64_t row_base,
                                        int32_t *__restrict__ row_ind) {
  const int64_t warp = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
  for (int64_t r = warp; r < nr; r += nwarps) {
    int64_t lo = rp[r] - base, hi = rp[r + 1] - base;
    lo = lo > b ? lo : b;
    hi = hi < er ? hi : er;
    for (int64_t i = lo + lane; i < hi; i += 32) row_ind[i] = (int32_t)(ra + r + row_base);
  }
}

struct HostLayout {  // offsets inside the workspace; the graph part does not depend on K
  size_t row_ptr, row_ind, col_ind, val, total;
  size_t X[kMaxK], O[kMaxK], out[kMaxK], plan[kMaxK];
};

// graph arrays, then per feature width k: X_k, O_k, S_O_k, plan workspace k (nk = 1 is
// gnn_run_host's layout)
bool layout(int64_t M, int64_t N, int64_t nnz, int32_t nk, const int32_t *K,
            const gnn_plan_opts_t *opts, HostLayout *l) {
  size_t o = 0;
  l->row_ptr = o; o += a256(4 * (size_t)(M + 1));
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
  cudaStream_t sin = nullptr, sout = nullptr, s2 = nullptr, sp = nullptr;
  cudaEvent_t ev[8] = {};
  int nev = 0;
  ~CallResources() {
    for (int i = 0; i < nev; ++i) cudaEventDestroy(ev[i]);
    if (s2) cudaStreamDestroy(s2);
    if (sp) cudaStreamDestroy(sp);
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
// GNN_HOST_TRACE=1: timing events at the pipeline's milestones (X uploaded; per piece:
// uploaded, planned, computed, downloaded), printed to stderr as ms since the call's entry
// once the call has finished (synchronises: a measurement aid, not for timed runs).
struct Trace {
  bool on = false;
  cudaEvent_t t0 = nullptr, tx = nullptr;
  cudaEvent_t ev[kMaxPieces][4] = {};
  int n = 0;
  Trace() {
    const char *e = getenv("GNN_HOST_TRACE");
    on = e && atoi(e) > 0;
  }
  cudaEvent_t mk() {
    cudaEvent_t x = nullptr;
    cudaEventCreate(&x);
    return x;
  }
  void entry(cudaStream_t s) {
    if (on) cudaEventRecord(t0 = mk(), s);
  }
  void xdone(cudaStream_t s) {
    if (on) cudaEventRecord(tx = mk(), s);
  }
  void mark(int p, int i, cudaStream_t s) {
    if (!on || p >= kMaxPieces) return;
    cudaEventRecord(ev[p][i] = mk(), s);
    if (p + 1 > n) n = p + 1;
  }
  ~Trace() {
    if (!on) return;
    cudaDeviceSynchronize();
    auto ms = [&](cudaEvent_t e) {
      float t = -1.f;
      if (e) cudaEventElapsedTime(&t, t0, e);
      return t;
    };
    fprintf(stderr, "gnn_run_host trace: copy-in done %.3f ms\n", ms(tx));
    for (int p = 0; p < n; ++p)
      fprintf(stderr, "  piece %2d: in %.3f  planned %.3f  computed %.3f  out %.3f\n", p,
              ms(ev[p][0]), ms(ev[p][1]), ms(ev[p][2]), ms(ev[p][3]));
    for (int p = 0; p < n; ++p)
      for (int i = 0; i < 4; ++i)
        if (ev[p][i]) cudaEventDestroy(ev[p][i]);
    if (tx) cudaEventDestroy(tx);
    if (t0) cudaEventDestroy(t0);
  }
};
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
  // record at the time it is enqueued, so a fixed set serves the whole call.
  CallResources res;
  Trace trace;  // declared after res: reported before the streams are released
  cudaEvent_t ev_entry, ev_done, ev_prep, ev_in, ev_o, ev_e, ev_x;
  cudaError_t e = cudaStreamCreateWithFlags(&res.sin, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&res.sout, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&res.s2, cudaStreamNonBlocking);
  if (e == cudaSuccess) e = cudaStreamCreateWithFlags(&res.sp, cudaStreamNonBlocking);
  cudaEvent_t *evs[7] = {&ev_entry, &ev_done, &ev_prep, &ev_in, &ev_o, &ev_e, &ev_x};
  for (int i = 0; i < 7 && e == cudaSuccess; ++i) e = res.event(evs[i]);
  // everything earlier on the caller's stream (e.g. the previous call still reading this
  // workspace) happens before this call's copies
  if (e == cudaSuccess) e = cudaEventRecord(ev_entry, s);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(res.sin, ev_entry, 0);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(res.sout, ev_entry, 0);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(res.s2, ev_entry, 0);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(res.sp, ev_entry, 0);
  if (e != cudaSuccess) return cuda_fail(e, "gnn_run_host streams/events");
  trace.entry(s);
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
  // the host half of every plan (C*, chunk count: scalar arithmetic, no device reads); the
  // plan kernel runs piece by piece below, as the row array arrives
  for (int k = 0; k < nk; ++k)
    if (gnn_status_t st = plan_create(&gd, Ks[k], opts, w + l.plan[k],
                                      gnn_plan_workspace_bytes(M, nnz, Ks[k], opts), stream,
                                      &plans.p[k], false))
      return st;
  // Pieces are ranges of nonzeros common to every width (width k takes the chunks that
  // end inside the piece).  Deterministic plans combine split rows after the whole SpMM
  // (fix-up pass): one piece.
  const bool det = opts && opts->deterministic;
  const int P = (nnz == 0 || det) ? 1 : host_pieces(nnz);
  const bool whole = P == 1;  // whole-plan launches (pre-zero / fix-up inside)
  // Chunk range of width k in piece p: the chunks that end inside the piece's nonzeros.
  int64_t cb[kMaxK][kMaxPieces + 1];
  for (int k = 0; k < nk; ++k) {
    const Plan *plan = reinterpret_cast<const Plan *>(plans.p[k]);
    cb[k][0] = 0;
    for (int p = 0; p < P; ++p)
      cb[k][p + 1] = p + 1 == P ? plan->info.num_chunks : (nnz * (p + 1) / P) / plan->info.chunk;
  }
  int64_t rows_done[kMaxK] = {};
  int units = 0;  // (width, piece) work units so far: they alternate between two streams
  // SpMM + SDDMM of width k on piece p, then the downloads of what became final.  The
  // stream first waits for the latest prep record (covers pieces 0..p, enqueued in piece
  // order) and, for a width whose X landed after the piece, the latest X record.
  auto compute = [&](int k, int p, bool wait_x, cudaEvent_t ev_x) -> gnn_status_t {
    const int32_t K = Ks[k];
    const Plan *plan = reinterpret_cast<const Plan *>(plans.p[k]);
    const int64_t C = plan->info.chunk, c0 = cb[k][p], c1 = cb[k][p + 1];
    if (!whole && c1 == c0) return GNN_OK;
    cudaStream_t sc = (units++ & 1) ? res.s2 : s;
    cudaError_t e = cudaStreamWaitEvent(sc, ev_prep, 0);
    if (e == cudaSuccess && wait_x) e = cudaStreamWaitEvent(sc, ev_x, 0);
    if (e != cudaSuccess) return cuda_fail(e, "gnn_run_host event");
    const float *X = (const float *)(w + l.X[k]);
    float *O = (float *)(w + l.O[k]), *out = (float *)(w + l.out[k]);
    float *Oh = O_host ? O_host[k] : nullptr, *Eh = out_host ? out_host[k] : nullptr;
    const int64_t eb = c0 * C, ee = c1 * C < nnz ? c1 * C : nnz;  // its nonzeros
    if (Oh) {
      if (gnn_status_t st = launch_spmm(plan, &gd, X, K, O, K, sc, GNN_F32, GNN_AGG_SUM, 0,
                                        "gnn_run_host spmm", whole ? -1 : c0, c1))
        return st;
      // rows final once chunks [0, c1) are done: up to the last chunk's last row, minus
      // that row if it continues into the next chunk (which also zeroes the empty rows
      // before its first row).  The copy-out stream waits for every unit of a width in
      // piece order, so the earlier pieces (on the other stream) are done too.
      int64_t done = M;  // (local rows: global row id - row_base)
      if (ee < nnz) {
        const int32_t rl = gh->row_ind[ee - 1];
        done = (gh->row_ind[ee] == rl ? rl : (int64_t)rl + 1) - r0;
      }
      e = cudaEventRecord(ev_o, sc);
      if (e == cudaSuccess) e = cudaStreamWaitEvent(res.sout, ev_o, 0);
      if (e == cudaSuccess && done > rows_done[k])
        e = cudaMemcpyAsync(Oh + rows_done[k] * K, O + rows_done[k] * K,
                            4 * (size_t)(done - rows_done[k]) * K, cudaMemcpyDeviceToHost,
                            res.sout);
      if (e != cudaSuccess) return cuda_fail(e, "gnn_run_host O download");
      if (done > rows_done[k]) rows_done[k] = done;
    }
    if (Eh && ee > eb) {
      // A1 = the shard's own rows of X (destination rows), A2T = all of X
      if (gnn_status_t st = launch_sddmm(plan, &gd, X + r0 * K, K, X, K, out, sc, GNN_F32,
                                         "gnn_run_host sddmm", whole ? -1 : c0, c1))
        return st;
      e = cudaEventRecord(ev_e, sc);
      if (e == cudaSuccess) e = cudaStreamWaitEvent(res.sout, ev_e, 0);
      if (e == cudaSuccess)
        e = cudaMemcpyAsync(Eh + eb, out + eb, 4 * (size_t)(ee - eb), cudaMemcpyDeviceToHost,
                            res.sout);
      if (e != cudaSuccess) return cuda_fail(e, "gnn_run_host S_O download");
    }
    return GNN_OK;
  };
  // X_k (width k, all N rows) uploads on the copy-in stream; width k then catches up on
  // the pieces that landed before it
  auto upload_x = [&](int k, int pieces_in) -> gnn_status_t {
    if (N > 0) {
      cudaError_t e = cudaMemcpyAsync(w + l.X[k], X_host[k], 4 * (size_t)N * Ks[k],
                                      cudaMemcpyHostToDevice, res.sin);
      if (e == cudaSuccess) e = cudaEventRecord(ev_x, res.sin);
      if (e != cudaSuccess) return cuda_fail(e, "gnn_run_host X upload");
    }
    for (int q = 0; q < pieces_in; ++q)
      if (gnn_status_t st = compute(k, q, N > 0, ev_x)) return st;
    return GNN_OK;
  };
  // Copy-in schedule.  Every width downloads the same S_O volume (4 B per nonzero) but
  // costs 4*N*K bytes of X to start, and the downloads are the longer PCIe direction: so
  // the narrow widths' X go first, one per piece (X_(0), piece 0, X_(1), piece 1, ...),
  // keeping the copy-out stream fed from the first piece on, and the widest width's X goes
  // half-way (before piece P/2), where its catch-up over every landed piece fills the
  // copy-out queue while the rest of the graph streams in (profiles/r01_v24_e2e_schedule.txt,
  // r01_v27_e2e_wide_x_at.txt: before piece 14 of 28 measured best, 24 / 18 / 10 within
  // 0.5-1.2 ms of it).  Pieces:
  // RowInd (+ the next piece's first entry, which the plan kernel's tail flag reads),
  // ColInd, Value.
  int xpos[kMaxK];
  {
    int order[kMaxK];
    for (int k = 0; k < nk; ++k) order[k] = k;
    for (int i = 1; i < nk; ++i)  // stable insertion sort by K
      for (int j = i; j > 0 && Ks[order[j]] < Ks[order[j - 1]]; --j) {
        const int t = order[j];
        order[j] = order[j - 1];
        order[j - 1] = t;
      }
    for (int j = 0; j < nk; ++j) xpos[order[j]] = j;
    if (nk >= 2) {
      int late = P / 2;
      if (const char *e = getenv("GNN_HOST_WIDE_X_AT")) late = atoi(e);  // tuning knob
      if (late > nk - 1) xpos[order[nk - 1]] = late < P ? late : P;
    }
  }
  gnn_status_t st = GNN_OK;
  int64_t b = 0;
  for (int p = 0; p < P && st == GNN_OK; ++p) {
    for (int k = 0; k < nk && st == GNN_OK; ++k)
      if (xpos[k] == p) st = upload_x(k, p);
    if (st != GNN_OK) break;
    const int64_t en = p + 1 == P ? nnz : nnz * (p + 1) / P;  // this piece: nonzeros [b, en)
    if (up && en > b) {
      const int64_t er = en < nnz ? en + 1 : nnz;
      if (gh->row_ptr) {
        // CSR upload: the offsets of the rows this piece spans (a few bytes) instead of its
        // RowInd (4 B per nonzero), decoded on the copy-in stream
        const int64_t ra = gh->row_ind[b] - r0, rb = gh->row_ind[er - 1] - r0;
        e = cudaMemcpyAsync(w + l.row_ptr + 4 * ra, gh->row_ptr + ra, 4 * (rb - ra + 2),
                            cudaMemcpyHostToDevice, res.sin);
        if (e == cudaSuccess) {
          int64_t blocks = ((rb - ra + 1) * 32 + 255) / 256;
          if (blocks > 4096) blocks = 4096;
          csr_range_to_coo_kernel<<<(unsigned)blocks, 256, 0, res.sin>>>(
              (const int32_t *)(w + l.row_ptr) + ra, rb - ra + 1, ra, gh->row_ptr[0], b, er, r0,
              (int32_t *)(w + l.row_ind));
          e = cudaGetLastError();
        }
      } else {
        e = cudaMemcpyAsync(w + l.row_ind + 4 * b, gh->row_ind + b, 4 * (er - b),
                            cudaMemcpyHostToDevice, res.sin);
      }
      if (e == cudaSuccess)
        e = cudaMemcpyAsync(w + l.col_ind + 4 * b, gh->col_ind + b, 4 * (en - b),
                            cudaMemcpyHostToDevice, res.sin);
      if (e == cudaSuccess && gh->val)
        e = cudaMemcpyAsync(w + l.val + 4 * b, gh->val + b, 4 * (en - b),
                            cudaMemcpyHostToDevice, res.sin);
      if (e != cudaSuccess) { st = cuda_fail(e, "gnn_run_host piece upload"); break; }
    }
    // plan + pre-zero of this piece's chunks on the prep stream, in piece order: a row
    // split across pieces is zeroed (by the chunk it starts in) before any later piece
    // adds into it, and a chunk's plan entry exists before the next chunk reads it
    trace.mark(p, 0, res.sin);
    if ((e = cudaEventRecord(ev_in, res.sin)) == cudaSuccess)
      e = cudaStreamWaitEvent(res.sp, ev_in, 0);
    if (e != cudaSuccess) { st = cuda_fail(e, "gnn_run_host event"); break; }
    for (int k = 0; k < nk && st == GNN_OK; ++k) {
      const Plan *plan = reinterpret_cast<const Plan *>(plans.p[k]);
      st = launch_plan_range(plan, res.sp, cb[k][p], cb[k][p + 1]);
      if (st == GNN_OK && O_host && O_host[k] && !whole)
        st = launch_spmm_prezero(plan, &gd, (float *)(w + l.O[k]), Ks[k], res.sp, cb[k][p],
                                 cb[k][p + 1]);
    }
    if (st != GNN_OK) break;
    trace.mark(p, 1, res.sp);
    if ((e = cudaEventRecord(ev_prep, res.sp)) != cudaSuccess) {
      st = cuda_fail(e, "gnn_run_host event");
      break;
    }
    // every width whose X has landed (X_k precedes piece xpos[k] on the copy-in stream)
    for (int k = 0; k < nk && st == GNN_OK; ++k)
      if (xpos[k] <= p) st = compute(k, p, false, ev_x);
    trace.mark(p, 2, (units & 1) ? s : res.s2);
    trace.mark(p, 3, res.sout);
    b = en;
  }
  for (int k = 0; k < nk && st == GNN_OK; ++k)  // fewer pieces than widths
    if (xpos[k] >= P) st = upload_x(k, P);
  trace.xdone(res.sin);
  // the caller's stream covers every copy and kernel of this call (the copy-out stream
  // waited for every piece; s2, the prep and the copy-in stream are joined explicitly)
  cudaError_t e2 = cudaEventRecord(ev_done, res.sout);
  if (e2 == cudaSuccess) e2 = cudaStreamWaitEvent(s, ev_done, 0);
  if (e2 == cudaSuccess) e2 = cudaEventRecord(ev_done, res.s2);
  if (e2 == cudaSuccess) e2 = cudaStreamWaitEvent(s, ev_done, 0);
  if (e2 == cudaSuccess) e2 = cudaEventRecord(ev_done, res.sp);
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

// ----------------------------------------------------------------------------------
// One message-passing step on device-resident data in ONE call (BJ configs[2]: a new
// sampled subgraph every step, re-planned every step): host DTP, then SpMM and SDDMM with
// the per-chunk boundary table recomputed inside the kernels (no plan kernel).  The SDDMM
// runs on a per-thread, per-device side stream forked from `stream` and joined back
// before return, so the two kernels overlap on graphs that fill only a few waves; the
// SpMM overlaps its pre-zero through a programmatic dependent launch.  No allocation, no
// host sync.
namespace gnn {
namespace {
struct SideStream {
  int device = -1;
  cudaStream_t s = nullptr;
  cudaEvent_t fork = nullptr, join = nullptr;
};
thread_local SideStream tl_side[8];
gnn_status_t side_stream(SideStream **out) {
  int dev = 0;
  cudaError_t e = cudaGetDevice(&dev);
  if (e != cudaSuccess) return cuda_fail(e, "gnn_plan_spmm_sddmm device");
  SideStream &t = tl_side[dev & 7];
  if (t.device != dev) {
    if (t.s) {  // another device used this slot: rebuild
      cudaStreamDestroy(t.s);
      cudaEventDestroy(t.fork);
      cudaEventDestroy(t.join);
      t.s = nullptr;
    }
    e = cudaStreamCreateWithFlags(&t.s, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&t.fork, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&t.join, cudaEventDisableTiming);
    if (e != cudaSuccess) return cuda_fail(e, "gnn_plan_spmm_sddmm side stream");
    t.device = dev;
  }
  *out = &t;
  return GNN_OK;
}
}  // namespace
}  // namespace gnn

extern "C" {

GNN_API gnn_status_t gnn_plan_spmm_sddmm(const gnn_graph_t *g, int32_t K,
                                         const gnn_plan_opts_t *opts, const float *X,
                                         int64_t ldx, float *O, int64_t ldo, float *out,
                                         void *workspace, size_t ws_bytes,
                                         gnn_stream_t stream) {
  if (!g || (!O && !out))
    return fail(GNN_ERR_INVALID_ARG, "gnn_plan_spmm_sddmm: NULL graph / no output");
  if (opts && opts->feature_dtype != GNN_F32)
    return fail(GNN_ERR_UNSUPPORTED, "gnn_plan_spmm_sddmm: fp32 features only");
  // Host DTP only: no plan kernel.  The kernels derive each chunk's boundary rows and flags
  // from row_ind themselves (the plan kernel's arithmetic), so the SDDMM -- which
  // never needs them -- starts at once on the side stream, and the SpMM is launched as a
  // programmatic dependent of the split-row pre-zero.  Deterministic plans keep the plan
  // kernel (their fix-up pass reads the arrays).
  // GNN_STEP_PLAN_KERNEL=1 restores the plan-kernel path (A/B measurements)
  const char *pk = getenv("GNN_STEP_PLAN_KERNEL");
  const bool det = (opts && opts->deterministic) || (pk && pk[0] == '1');
  gnn_plan_t plan = nullptr;
  if (gnn_status_t st = plan_create(g, K, opts, workspace, ws_bytes, stream, &plan, det))
    return st;
  struct Guard {
    gnn_plan_t p;
    ~Guard() { gnn_plan_destroy(p); }
  } guard{plan};
  Plan *p = reinterpret_cast<Plan *>(plan);
  p->inline_plan = !det;
  cudaStream_t s = (cudaStream_t)stream;
  // both outputs: one fused launch where the shape has an instance and K <= 32 (measured on
  // 20 C3 subgraphs: K=32 0.0402 -> 0.0367 ms, but K=64 0.0489 -> 0.0523 and K=128 0.0684
  // -> 0.0738: the fused kernel runs the SpMM half at SDDMM's 128-register budget;
  // profiles/r02_s9_c3_fused_ab.txt).  GNN_STEP_FUSED=0 / 1: never / whenever possible.
  const char *fz = getenv("GNN_STEP_FUSED");
  const bool fuse = fz ? fz[0] == '1' : K <= 32;
  if (O && out && !det && fuse) {
    const gnn_status_t st = launch_step_fused(p, g, X, ldx, O, ldo, out, stream);
    if (st != GNN_ERR_UNSUPPORTED) return st;
  }
  SideStream *side = nullptr;
  const bool fork = O && out && g->nnz > 0;
  if (fork) {
    if (gnn_status_t st = side_stream(&side)) return st;
    cudaError_t e = cudaEventRecord(side->fork, s);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(side->s, side->fork, 0);
    if (e != cudaSuccess) return cuda_fail(e, "gnn_plan_spmm_sddmm fork");
  }
  gnn_status_t st = GNN_OK;
  // (the launch order and a low-priority side stream were measured to make no difference,
  // profiles/r02_s9_c3_fused_ab.txt)
  if (out)  // A1 = the graph's own rows of X (row_base), A2T = all of X
    st = launch_sddmm(p, g, X ? X + g->row_base * ldx : nullptr, ldx, X, ldx, out,
                      fork ? side->s : s, GNN_F32, "gnn_plan_spmm_sddmm sddmm", -1, 0);
  if (st == GNN_OK && O)
    st = launch_spmm(p, g, X, ldx, O, ldo, s, GNN_F32, GNN_AGG_SUM, 0,
                     "gnn_plan_spmm_sddmm spmm", -1, 0);
  if (fork) {  // join even after an error, so `stream` covers everything enqueued
    cudaError_t e = cudaEventRecord(side->join, side->s);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(s, side->join, 0);
    if (e != cudaSuccess && st == GNN_OK) st = cuda_fail(e, "gnn_plan_spmm_sddmm join");
  }
  return st;
}

}  // extern "C"
