// spmm_kernel.cuh -- the hybrid-parallel SpMM kernel template (see spmm.cu for the
// design notes) and its dispatch table; instantiated per feature type in
// spmm_f32.cu / spmm_bf16.cu so the two halves compile in parallel.
#pragma once
#include <math.h>

#include <type_traits>
#include "device.cuh"
#include "internal.cuh"

namespace gnn {

// Register budget and feature vectors in flight per lane (U * R), per instantiation --
// the occupancy lever of PAPER.md P:392 ("register pressure" at large K).  Measured on
// the GCR-reordered C4 and C5 (profiles/r02_s1_sweep_*.txt, 4-warp blocks):
//   fp32 rows of one 256-bit vector per lane (every K once rows of two vectors run on
//   twice the lanes, below): 80 registers (3 resident 8-warp blocks / 6 of 4 warps per SM
//   instead of 2 / 4) with 4 vectors in flight instead of 8: C4 K=32 0.890 -> 0.849 ms,
//   K=64 1.594 -> 1.510, K=128 2.974 -> 2.942, K=256 5.942 -> 5.871, C5 K=256 8.74 -> 8.61;
//   bf16 rows of >= 8 lanes: 96 registers, 4 in flight (5 resident 4-warp blocks): C4
//   K=256 3.91 -> 3.75 ms; everything else (narrow bf16 rows, max / min, two-vector rows
//   that stay so) keeps 128 registers and the round-1 depths (r01_sweep4 / 12 / 19).
// GNN_SPMM_REGS / GNN_SPMM_DEPTH8 / GNN_SPMM_DEPTH_R2 override the table (build sweeps).
#ifndef GNN_SPMM_REGS_F32
#define GNN_SPMM_REGS_F32 80  // lean fp32 rows (one 256-bit vector per lane), L <= 8 lanes
#endif
// ... rows of >= 16 lanes (K >= 128): 72 registers (14 resident 2-warp blocks instead of 12,
// 8 B of spill in a cold path): C4 K=128 2.820 -> 2.745 ms, K=256 5.62-5.69 -> 5.54-5.55,
// C5 K=256 -1%; at L <= 8 it measured 0.1-0.5% slower and 64 registers lose 4-11%
// everywhere (profiles/r02_s49_sweep_spmm_regs.txt)
#ifndef GNN_SPMM_REGS_F32_WIDE
#define GNN_SPMM_REGS_F32_WIDE 72
#endif
#ifndef GNN_SPMM_REGS_BF16
#define GNN_SPMM_REGS_BF16 96  // lean bf16 rows of >= 8 lanes (88: 84 used, no spill, but
                               // K=256 2% slower, r02_s51)
#endif
#ifndef GNN_SPMM_DEPTH_R2
#define GNN_SPMM_DEPTH_R2 4
#endif
template <typename TF, int VW, int L, int R, int AGG>
struct SpmmTune {
  static constexpr bool wide = VW * TF::bytes == 32;  // 256-bit vectors
  static constexpr bool f32 = TF::bytes == 4;
  static constexpr bool lean = AGG == 0 && R == 1 && wide && (f32 || L >= 8);
#if defined(GNN_SPMM_REGS)
  static constexpr int regs = GNN_SPMM_REGS;
#else
  static constexpr int regs =
      lean ? (f32 ? (L >= 16 ? GNN_SPMM_REGS_F32_WIDE : GNN_SPMM_REGS_F32) : GNN_SPMM_REGS_BF16)
           : 128;
#endif
#if defined(GNN_SPMM_DEPTH8)
  static constexpr int depth = wide ? GNN_SPMM_DEPTH8 : 8;
#else
  static constexpr int depth = R == 2 ? GNN_SPMM_DEPTH_R2 : ((lean || (wide && L <= 2)) ? 4 : 8);
#endif
};

// Aggregators of the node-wise MPP op (Eq. 1): ⊕ = sum (SpMM proper; mean is
// sum followed by a row scale), max or min of the terms v_i * A[col_i].
enum : int { kAggSum = 0, kAggMax = 1, kAggMin = 2 };

template <int AGG>
__device__ __forceinline__ float agg_init() {
  if constexpr (AGG == kAggSum) return 0.f;
  else if constexpr (AGG == kAggMax) return -INFINITY;
  else return INFINITY;
}

// float atomic max / min through the ordered-integer trick (there is no red.max.f32):
// floats with the sign bit clear order like signed ints, those with it set (negatives and
// -0.0) reversed like unsigned.  The branch tests the sign BIT, not v >= 0: -0.0 >= 0 is
// true, but as a signed int -0.0 is INT_MIN and would beat every negative value in a
// signed atomicMin (and lose to them in atomicMax).
__device__ __forceinline__ void atomic_max_f32(float *p, float v) {
  if (!(__float_as_uint(v) >> 31)) atomicMax(reinterpret_cast<int *>(p), __float_as_int(v));
  else atomicMin(reinterpret_cast<unsigned *>(p), __float_as_uint(v));
}
__device__ __forceinline__ void atomic_min_f32(float *p, float v) {
  if (!(__float_as_uint(v) >> 31)) atomicMin(reinterpret_cast<int *>(p), __float_as_int(v));
  else atomicMax(reinterpret_cast<unsigned *>(p), __float_as_uint(v));
}

// Flush the accumulator of row `cur` (Algo 3 line 15, "AtomicStore"): rows shared
// with a neighbouring chunk are combined atomically (vector add, or float max/min), rows
// owned by this chunk get a plain vector store (or O += acc when accumulating, beta = 1).
template <int VW, int AGG>
__device__ __forceinline__ void flush_row(float *Ok, int64_t ldo, int64_t row_base, int32_t cur,
                                          int32_t rf, int32_t rl, uint32_t fl, bool accum,
                                          const float (&acc)[VW]) {
  float *o = Ok + ((int64_t)cur - row_base) * ldo;
  const bool shared = (cur == rf && (fl & 1u)) || (cur == rl && (fl & 2u));
  if constexpr (AGG == kAggSum) {
    if (shared || accum) red_add<VW>(o, acc);
    else st_vec<VW>(o, acc);
  } else {
    if (shared) {
#pragma unroll
      for (int v = 0; v < VW; ++v) {
        if constexpr (AGG == kAggMax) atomic_max_f32(o + v, acc[v]);
        else atomic_min_f32(o + v, acc[v]);
      }
    } else {
      st_vec<VW>(o, acc);
    }
  }
}

template <int AGG, typename TF, int VW>
__device__ __forceinline__ void accumulate(float (&acc)[VW], float s, const FeatVec<TF, VW> &x) {
  if constexpr (AGG == kAggSum) {
    axpy_f<TF, VW>(acc, s, x);
  } else {
#pragma unroll
    for (int v = 0; v < VW; ++v) {
      const float t = s * x.get(v);
      acc[v] = AGG == kAggMax ? fmaxf(acc[v], t) : fminf(acc[v], t);
    }
  }
}

// L lanes per (chunk, K-slice) work item, R VW-wide vectors per lane (plan rule step 2).
// TF: feature element type (F32 or BF16); accumulation and O are fp32.
// The kernel body with the block index as a parameter (bid), so a fused launch can run it
// on a sub-range of its blocks (step_fused.cu).
template <typename TF, int VW, int L, int R, int VWS, int AGG>
__device__ __forceinline__ void spmm_body(const SparseArgs &a, const void *__restrict__ A,
                                          const int64_t lda, float *__restrict__ O,
                                          const int64_t ldo, const int64_t bid) {
  constexpr int ES = TF::bytes;
  constexpr int Lg = L;
  constexpr int G = 32 / Lg;
  using Tiles = TilesFor<L, VWS>;
  constexpr int T = Tiles::T;  // nonzeros per tile per group
  // U nonzeros per batch: FeatDepth vectors in flight per lane, whole sparse vectors
  constexpr int D = SpmmTune<TF, VW, L, R, AGG>::depth / R;
  constexpr int U = D > T ? T : (D < VWS ? VWS : D);
  static_assert(T % U == 0 && U % VWS == 0, "tile / prefetch shape");
  const int lane = threadIdx.x & 31;
  const int g = lane / Lg;
  const int l = lane & (Lg - 1);
  const int64_t item =
      a.c_begin * a.slices + (bid * (blockDim.x >> 5) + (threadIdx.x >> 5)) * G + g;
  const bool item_ok = item < a.c_end * a.slices;
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
  // sparse tiles: per-warp double-buffered shared-memory ring (TMA bulk copies, or
  // cp.async for narrow sparse vectors), one tile ahead of use -- the first tile is
  // requested before the chunk's boundary rows are read, so the two latencies overlap
  extern __shared__ int32_t gnn_smem[];
  Tiles tiles;
  {
    const int64_t item0 =
        a.c_begin * a.slices + (bid * (blockDim.x >> 5) + (threadIdx.x >> 5)) * G;
    tiles.init(gnn_smem + (threadIdx.x >> 5) * Tiles::WARP_WORDS, lane, a.row_ind, a.col_ind,
               a.val, [&](int gg, int64_t &cs_, int &n_) {
                 const int64_t it = item0 + gg;
                 cs_ = 0;
                 n_ = 0;
                 if (it < a.c_end * a.slices) {
                   cs_ = (it / a.slices) * a.chunk;
                   n_ = (int)(min(cs_ + (int64_t)a.chunk, a.nnz) - cs_);
                 }
               },
               cs, n);
  }
  tiles.issue(0, 0, lane);
  int32_t rf = 0, rl = 0;
  uint32_t fl = 0;
  if (item_ok) chunk_rows(a, c, rf, rl, fl);
  // feature row c of A starts at Ab + c * ldaB (one IMAD.WIDE.U32 per gather, row_addr)
  const char *__restrict__ Ab = reinterpret_cast<const char *>(A) + (int64_t)k0 * ES;
  const uint32_t ldaB = (uint32_t)lda * (uint32_t)ES;
  float *__restrict__ Ok = O + k0;  // row r at Ok + (r - row_base) * ldo
  const bool full = a.K == a.slices * L * R * VW;  // (warp-uniform) no absent columns

  auto zero_row = [&](int64_t row) {  // rows without nonzeros: 0 (untouched if beta = 1)
    if (a.accum) return;
#pragma unroll
    for (int r = 0; r < R; ++r)
      if (col_ok[r]) st_zero<VW>(Ok + (row - a.row_base) * ldo + r * Lg * VW);
  };
  float acc[R][VW];
  // Launched as a programmatic dependent of the pre-zero kernel (gnn_plan_spmm_sddmm):
  // everything up to the first flush of a row shared with another chunk overlaps the
  // pre-zero; that flush waits for it (griddepcontrol.wait is a no-op otherwise).
  bool pdl_waited = false;
  auto flush = [&](int32_t row) {
    if (!pdl_waited && ((row == rf && (fl & 1u)) || (row == rl && (fl & 2u)))) {
      asm volatile("griddepcontrol.wait;" ::: "memory");
      pdl_waited = true;
    }
    if (a.carry) {  // deterministic plan: split rows go to this chunk's partial slots
      const bool shared = (row == rf && (fl & 1u)) || (row == rl && (fl & 2u));
      if (shared) {
        float *cp = a.carry + (c * 2 + (row == rf ? 0 : 1)) * (int64_t)a.K + k0;
#pragma unroll
        for (int r = 0; r < R; ++r)
          if (col_ok[r]) st_vec<VW>(cp + r * Lg * VW, acc[r]);
        return;
      }
    }
#pragma unroll
    for (int r = 0; r < R; ++r)
      if (col_ok[r])
        flush_row<VW, AGG>(Ok + r * Lg * VW, ldo, a.row_base, row, rf, rl, fl, a.accum != 0,
                           acc[r]);
  };

  // empty rows between the previous chunk's last row and ours are ours to zero
  if (item_ok) {
    const int64_t prev = (c == 0) ? a.row_base - 1 : (int64_t)prev_chunk_last_row(a, c);
    for (int64_t r = prev + 1; r < rf; ++r) zero_row(r);
  }

#pragma unroll
  for (int r = 0; r < R; ++r)
#pragma unroll
    for (int v = 0; v < VW; ++v) acc[r][v] = agg_init<AGG>();
  int32_t cur = -1;


  const int ntiles = (a.chunk + T - 1) / T;  // warp-uniform trip count
  for (int t = 0; t < ntiles; ++t) {
    const int tb = t * T;
    const int st = t & 1;
    __syncwarp();  // every lane is done with the stage the next copy overwrites
    if (t + 1 < ntiles) tiles.issue(st ^ 1, tb + T, lane);
    else tiles.skip();
    tiles.wait(st, t);  // tile t has landed
    __syncwarp();       // (and the plain-load tails written by other lanes are visible)
    const int32_t *s_row = tiles.rows(st, g);
    const int32_t *s_col = tiles.cols(st, g);
    const float *s_val = tiles.vals(st, g);
    const int32_t r_first = s_row[0];
    const bool fast_g = (tb + T <= n) && r_first == s_row[T - 1];
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
          for (int v = 0; v < VW; ++v) acc[r][v] = agg_init<AGG>();
      }
      // FULL: every lane's columns exist (K is a whole number of slices): the loads need no
      // predicate and no zero-fill (a group past the last chunk reads the zero-filled tile,
      // i.e. row 0, and never flushes) -- one register-zeroing instruction less per pair of
      // loaded values
      auto fast_tile = [&](auto full_tag) {
        constexpr bool FULL = decltype(full_tag)::value;
#pragma unroll 1
        for (int jj = 0; jj < T; jj += U) {
          uint32_t cj[U];
          float vj[U];
#pragma unroll
          for (int u = 0; u < U; ++u) {
            cj[u] = (uint32_t)s_col[jj + u];
            vj[u] = s_val[jj + u];  // (1.0 when val == NULL: tiles.init)
          }
          FeatVec<TF, VW> x[U][R];
#pragma unroll
          for (int u = 0; u < U; ++u) {
            const char *rowp = row_addr(Ab, cj[u], ldaB);
#pragma unroll
            for (int r = 0; r < R; ++r) {
              if (FULL || col_ok[r]) x[u][r].load(rowp + r * Lg * VW * ES);
              else x[u][r].zero();
            }
          }
#pragma unroll
          for (int u = 0; u < U; ++u)
#pragma unroll
            for (int r = 0; r < R; ++r) accumulate<AGG, TF, VW>(acc[r], vj[u], x[u][r]);
        }
      };
      if (full) fast_tile(std::true_type{});
      else fast_tile(std::false_type{});
    } else {
      // ---- general path: per-nonzero row-switch procedure
      // WHOLE (warp-uniform): every group's tile lies inside its chunk, so no per-nonzero
      // validity test (a group past the last chunk reads the zero-filled tile -- row 0 --
      // and never flushes: its first row switch starts from cur = -1 and the final flush
      // below is guarded by item_ok)
      auto general_tile = [&](auto full_tag, auto whole_tag) {
        constexpr bool FULL = decltype(full_tag)::value;
        constexpr bool WHOLE = decltype(whole_tag)::value;
#pragma unroll 1
        for (int jj = 0; jj < T; jj += U) {
          int32_t rj[U];
          uint32_t cj[U];
          float vj[U];
#pragma unroll
          for (int u = 0; u < U; ++u) {
            rj[u] = s_row[jj + u];
            cj[u] = (uint32_t)s_col[jj + u];
            vj[u] = s_val[jj + u];  // (1.0 when val == NULL: tiles.init)
          }
          FeatVec<TF, VW> x[U][R];
#pragma unroll
          for (int u = 0; u < U; ++u) {
            const char *rowp = row_addr(Ab, cj[u], ldaB);
#pragma unroll
            for (int r = 0; r < R; ++r) {
              // (FULL: entries past the chunk end read row 0 of the zero-filled tile and are
              // not accumulated)
              if (FULL || (col_ok[r] && (WHOLE || tb + jj + u < n)))
                x[u][r].load(rowp + r * Lg * VW * ES);
              else
                x[u][r].zero();
            }
          }
          // (warp-uniform) no group switches rows within this batch (rows are sorted, so
          // the batch's last row decides): plain accumulation, no per-nonzero tests
          if (WHOLE && __all_sync(kFull, rj[U - 1] == cur || !item_ok)) {
#pragma unroll
            for (int u = 0; u < U; ++u)
#pragma unroll
              for (int r = 0; r < R; ++r) accumulate<AGG, TF, VW>(acc[r], vj[u], x[u][r]);
            continue;
          }
#pragma unroll
          for (int u = 0; u < U; ++u) {
            if (WHOLE || tb + jj + u < n) {
              if (rj[u] != cur) {  // row-switch procedure
                if (cur >= 0) {
                  flush(cur);
                  for (int64_t r = (int64_t)cur + 1; r < rj[u]; ++r) zero_row(r);
                }
                cur = rj[u];
                if constexpr (AGG == kAggSum) {
                  // the new row starts at its first term (v*x, = 0 + v*x): both branches
                  // write the accumulator in place, no merge copies per nonzero
#pragma unroll
                  for (int r = 0; r < R; ++r)
#pragma unroll
                    for (int v = 0; v < VW; ++v) acc[r][v] = vj[u] * x[u][r].get(v);
                } else {
#pragma unroll
                  for (int r = 0; r < R; ++r) {
#pragma unroll
                    for (int v = 0; v < VW; ++v) acc[r][v] = agg_init<AGG>();
                    accumulate<AGG, TF, VW>(acc[r], vj[u], x[u][r]);
                  }
                }
              } else {
#pragma unroll
                for (int r = 0; r < R; ++r) accumulate<AGG, TF, VW>(acc[r], vj[u], x[u][r]);
              }
            }
          }
        }
      };
      if (__all_sync(kFull, tb + T <= n || !item_ok)) {
        if (full) general_tile(std::true_type{}, std::true_type{});
        else general_tile(std::false_type{}, std::true_type{});
      } else {
        if (full) general_tile(std::true_type{}, std::false_type{});
        else general_tile(std::false_type{}, std::false_type{});
      }
    }
  }
  if (cur >= 0 && item_ok) flush(cur);
  // trailing empty rows after the last chunk
  if (item_ok && c == a.num_chunks - 1) {
    for (int64_t r = (int64_t)rl + 1; r < a.row_base + a.M; ++r) zero_row(r);
  }
}

template <typename TF, int VW, int L, int R, int VWS, int AGG>
__global__ void __maxnreg__((SpmmTune<TF, VW, L, R, AGG>::regs))
    spmm_kernel(const SparseArgs a, const void *__restrict__ A, const int64_t lda,
                float *__restrict__ O, const int64_t ldo) {
  spmm_body<TF, VW, L, R, VWS, AGG>(a, A, lda, O, ldo, blockIdx.x);
}

using SpmmFn = void (*)(const SparseArgs, const void *__restrict__, const int64_t,
                        float *__restrict__, const int64_t);

template <typename TF, int VW, int L, int R, int AGG>
SpmmFn spmm_pick_vws(int vws) {
  switch (vws) {
    case 1: return spmm_kernel<TF, VW, L, R, 1, AGG>;
    case 2: return spmm_kernel<TF, VW, L, R, 2, AGG>;
    case 4: return spmm_kernel<TF, VW, L, R, 4, AGG>;
  }
  return nullptr;
}
template <typename TF, int VW, int AGG>
SpmmFn spmm_pick_l(int L, int R, int vws) {
  if (R == 2) {  // the plan uses R = 2 only for rows of >= 16 vectors, i.e. L >= 8
    switch (L) {
      case 8: return spmm_pick_vws<TF, VW, 8, 2, AGG>(vws);
      case 16: return spmm_pick_vws<TF, VW, 16, 2, AGG>(vws);
      case 32: return spmm_pick_vws<TF, VW, 32, 2, AGG>(vws);
    }
    return nullptr;
  }
  switch (L) {
    case 1: return spmm_pick_vws<TF, VW, 1, 1, AGG>(vws);
    case 2: return spmm_pick_vws<TF, VW, 2, 1, AGG>(vws);
    case 4: return spmm_pick_vws<TF, VW, 4, 1, AGG>(vws);
    case 8: return spmm_pick_vws<TF, VW, 8, 1, AGG>(vws);
    case 16: return spmm_pick_vws<TF, VW, 16, 1, AGG>(vws);
    case 32: return spmm_pick_vws<TF, VW, 32, 1, AGG>(vws);
  }
  return nullptr;
}

// dynamic shared memory of spmm_kernel<.., L, .., VWS> per warp
inline int spmm_tile_bytes_per_warp(int L, int vws) { return tile_bytes_per_warp(L, vws); }

template <typename TF, int AGG>
SpmmFn spmm_pick_vw(int vw, int L, int R, int vws);

// defined in spmm_f32*.cu / spmm_bf16.cu (one translation unit per aggregator)
SpmmFn pick_spmm_f32(int vw, int L, int R, int vws);
SpmmFn pick_spmm_f32_max(int vw, int L, int R, int vws);
SpmmFn pick_spmm_f32_min(int vw, int L, int R, int vws);
SpmmFn pick_spmm_bf16(int vw, int L, int R, int vws);

}  // namespace gnn
