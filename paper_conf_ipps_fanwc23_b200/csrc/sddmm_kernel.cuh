// sddmm_kernel.cuh -- the hybrid-parallel SDDMM kernel template (design notes in
// sddmm.cu) and its dispatch table; instantiated per feature type in sddmm_f32.cu /
// sddmm_bf16.cu.
#pragma once
#include <type_traits>

#include "device.cuh"
#include "internal.cuh"

namespace gnn {

// Lane mapping of SDDMM.  A K-slice holds V = L * R VW-wide vectors (plan rule step 2);
// SDDMM spreads them over Lg = V / Rsd lanes with Rsd vectors per lane, so each dot
// product is reduced over Lg lanes and 32 / Lg nonzeros are in flight per warp step;
// U = nonzeros per batch per group, U * Rsd = 8 feature vectors in flight per lane.
// Measured on the GCR-reordered C4.  Round 1 (r01_sweep8) preferred Rsd = 2 from V = 8
// (K=64 2.07 -> 1.94 ms, K=128 4.82 -> 3.61, K=256 8.85 -> 7.05); with the round-2 launch
// shape one vector per lane wins up to V = 16: fp32 K=64 1.652 -> 1.544 ms, K=128 3.039 ->
// 2.983, bf16 K=128 1.719 -> 1.662, bf16 K=256 3.211 -> 3.164; at V = 32 (fp32 K=256) the
// two are equal (profiles/r02_s13_sweep_c4_sddmm_r1_k64.txt, r02_s15_sweep_sddmm_r.txt).
#ifndef GNN_SDDMM_R2_FROM
#define GNN_SDDMM_R2_FROM 32  // smallest V that uses Rsd = 2
#endif
#ifndef GNN_SDDMM_UR
#define GNN_SDDMM_UR 8       // U * Rsd: feature vectors in flight per lane
#endif
#ifndef GNN_SDDMM_BF16_NARROW
#define GNN_SDDMM_BF16_NARROW 1  // bf16 K = 32: 4 lanes x 8 instead of 2 lanes x 16
#endif
#ifndef GNN_SDDMM_PIPE
#define GNN_SDDMM_PIPE 1     // next batch's loads issued before this batch's reduction
#endif
#ifndef GNN_SDDMM_NARROW_MIN_BYTES
#define GNN_SDDMM_NARROW_MIN_BYTES 32  // ... only vectors of at least this many bytes (16:
                                       // bf16 K=32 as 8-byte vectors, 3% slower on C4, r02_s41)
#endif
#ifndef GNN_SDDMM_NARROW_LG8
#define GNN_SDDMM_NARROW_LG8 1  // 4 x 32-byte single-slice rows run as 8 x 16-byte (sddmm.cu;
                                // C4 fp32 K=32 0.924 -> 0.891 ms, bf16 K=64 0.984 -> 0.964, r02_s38)
#endif
#ifndef GNN_SDDMM_PIPE_GENERAL
#define GNN_SDDMM_PIPE_GENERAL 1  // ... also on tiles with row switches (r01_sweep40)
#endif
template <int VW, int V, int SMAX>
struct SddmmShape {
  static constexpr int R = (V >= GNN_SDDMM_R2_FROM && V >= 2) ? 2 : 1;
  static constexpr int Lg = V / R;
  static constexpr int depth = GNN_SDDMM_UR / R > 1 ? GNN_SDDMM_UR / R : 1;
};
// Register budget per thread: 128 = 8 resident 2-warp blocks per SM, 96 = 10.  Rows of
// one vector per lane (R = 1: fp32 K <= 128, bf16 K <= 256) fit 96 without spilling and
// gain from the extra warps (fp32 C4 K=32 0.891 -> 0.859 ms, K=64 1.496 -> 1.461, K=128
// 2.860 -> 2.773, C5 K=64 2.154 -> 2.063, C3 step 0.0599 -> 0.0590; bf16 C4 K=128 1.592
// -> 1.513, K=256 3.009 -> 2.866); two-vector rows (R = 2, fp32 K = 256) lose 7-9% at 96
// and keep 128 (profiles/r02_s47_sweep_sddmm_regs.txt, r02_s48_sweep_sddmm_regs_r1.txt).
#ifndef GNN_SDDMM_REGS
#define GNN_SDDMM_REGS 128
#endif
#ifndef GNN_SDDMM_REGS_R1
#define GNN_SDDMM_REGS_R1 96
#endif
#ifndef GNN_SDDMM_REGS_BF16
#define GNN_SDDMM_REGS_BF16 GNN_SDDMM_REGS
#endif
template <typename TF, int VW, int V, int SMAX>
struct SddmmRegs {
  static constexpr int value = (SddmmShape<VW, V, SMAX>::R == 1 && SMAX == 1)
                                   ? GNN_SDDMM_REGS_R1
                                   : (TF::bytes == 2 ? GNN_SDDMM_REGS_BF16 : GNN_SDDMM_REGS);
};

// WarpReduce (Algo 4 line 12) of U partial dot products at once over the group's L
// lanes, as a transposed butterfly: each halving step exchanges half of the values
// (U/2 + U/4 + ... shuffles instead of U * log2 L).  Afterwards value u lives in lane
// l with u = l * U / L (U <= L; lanes l % (L/U) == 0 are its owners) or, for U > L, in
// slot i of lane l with u = l * (U/L) + i.  Then S_O = sum * v (Algo 2 line 6) is
// stored for the first `valid` of the U nonzeros at out[0..U).
template <int U, int L>
__device__ __forceinline__ void reduce_scale_store(float (&part)[U], const float *sval,
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
  // the owner lane of nonzero u reads its value straight from the shared-memory tile
  if constexpr (U <= L) {
    constexpr int R = L / U;
    const int u = l / R;
    if (l % R == 0 && u < valid) {
#if GNN_OUT_STREAMING
      __stcs(out + u, part[0] * (sval ? sval[u] : 1.f));
#else
      out[u] = part[0] * (sval ? sval[u] : 1.f);
#endif
    }
  } else {
    // this lane holds P consecutive results: one vector store for a full, aligned batch
    // (the scalar stores of narrow rows -- 64-byte rows: 16 groups x 4 stores per batch
    // -- were a visible share of the L1 store wavefronts)
    if constexpr (P == 2 || P == 4) {
      float *o = out + l * P;
      if (valid >= U && (reinterpret_cast<uintptr_t>(o) & (4 * P - 1)) == 0) {
        float v[P];
#pragma unroll
        for (int i = 0; i < P; ++i) v[i] = part[i] * (sval ? sval[l * P + i] : 1.f);
#if GNN_OUT_STREAMING
        if constexpr (P == 4) __stcs(reinterpret_cast<float4 *>(o), make_float4(v[0], v[1], v[2], v[3]));
        else __stcs(reinterpret_cast<float2 *>(o), make_float2(v[0], v[1]));
#else
        if constexpr (P == 4) *reinterpret_cast<float4 *>(o) = make_float4(v[0], v[1], v[2], v[3]);
        else *reinterpret_cast<float2 *>(o) = make_float2(v[0], v[1]);
#endif
        return;
      }
    }
#pragma unroll
    for (int i = 0; i < P; ++i) {
      const int u = l * P + i;
      if (u < valid) {
#if GNN_OUT_STREAMING
        __stcs(out + u, part[i] * (sval ? sval[u] : 1.f));
#else
        out[u] = part[i] * (sval ? sval[u] : 1.f);
#endif
      }
    }
  }
}

// L here is V, the number of VW-wide vectors in one K-slice (plan lanes x vecs).
// The kernel body with the block index as a parameter (see spmm_body).
template <typename TF, int VW, int L, int VWS, int SMAX>
__device__ __forceinline__ void sddmm_body(const SparseArgs &a, const void *__restrict__ A1,
                                           const int64_t lda1, const void *__restrict__ A2T,
                                           const int64_t lda2, float *__restrict__ out,
                                           const int64_t bid) {
  constexpr int ES = TF::bytes;
  using Sh = SddmmShape<VW, L, SMAX>;
  constexpr int R = Sh::R, Lg = Sh::Lg;
  constexpr int G = 32 / Lg;
  using Tiles = TilesFor<Lg, VWS>;
  constexpr int T = Tiles::T;
  constexpr int U0 = Sh::depth > VWS ? Sh::depth : VWS;
  constexpr int U = U0 < T ? U0 : T;
  static_assert(T % U == 0 && U % VWS == 0, "tile / prefetch shape");
  const int lane = threadIdx.x & 31;
  const int g = lane / Lg;
  const int l = lane & (Lg - 1);
  const int64_t c =
      a.c_begin + (bid * (blockDim.x >> 5) + (threadIdx.x >> 5)) * G + g;
  const bool item_ok = c < a.c_end;
  if (!__any_sync(kFull, item_ok)) return;
  const int64_t cs = c * a.chunk;
  const int n = item_ok ? (int)(min(cs + (int64_t)a.chunk, a.nnz) - cs) : 0;
  const int S = a.slices;  // <= SMAX (host-checked)
  const uint32_t ld2B = (uint32_t)lda2 * (uint32_t)ES;
  const char *__restrict__ A2b = reinterpret_cast<const char *>(A2T);

  // column of vector r of slice sl owned by lane l: (sl*L + r*Lg + l) * VW
  FeatVec<TF, VW> a1[SMAX][R];
  int32_t cur[SMAX];  // row whose A1 slice is cached, per slice
#pragma unroll
  for (int sl = 0; sl < SMAX; ++sl) {
    cur[sl] = -1;
#pragma unroll
    for (int r = 0; r < R; ++r) a1[sl][r].zero();
  }

  const float *__restrict__ vi = a.val ? a.val + cs : nullptr;
  float *__restrict__ oc = out + cs;
  // sparse tiles: per-warp double-buffered shared-memory ring (TMA bulk copies, or
  // cp.async for narrow sparse vectors), one tile ahead of use
  extern __shared__ int32_t gnn_smem[];
  Tiles tiles;
  {
    const int64_t c0 =
        a.c_begin + (bid * (blockDim.x >> 5) + (threadIdx.x >> 5)) * G;
    tiles.init(gnn_smem + (threadIdx.x >> 5) * Tiles::WARP_WORDS, lane, a.row_ind, a.col_ind,
               a.val, [&](int gg, int64_t &cs_, int &n_) {
                 const int64_t cc = c0 + gg;
                 cs_ = 0;
                 n_ = 0;
                 if (cc < a.c_end) {
                   cs_ = cc * a.chunk;
                   n_ = (int)(min(cs_ + (int64_t)a.chunk, a.nnz) - cs_);
                 }
               },
               cs, n);
  }
  tiles.issue(0, 0, lane);

  auto load_a1_slice = [&](int sl, int32_t row) {
    const char *base = reinterpret_cast<const char *>(A1) +
                       (((int64_t)row - a.row_base) * lda1 + (sl * L + l) * VW) * ES;
#pragma unroll
    for (int r = 0; r < R; ++r) {
      const int k0 = (sl * L + r * Lg + l) * VW;
      if (k0 < a.K) a1[sl][r].load(base + r * Lg * VW * ES);
    }
    cur[sl] = row;
  };

  // (warp-uniform) every lane's columns exist: K is a whole number of slices
  const bool full = a.K == S * L * VW;
  const int ntiles = (a.chunk + T - 1) / T;
  for (int t = 0; t < ntiles; ++t) {
    const int tb = t * T;
    const int st = t & 1;
    __syncwarp();  // every lane is done with the stage the next copy overwrites
    if (t + 1 < ntiles) tiles.issue(st ^ 1, tb + T, lane);
    else tiles.skip();
    tiles.wait(st, t);  // tile t has landed
    __syncwarp();
    const int32_t *s_row = tiles.rows(st, g);
    const int32_t *s_col = tiles.cols(st, g);
    const float *s_val = tiles.vals(st, g);
    const int32_t r_first = s_row[0];
    const bool fast =
        __all_sync(kFull, ((tb + T <= n) && r_first == s_row[T - 1]) || !item_ok);
    if (fast && item_ok && r_first != cur[0]) {  // row switch at the tile start
#pragma unroll
      for (int sl = 0; sl < SMAX; ++sl)
        if (sl < S) load_a1_slice(sl, r_first);
    }
    // The batch loop is instantiated twice: FAST (whole tile in one row, every nonzero
    // valid: no per-nonzero row or bounds logic) and general.
    auto run_tile = [&](auto fast_tag, auto full_tag) {
      constexpr bool FAST = decltype(fast_tag)::value;
      constexpr bool FULL = decltype(full_tag)::value;
#pragma unroll 1
      for (int jj = 0; jj < T; jj += U) {
        int32_t rj[U];
        uint32_t cj[U];
        float part[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          cj[u] = (uint32_t)s_col[jj + u];
          if constexpr (!FAST) rj[u] = s_row[jj + u];
          part[u] = 0.f;
        }
        const int valid = n - (tb + jj);
#pragma unroll
        for (int sl = 0; sl < SMAX; ++sl) {
          if (sl < S) {
            // this lane's first element of slice sl; vector r sits r*Lg*VW elements on
            const char *A2l = A2b + (int64_t)((sl * L + l) * VW) * ES;
            bool lane_ok[R];
#pragma unroll
            for (int r = 0; r < R; ++r) lane_ok[r] = item_ok && (sl * L + r * Lg + l) * VW < a.K;
            FeatVec<TF, VW> x[U][R];
#pragma unroll
            for (int u = 0; u < U; ++u) {
              const char *rowp = row_addr(A2l, cj[u], ld2B);
#pragma unroll
              for (int r = 0; r < R; ++r) {
                // FULL (no absent columns): no predicate, no zero-fill -- a nonzero past
                // the chunk end reads row 0 of the zero-filled tile and is not stored
                if (FULL || (lane_ok[r] && (FAST || u < valid)))
                  x[u][r].load(rowp + r * Lg * VW * ES);
                else x[u][r].zero();
              }
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
              if constexpr (!FAST) {
                if (item_ok && u < valid && rj[u] != cur[sl]) {
                  // row-switch procedure: load the new A1 row (Algo 4 lines 8-11)
                  load_a1_slice(sl, rj[u]);
                }
              }
#pragma unroll
              for (int r = 0; r < R; ++r) part[u] = dot_f<TF, VW>(part[u], a1[sl][r], x[u][r]);
            }
          }
        }
        reduce_scale_store<U, Lg>(part, vi ? s_val + jj : nullptr, l, oc + tb + jj,
                                  item_ok ? (FAST ? U : valid) : 0);
      }
    };
#if GNN_SDDMM_PIPE
    // FAST tiles of single-slice rows, software-pipelined: the next batch's feature rows
    // are requested as soon as this batch's dot products have consumed their registers,
    // BEFORE this batch's shuffle reduction and store, so the memory pipe is not idle
    // while the butterfly runs (same registers: x is dead after the dots).
    auto run_fast_pipelined = [&](auto full_tag) {
      constexpr bool FULL = decltype(full_tag)::value;
      const char *A2l = A2b + (int64_t)(l * VW) * ES;
      bool lane_ok[R];
#pragma unroll
      for (int r = 0; r < R; ++r) lane_ok[r] = item_ok && (r * Lg + l) * VW < a.K;
      FeatVec<TF, VW> x[U][R];
      auto load_batch = [&](int jj) {
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const char *rowp = row_addr(A2l, (uint32_t)s_col[jj + u], ld2B);
#pragma unroll
          for (int r = 0; r < R; ++r) {
            if (FULL || lane_ok[r]) x[u][r].load(rowp + r * Lg * VW * ES);
            else x[u][r].zero();
          }
        }
      };
      load_batch(0);
#pragma unroll 1
      for (int jj = 0; jj < T; jj += U) {
        float part[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          part[u] = 0.f;
#pragma unroll
          for (int r = 0; r < R; ++r) part[u] = dot_f<TF, VW>(part[u], a1[0][r], x[u][r]);
        }
        if (jj + U < T) load_batch(jj + U);
        reduce_scale_store<U, Lg>(part, vi ? s_val + jj : nullptr, l, oc + tb + jj,
                                  item_ok ? U : 0);
      }
    };
    // measured (profiles/r01_sweep39): a gain where the butterfly is long (Lg >= 8 lanes per
    // dot product: fp32 K=256 6.47 -> 6.16 ms, K=128 3.21 -> 3.11 ms, bf16 K=256 3.48 ->
    // 3.41 ms), a small loss at Lg = 4 (fp32 K=64 +0.7%, bf16 K=64 +2.6%)
#if GNN_SDDMM_PIPE_GENERAL
    // the same pipelining for tiles with row switches / a partial last tile: the next
    // batch's A2T rows do not depend on the row switches of this one
    auto run_general_pipelined = [&](auto full_tag, auto whole_tag) {
      constexpr bool FULL = decltype(full_tag)::value;
      constexpr bool WHOLE = decltype(whole_tag)::value;  // tile inside every chunk
      const char *A2l = A2b + (int64_t)(l * VW) * ES;
      bool lane_ok[R];
#pragma unroll
      for (int r = 0; r < R; ++r) lane_ok[r] = item_ok && (r * Lg + l) * VW < a.K;
      FeatVec<TF, VW> x[U][R];
      auto load_batch = [&](int jj) {
        const int valid = WHOLE ? U : n - (tb + jj);
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const char *rowp = row_addr(A2l, (uint32_t)s_col[jj + u], ld2B);
#pragma unroll
          for (int r = 0; r < R; ++r) {
            if (FULL || (lane_ok[r] && (WHOLE || u < valid)))
              x[u][r].load(rowp + r * Lg * VW * ES);
            else
              x[u][r].zero();
          }
        }
      };
      load_batch(0);
#pragma unroll 1
      for (int jj = 0; jj < T; jj += U) {
        const int valid = WHOLE ? U : n - (tb + jj);
        float part[U];
        if (WHOLE && __all_sync(kFull, s_row[jj + U - 1] == cur[0] || !item_ok)) {
          // no group switches rows within this batch (rows are sorted): no per-nonzero
          // row test, the cached A1 row serves all U dot products
#pragma unroll
          for (int u = 0; u < U; ++u) {
            part[u] = 0.f;
#pragma unroll
            for (int r = 0; r < R; ++r) part[u] = dot_f<TF, VW>(part[u], a1[0][r], x[u][r]);
          }
        } else {
#pragma unroll
          for (int u = 0; u < U; ++u) {
            part[u] = 0.f;
            const int32_t rj = s_row[jj + u];
            if (item_ok && (WHOLE || u < valid) && rj != cur[0])
              load_a1_slice(0, rj);  // Algo 4 l. 8-11
#pragma unroll
            for (int r = 0; r < R; ++r) part[u] = dot_f<TF, VW>(part[u], a1[0][r], x[u][r]);
          }
        }
        if (jj + U < T) load_batch(jj + U);
        reduce_scale_store<U, Lg>(part, vi ? s_val + jj : nullptr, l, oc + tb + jj,
                                  item_ok ? valid : 0);
      }
    };
#endif
    if constexpr (SMAX == 1 && Lg >= 8) {
      if (fast) {
        if (full) run_fast_pipelined(std::true_type{});
        else run_fast_pipelined(std::false_type{});
        continue;
      }
#if GNN_SDDMM_PIPE_GENERAL
      // (warp-uniform) every group's tile lies inside its chunk: no per-nonzero bounds test
      if (__all_sync(kFull, tb + T <= n || !item_ok)) {
        if (full) run_general_pipelined(std::true_type{}, std::true_type{});
        else run_general_pipelined(std::false_type{}, std::true_type{});
      } else {
        if (full) run_general_pipelined(std::true_type{}, std::false_type{});
        else run_general_pipelined(std::false_type{}, std::false_type{});
      }
      continue;
#endif
    }
#endif
    if (fast) {
      if (full) run_tile(std::true_type{}, std::true_type{});
      else run_tile(std::true_type{}, std::false_type{});
    } else {
      if (full) run_tile(std::false_type{}, std::true_type{});
      else run_tile(std::false_type{}, std::false_type{});
    }
  }
}

template <typename TF, int VW, int L, int VWS, int SMAX>
__global__ void __maxnreg__((SddmmRegs<TF, VW, L, SMAX>::value))
    sddmm_kernel(const SparseArgs a, const void *__restrict__ A1, const int64_t lda1,
                 const void *__restrict__ A2T, const int64_t lda2, float *__restrict__ out) {
  sddmm_body<TF, VW, L, VWS, SMAX>(a, A1, lda1, A2T, lda2, out, blockIdx.x);
}

using SddmmFn = void (*)(const SparseArgs, const void *__restrict__, const int64_t,
                         const void *__restrict__, const int64_t, float *__restrict__);

template <typename TF, int VW, int V, int SMAX>
SddmmFn pick_sddmm_vws(int vws) {
  // a batch must cover whole sparse vectors: narrow the sparse loads when U < vw_sparse
  constexpr int D = SddmmShape<VW, V, SMAX>::depth;
  while (vws > D) vws >>= 1;
  switch (vws) {
    case 1: return sddmm_kernel<TF, VW, V, 1, SMAX>;
    case 2: return sddmm_kernel<TF, VW, V, 2, SMAX>;
    case 4: return sddmm_kernel<TF, VW, V, 4, SMAX>;
  }
  return nullptr;
}
template <typename TF, int VW>
SddmmFn pick_sddmm_v(int V, int vws, int S) {
  if (S > 1) return V == 64 ? pick_sddmm_vws<TF, VW, 64, 4>(vws) : nullptr;
  switch (V) {
    case 1: return pick_sddmm_vws<TF, VW, 1, 1>(vws);
    case 2: return pick_sddmm_vws<TF, VW, 2, 1>(vws);
    case 4: return pick_sddmm_vws<TF, VW, 4, 1>(vws);
    case 8: return pick_sddmm_vws<TF, VW, 8, 1>(vws);
    case 16: return pick_sddmm_vws<TF, VW, 16, 1>(vws);
    case 32: return pick_sddmm_vws<TF, VW, 32, 1>(vws);
    case 64: return pick_sddmm_vws<TF, VW, 64, 1>(vws);
  }
  return nullptr;
}
// defined in sddmm_f32.cu / sddmm_bf16.cu (V = L * R vectors per slice, S <= 4 slices)
SddmmFn pick_sddmm_f32(int vw, int V, int vws, int S);
SddmmFn pick_sddmm_bf16(int vw, int V, int vws, int S);

// dynamic shared memory per warp of the instantiation with Lg lanes per dot product
inline int sddmm_tile_bytes_per_warp(int lg, int vws) { return tile_bytes_per_warp(lg, vws); }
// the vw_sparse the dispatcher actually instantiates (a batch must cover whole vectors)
inline int sddmm_effective_vws(int V, int S, int vws) {
  const int r = S > 1 ? 2 : ((V >= GNN_SDDMM_R2_FROM && V >= 2) ? 2 : 1);
  int depth = GNN_SDDMM_UR / r;
  if (depth < 1) depth = 1;
  while (vws > depth) vws >>= 1;
  return vws;
}

// lanes per dot product of the instantiation pick_sddmm_* returns
inline int sddmm_group_lanes(int V, int S) {
  if (S > 1) return SddmmShape<8, 64, 4>::Lg;
  const int r = (V >= GNN_SDDMM_R2_FROM && V >= 2) ? 2 : 1;
  return V / r;
}
}  // namespace gnn
