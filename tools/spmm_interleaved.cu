// spmm_interleaved.cu -- EXPERIMENT (not the product; verdict round 1, item 8): the SpMM
// lane mapping named in BASELINE.json's north_star -- the G lane groups of a warp take
// INTERLEAVED nonzeros of one chunk and merge their partial rows with a warp-shuffle
// reduction -- measured against the product's mapping (each group walks its own chunk).
// The cross-group reduction runs only where a row ENDS (not per nonzero): partial sums of
// a row that continues into the next window stay in each group's registers.
//
// fp32, sum, VW = 8 (K = 8 L), L = K / 8 lanes per group, G = 32 / L groups, one warp per
// chunk of C consecutive nonzeros.  A window is G * 4 consecutive nonzeros: group g takes
// entries g, g + G, g + 2G, g + 3G (4 feature rows in flight per lane, as the product's
// lean kernels).  For each distinct row r in the window (warp min over unprocessed rows),
// every group adds its entries of row r; if r ends inside the window (or at the chunk
// end), a log2(G)-round xor butterfly over the groups sums the partials and group 0
// flushes: plain store for a row owned by the chunk, red.add for a row shared with a
// neighbouring chunk.  O must be zeroed first (exp_spmm_interleaved does a memset).
// Built into variants/libgnnexp.so (make exp); tools/interleaved_ab.py times it.
#include <cuda_runtime.h>
#include <stdint.h>

#include "../paper_conf_ipps_fanwc23_b200/csrc/device.cuh"

namespace {
using namespace gnn;

template <int L>
__global__ void __launch_bounds__(128) spmm_interleaved_kernel(
    const int32_t *__restrict__ row_ind, const int32_t *__restrict__ col_ind,
    const float *__restrict__ val, int64_t nnz, int32_t C, const float *__restrict__ A,
    int64_t lda, float *__restrict__ O, int64_t ldo) {
  constexpr int G = 32 / L, U = 4, W = G * U;
  const int lane = threadIdx.x & 31, g = lane / L, l = lane % L;
  const int64_t c = (int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  const int64_t cs = c * C;
  if (cs >= nnz) return;  // warp-uniform
  const int64_t ce = cs + C < nnz ? cs + C : nnz;
  const int32_t rf = row_ind[cs], rl = row_ind[ce - 1];
  const bool head = cs > 0 && row_ind[cs - 1] == rf;
  const bool tail = ce < nnz && row_ind[ce] == rl;
  const float *Al = A + l * 8;
  float acc[8];
#pragma unroll
  for (int v = 0; v < 8; ++v) acc[v] = 0.f;
  for (int64_t b = cs; b < ce; b += W) {
    int32_t r[U];
    float vv[U], x[U][8];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t i = b + g + (int64_t)G * u;
      if (i < ce) {
        r[u] = __ldg(row_ind + i);
        vv[u] = val ? __ldg(val + i) : 1.f;
        ld_feat<8>(Al + (int64_t)__ldg(col_ind + i) * lda, x[u]);
      } else {
        r[u] = INT32_MAX;
        vv[u] = 0.f;
#pragma unroll
        for (int v = 0; v < 8; ++v) x[u][v] = 0.f;
      }
    }
    const int64_t we = b + W < ce ? b + W : ce;  // window end
    const int32_t r_last = __ldg(row_ind + we - 1);
    // does the window's last row continue past it (into the next window of this chunk)?
    const bool last_continues = we < ce && __ldg(row_ind + we) == r_last;
    unsigned done = 0;  // per-lane bitmask of processed u
    for (;;) {
      int32_t mine = INT32_MAX;
#pragma unroll
      for (int u = 0; u < U; ++u)
        if (!(done >> u & 1) && r[u] < mine) mine = r[u];
      const int32_t row = __reduce_min_sync(kFull, mine);
      if (row == INT32_MAX) break;
#pragma unroll
      for (int u = 0; u < U; ++u)
        if (r[u] == row) {
          axpy<8>(acc, vv[u], x[u]);
          done |= 1u << u;
        }
      if (row == r_last && last_continues) break;  // row goes on: keep the partials
      // row ends here: sum the G groups' partials (xor butterfly), group 0 flushes
#pragma unroll
      for (int o = L; o < 32; o <<= 1)
#pragma unroll
        for (int v = 0; v < 8; ++v) acc[v] += __shfl_xor_sync(kFull, acc[v], o);
      if (g == 0 && l * 8 < 8 * L) {
        float *o = O + (int64_t)row * ldo + l * 8;
        if ((row == rf && head) || (row == rl && tail)) red_add<8>(o, acc);
        else st_vec<8>(o, acc);
      }
#pragma unroll
      for (int v = 0; v < 8; ++v) acc[v] = 0.f;
    }
  }
}
// Control with the same memory code: each group walks its OWN chunk (the product's
// mapping), 4 nonzeros in flight per lane, a row's sum flushed by the group at its end.
template <int L>
__global__ void __launch_bounds__(128) spmm_ownchunk_kernel(
    const int32_t *__restrict__ row_ind, const int32_t *__restrict__ col_ind,
    const float *__restrict__ val, int64_t nnz, int32_t C, const float *__restrict__ A,
    int64_t lda, float *__restrict__ O, int64_t ldo) {
  constexpr int G = 32 / L, U = 4;
  const int lane = threadIdx.x & 31, g = lane / L, l = lane % L;
  const int64_t c = ((int64_t)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)) * G + g;
  const int64_t cs = c * C;
  if (cs >= nnz) return;  // (group-uniform; no warp collectives below)
  const int64_t ce = cs + C < nnz ? cs + C : nnz;
  const int32_t rf = row_ind[cs], rl = row_ind[ce - 1];
  const bool head = cs > 0 && row_ind[cs - 1] == rf;
  const bool tail = ce < nnz && row_ind[ce] == rl;
  const float *Al = A + l * 8;
  float acc[8];
#pragma unroll
  for (int v = 0; v < 8; ++v) acc[v] = 0.f;
  int32_t cur = rf;
  for (int64_t b = cs; b < ce; b += U) {
    int32_t r[U];
    float vv[U], x[U][8];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t i = b + u;
      if (i < ce) {
        r[u] = __ldg(row_ind + i);
        vv[u] = val ? __ldg(val + i) : 1.f;
        ld_feat<8>(Al + (int64_t)__ldg(col_ind + i) * lda, x[u]);
      } else {
        r[u] = -1;
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if (r[u] < 0) continue;
      if (r[u] != cur) {
        float *o = O + (int64_t)cur * ldo + l * 8;
        if ((cur == rf && head) || (cur == rl && tail)) red_add<8>(o, acc);
        else st_vec<8>(o, acc);
#pragma unroll
        for (int v = 0; v < 8; ++v) acc[v] = 0.f;
        cur = r[u];
      }
      axpy<8>(acc, vv[u], x[u]);
    }
  }
  float *o = O + (int64_t)cur * ldo + l * 8;
  if ((cur == rf && head) || (cur == rl && tail)) red_add<8>(o, acc);
  else st_vec<8>(o, acc);
}
}  // namespace

extern "C" __attribute__((visibility("default"))) int exp_spmm_ownchunk(
    const int32_t *row_ind, const int32_t *col_ind, const float *val, int64_t nnz, int64_t M,
    int32_t K, int32_t C, const float *A, int64_t lda, float *O, int64_t ldo, int zero_O,
    void *stream) {
  cudaStream_t s = (cudaStream_t)stream;
  if (zero_O) cudaMemsetAsync(O, 0, sizeof(float) * M * ldo, s);
  if (nnz == 0) return 0;
  const int64_t nch = (nnz + C - 1) / C;
  const int G = 32 / (K / 8);
  const unsigned blocks = (unsigned)((nch + 4 * G - 1) / (4 * G));
  switch (K) {
    case 32: spmm_ownchunk_kernel<4><<<blocks, 128, 0, s>>>(row_ind, col_ind, val, nnz, C, A, lda, O, ldo); break;
    case 64: spmm_ownchunk_kernel<8><<<blocks, 128, 0, s>>>(row_ind, col_ind, val, nnz, C, A, lda, O, ldo); break;
    case 128: spmm_ownchunk_kernel<16><<<blocks, 128, 0, s>>>(row_ind, col_ind, val, nnz, C, A, lda, O, ldo); break;
    case 256: spmm_ownchunk_kernel<32><<<blocks, 128, 0, s>>>(row_ind, col_ind, val, nnz, C, A, lda, O, ldo); break;
    default: return 1;
  }
  return cudaGetLastError() == cudaSuccess ? 0 : 2;
}

extern "C" __attribute__((visibility("default"))) int exp_spmm_interleaved(
    const int32_t *row_ind, const int32_t *col_ind, const float *val, int64_t nnz, int64_t M,
    int32_t K, int32_t C, const float *A, int64_t lda, float *O, int64_t ldo, int zero_O,
    void *stream) {
  cudaStream_t s = (cudaStream_t)stream;
  if (zero_O) cudaMemsetAsync(O, 0, sizeof(float) * M * ldo, s);
  if (nnz == 0) return 0;
  const int64_t nch = (nnz + C - 1) / C;
  const unsigned blocks = (unsigned)((nch + 3) / 4);
  switch (K) {
    case 32: spmm_interleaved_kernel<4><<<blocks, 128, 0, s>>>(row_ind, col_ind, val, nnz, C, A, lda, O, ldo); break;
    case 64: spmm_interleaved_kernel<8><<<blocks, 128, 0, s>>>(row_ind, col_ind, val, nnz, C, A, lda, O, ldo); break;
    case 128: spmm_interleaved_kernel<16><<<blocks, 128, 0, s>>>(row_ind, col_ind, val, nnz, C, A, lda, O, ldo); break;
    case 256: spmm_interleaved_kernel<32><<<blocks, 128, 0, s>>>(row_ind, col_ind, val, nnz, C, A, lda, O, ldo); break;
    default: return 1;
  }
  return cudaGetLastError() == cudaSuccess ? 0 : 2;
}
