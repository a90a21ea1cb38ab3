// spmm_f32_max.cu -- fp32-feature SpMM with the max aggregator (MPP Eq. 1).
#include "spmm_kernel.cuh"

namespace gnn {
SpmmFn pick_spmm_f32_max(int vw, int L, int R, int vws) {
  switch (vw) {
    case 1: return spmm_pick_l<F32, 1, kAggMax>(L, R, vws);
    case 2: return spmm_pick_l<F32, 2, kAggMax>(L, R, vws);
    case 4: return spmm_pick_l<F32, 4, kAggMax>(L, R, vws);
    case 8: return spmm_pick_l<F32, 8, kAggMax>(L, R, vws);
  }
  return nullptr;
}
}  // namespace gnn
