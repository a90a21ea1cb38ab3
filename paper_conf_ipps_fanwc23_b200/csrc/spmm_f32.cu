// spmm_f32.cu -- fp32-feature SpMM instantiations, sum aggregator (VW in fp32 elements).
#include "spmm_kernel.cuh"

namespace gnn {
SpmmFn pick_spmm_f32(int vw, int L, int R, int vws) {
  switch (vw) {
    case 1: return spmm_pick_l<F32, 1, kAggSum>(L, R, vws);
    case 2: return spmm_pick_l<F32, 2, kAggSum>(L, R, vws);
    case 4: return spmm_pick_l<F32, 4, kAggSum>(L, R, vws);
    case 8: return spmm_pick_l<F32, 8, kAggSum>(L, R, vws);
  }
  return nullptr;
}
}  // namespace gnn
