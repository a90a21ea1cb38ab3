// spmm_f32.cu -- fp32-feature SpMM instantiations (VW in fp32 elements: 1, 2, 4, 8).
#include "spmm_kernel.cuh"

namespace gnn {
SpmmFn pick_spmm_f32(int vw, int L, int R, int vws) {
  switch (vw) {
    case 1: return spmm_pick_l<F32, 1>(L, R, vws);
    case 2: return spmm_pick_l<F32, 2>(L, R, vws);
    case 4: return spmm_pick_l<F32, 4>(L, R, vws);
    case 8: return spmm_pick_l<F32, 8>(L, R, vws);
  }
  return nullptr;
}
}  // namespace gnn
