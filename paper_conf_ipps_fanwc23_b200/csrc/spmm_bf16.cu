// spmm_bf16.cu -- bf16-feature SpMM instantiations (half the gathered bytes, fp32 accumulation and output; VW in bf16 elements).
#include "spmm_kernel.cuh"

namespace gnn {
SpmmFn pick_spmm_bf16(int vw, int L, int R, int vws) {
  switch (vw) {
    case 2: return spmm_pick_l<BF16, 2, kAggSum>(L, R, vws);
    case 4: return spmm_pick_l<BF16, 4, kAggSum>(L, R, vws);
    case 8: return spmm_pick_l<BF16, 8, kAggSum>(L, R, vws);
    case 16: return spmm_pick_l<BF16, 16, kAggSum>(L, R, vws);
  }
  return nullptr;
}
}  // namespace gnn
