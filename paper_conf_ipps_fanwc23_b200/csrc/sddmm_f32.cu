// sddmm_f32.cu -- fp32-feature SDDMM instantiations (VW in fp32 elements: 1, 2, 4, 8).
#include "sddmm_kernel.cuh"

namespace gnn {
SddmmFn pick_sddmm_f32(int vw, int V, int vws, int S) {
  if (S > 4) return nullptr;
  switch (vw) {
    case 1: return pick_sddmm_v<F32, 1>(V, vws, S);
    case 2: return pick_sddmm_v<F32, 2>(V, vws, S);
    case 4: return pick_sddmm_v<F32, 4>(V, vws, S);
    case 8: return pick_sddmm_v<F32, 8>(V, vws, S);
  }
  return nullptr;
}
}  // namespace gnn
