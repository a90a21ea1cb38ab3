// sddmm_bf16.cu -- bf16-feature SDDMM instantiations (VW in bf16
// elements: 2, 4, 8, 16; products and sums in fp32).
#include "sddmm_kernel.cuh"

namespace gnn {
SddmmFn pick_sddmm_bf16(int vw, int V, int vws, int S) {
  if (S > 4) return nullptr;
  switch (vw) {
    case 2: return pick_sddmm_v<BF16, 2>(V, vws, S);
    case 4: return pick_sddmm_v<BF16, 4>(V, vws, S);
    case 8: return pick_sddmm_v<BF16, 8>(V, vws, S);
    case 16: return pick_sddmm_v<BF16, 16>(V, vws, S);
  }
  return nullptr;
}
}  // namespace gnn
