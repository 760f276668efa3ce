// Value-indexed BRO-ELL instances, fp32 (see kern_ell.cuh; reading R28).
#include "kern_ell.cuh"
namespace bro {
template <> KernelRef bro_ell_vi_ref<float>(int V, int R, int inst, int cb) {
  return bro_ell_vi_ref_impl<float>(V, R, inst, cb);
}
}  // namespace bro
