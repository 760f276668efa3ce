// Value-indexed BRO-ELL instances, fp64 (see kern_ell.cuh; reading R28).
#include "kern_ell.cuh"
namespace bro {
template <> KernelRef bro_ell_vi_ref<double>(int V, int R, int inst, int cb) {
  return bro_ell_vi_ref_impl<double>(V, R, inst, cb);
}
}  // namespace bro
