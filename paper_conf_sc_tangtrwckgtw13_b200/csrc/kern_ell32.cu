// BRO-ELL instances, fp32 (see kern_ell.cuh).
#include "kern_ell.cuh"
namespace bro {
template <> KernelRef bro_ell_ref<float>(int V, int R, int inst, int mode) {
  return bro_ell_ref_impl<float>(V, R, inst, mode);
}
template <> KernelRef bro_ell_xstage_ref<float>(int V) { return bro_ell_xstage_ref_impl<float>(V); }
}  // namespace bro
