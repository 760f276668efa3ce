// BRO-ELL instances, fp64 (see kern_ell.cuh).
#include "kern_ell.cuh"
namespace bro {
template <> KernelRef bro_ell_ref<double>(int V, int R, int inst, int mode) {
  return bro_ell_ref_impl<double>(V, R, inst, mode);
}
template <> KernelRef bro_ell_xstage_ref<double>(int V) { return bro_ell_xstage_ref_impl<double>(V); }
}  // namespace bro
