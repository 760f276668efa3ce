// Plain ELLPACK, (BRO-)COO, fix-up and replicate instances.
#include "kernels.cuh"
#include "launch.hpp"

namespace bro {

constexpr int kPlainThreads = 256;
// COO: one warp per interval, 8-warp blocks, <= 128 registers (16 warps/SM)
constexpr int kCooWarps = 8;
constexpr int kCooMinBlocks = 2;

template <typename T>
static KernelRef plain_ell_impl(int mode) {
  using namespace dev;
  switch (mode) {
    case 0: return {(const void*)&ell_spmv<T, kPlainThreads, kSpmv>, kPlainThreads};
    case 1: return {(const void*)&ell_spmv<T, kPlainThreads, kScatter>, kPlainThreads};
    case 2: return {(const void*)&ell_spmv<T, kPlainThreads, kDecode>, kPlainThreads};
  }
  return {};
}

template <typename T, bool kBro, int TT>
static KernelRef coo_pick(int mode) {
  using namespace dev;
  if (mode == 2) return {(const void*)&coo_spmv<T, kBro, TT, kCooWarps, kCooMinBlocks, kDecode>, 32 * kCooWarps};
  return {(const void*)&coo_spmv<T, kBro, TT, kCooWarps, kCooMinBlocks, kSpmv>, 32 * kCooWarps};
}

template <typename T, bool kBro>
static KernelRef coo_pick_t(int TT, int mode) {
  switch (TT) {
    case 8: return coo_pick<T, kBro, 8>(mode);
    case 16: return coo_pick<T, kBro, 16>(mode);
    case 32: return coo_pick<T, kBro, 32>(mode);
  }
  return {};
}

template <typename T>
static KernelRef coo_impl(bool bro, int TT, int mode) {
  return bro ? coo_pick_t<T, true>(TT, mode) : coo_pick_t<T, false>(TT, mode);
}

template <> KernelRef plain_ell_ref<double>(int mode) { return plain_ell_impl<double>(mode); }
template <> KernelRef plain_ell_ref<float>(int mode) { return plain_ell_impl<float>(mode); }
template <> KernelRef coo_ref<double>(bool bro, int TT, int mode) { return coo_impl<double>(bro, TT, mode); }
template <> KernelRef coo_ref<float>(bool bro, int TT, int mode) { return coo_impl<float>(bro, TT, mode); }
template <> KernelRef fixup_ref<double>() { return {(const void*)&dev::coo_fixup<double>, 256}; }
template <> KernelRef fixup_ref<float>() { return {(const void*)&dev::coo_fixup<float>, 256}; }
template <> KernelRef replicate_ref<double>() { return {(const void*)&dev::replicate_y<double>, 256}; }
template <> KernelRef replicate_ref<float>() { return {(const void*)&dev::replicate_y<float>, 256}; }

}  // namespace bro
