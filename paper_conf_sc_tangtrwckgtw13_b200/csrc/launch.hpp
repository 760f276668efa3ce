// Kernel table shared by the host API (capi.cu) and the kernel translation
// units (kern_*.cu): every kernel of a family has the same signature, so a
// handle resolves its instances once at create time (per device) and launches
// them through cudaLaunchKernel.
#pragma once

namespace bro {

struct KernelRef {
  const void* fn = nullptr;
  int threads = 0;
  int warps_per_block() const { return threads / 32; }
};

// BRO-ELL kernel instances (bro_opts_t.ell_kernel; 0 = chosen at create)
enum EllInst { ELL_AUTO = 0, ELL_TINY = 1, ELL_FEW = 2, ELL_SMALL = 3, ELL_MID = 4, ELL_GEN = 5, ELL_SPLIT = 6,
               ELL_SPLIT2 = 7, ELL_LAST = 7 };
// the x-window-staged variant of the few-slice instance (bro_ell_xstage_ref)
constexpr int kXStageMaxBytes = 96 * 1024;  // largest x window staged per block
constexpr int kEllTinyCols = 4;   // TINY: every slice has <= 4 columns
constexpr int kEllRowsSmall = 10; // SMALL: every row stream < 10 symbols
constexpr int kEllRowsMid = 18;   // MID:   < 18 symbols
constexpr int kEllRowsGen = 34;   // GEN:   any

// mode: 0 = y = A.x, 1 = scatter (y into every destination), 2 = decode
template <typename T> KernelRef bro_ell_ref(int V, int R, int inst, int mode);
template <typename T> KernelRef bro_ell_xstage_ref(int V);  // few-slice instance, x window in shared memory
template <typename T> KernelRef bro_ell_vi_ref(int V, int R, int inst, int cb);  // value-indexed, spmv mode
template <typename T> KernelRef plain_ell_ref(int mode);
template <typename T> KernelRef coo_ref(bool bro, int TT, int mode);  // mode 0 or 2
template <typename T> KernelRef fixup_ref();
template <typename T> KernelRef replicate_ref();

}  // namespace bro
