// BRO-ELL instance table (included by kern_ell64.cu / kern_ell32.cu, one
// translation unit per value type so the two compile in parallel).
//
// Instances (R = rows per lane: 1 for h = 32, 2 for h = 64):
//   TINY  every slice <= 4 columns: register-resident decode
//   FEW   fewer slices than resident warps (R = 1): 16 (fp64) / 32 (fp32)
//         columns in flight per warp at ~128 registers — every warp is
//         resident anyway, so registers buy memory-level parallelism
//   SMALL every row stream < 10 symbols: 10-row window (less shared memory,
//         more L1 for the x gather); + TMA L2 prefetch of the next slice
//   MID   < 18 symbols: 18-row window
//   GEN   any slice: 34-row window
// Launch bounds fix the register budget: kMinBlocks blocks of kWarps warps.
// Every configuration below was chosen by in-process A/B on B200
// (scripts/ab.py; profiles/r02/README.md lists the measurements).
#pragma once
#include "kernels.cuh"
#include "launch.hpp"

namespace bro {

template <typename T, int V, int R, int M, int VI = 0>
KernelRef ell_pick(int inst) {
  using namespace dev;
  constexpr bool f64 = sizeof(T) == 8;
  constexpr int SB = 4;  // symbol rows per staging round trip (measured best, profiles/r02/)
  if ((inst == ELL_FEW || inst == ELL_SPLIT || inst == ELL_SPLIT2) && R == 2) inst = ELL_GEN;
  if constexpr (R == 1) {
    switch (inst) {
      case ELL_TINY: return {(const void*)&bro_ell_tiny<T, V, 1, 8, f64 ? 5 : 6, M, VI>, 256};
      case ELL_FEW:
        if constexpr (f64) return {(const void*)&bro_ell_od<T, V, 1, 8, 2, 16, kEllRowsGen, M, 0, false, 0, false, SB, false, 1, VI>, 256};
        else return {(const void*)&bro_ell_od<T, V, 1, 4, 2, 32, kEllRowsGen, M, 0, false, 0, false, SB, false, 1, VI>, 128};
      case ELL_SMALL:
        // fp64: 24 warps/SM, pipelined 4-column groups, TMA L2 prefetch of the
        // warp's next slice; fp32: 32 warps/SM, 8-column groups
        if constexpr (f64) return {(const void*)&bro_ell_od<T, V, 1, 8, 3, 4, kEllRowsSmall, M, 1, false, 0, true, SB, false, 1, VI>, 256};
        else return {(const void*)&bro_ell_od<T, V, 1, 16, 2, 8, kEllRowsSmall, M, 0, false, 0, false, SB, false, 1, VI>, 512};
      case ELL_MID:
        // C4's ELL part: short slices, latency-bound per slice; fp64 at 40
        // warps/SM with 4-column groups, fp32 at 32 with 8
        if constexpr (f64) return {(const void*)&bro_ell_od<T, V, 1, 8, 5, 4, kEllRowsMid, M, 0, false, 0, false, SB, false, 1, VI>, 256};
        else return {(const void*)&bro_ell_od<T, V, 1, 8, 4, 8, kEllRowsMid, M, 0, false, 0, false, SB, false, 1, VI>, 256};
      case ELL_GEN: return {(const void*)&bro_ell_od<T, V, 1, 8, 4, 8, kEllRowsGen, M, 0, false, 0, false, SB, false, 1, VI>, 256};
      // few long slices: 4 (SPLIT) or 2 (SPLIT2) warps per slice, 8-column groups, 32 warps/SM
      case ELL_SPLIT:
        return {(const void*)&bro_ell_od<T, V, 1, 8, 4, 8, kEllRowsGen, M, 0, false, 0, false, SB, false, 4, VI>, 256};
      case ELL_SPLIT2:
        return {(const void*)&bro_ell_od<T, V, 1, 8, 4, 8, kEllRowsGen, M, 0, false, 0, false, SB, false, 2, VI>, 256};
    }
  } else {
    switch (inst) {
      case ELL_TINY: return {(const void*)&bro_ell_tiny<T, V, 2, 8, 4, M, VI>, 256};
      case ELL_SMALL:
        // TMA L2 prefetch of the warp's next slice; the prefetched bytes wait in
        // L2 for about one slice time, so the warps per SM are chosen to keep
        // them near 35-40 MB chip-wide: 16 warps (fp64, 14.7 KB slices of C5),
        // 32 warps (fp32, 8.7 KB).  Value-indexed fp64 slices are 4x smaller:
        // 24 warps (C5 fp64 311 vs 400 us at 16, profiles/r02/s2/vi/)
        if constexpr (f64 && VI > 0) return {(const void*)&bro_ell_od<T, V, 2, 8, 3, 4, kEllRowsSmall, M, 1, false, 0, false, SB, false, 1, VI>, 256};
        else if constexpr (f64) return {(const void*)&bro_ell_od<T, V, 2, 8, 2, 4, kEllRowsSmall, M, 1, false, 0, false, SB, false, 1, VI>, 256};
        else return {(const void*)&bro_ell_od<T, V, 2, 8, 4, 4, kEllRowsSmall, M, 1, false, 0, false, SB, false, 1, VI>, 256};
      case ELL_MID: return {(const void*)&bro_ell_od<T, V, 2, 8, 3, 4, kEllRowsMid, M, 0, false, 0, false, SB, false, 1, VI>, 256};
      case ELL_GEN: return {(const void*)&bro_ell_od<T, V, 2, 4, 4, 4, kEllRowsGen, M, 0, false, 0, false, SB, false, 1, VI>, 128};

    }
  }
  return {};
}

template <typename T, int V, int R>
KernelRef ell_pick_mode(int inst, int mode) {
  switch (mode) {
    case 0: return ell_pick<T, V, R, dev::kSpmv>(inst);
    case 1: return ell_pick<T, V, R, dev::kScatter>(inst);
    case 2: return ell_pick<T, V, R, dev::kDecode>(inst);
  }
  return {};
}

// the few-slice instance with its block's x window staged in shared memory
// (same launch shape as ELL_FEW, spmv mode)
template <typename T, int V>
KernelRef ell_xstage_pick() {
  using namespace dev;
  constexpr bool f64 = sizeof(T) == 8;
  if constexpr (f64) return {(const void*)&bro_ell_od<T, V, 1, 8, 2, 16, kEllRowsGen, kSpmv, 0, false, 0, false, 4, true>, 256};
  else return {(const void*)&bro_ell_od<T, V, 1, 4, 2, 32, kEllRowsGen, kSpmv, 0, false, 0, false, 4, true>, 128};
}

template <typename T>
KernelRef bro_ell_xstage_ref_impl(int V) {
  return V == 1 ? ell_xstage_pick<T, 1>() : ell_xstage_pick<T, 4>();
}

// value-indexed instances (spmv mode; cb = bytes per value code)
template <typename T>
KernelRef bro_ell_vi_ref_impl(int V, int R, int inst, int cb) {
  using dev::kSpmv;
  const bool one = cb == 1;
  if (V == 1 && R == 1) return one ? ell_pick<T, 1, 1, kSpmv, 1>(inst) : ell_pick<T, 1, 1, kSpmv, 2>(inst);
  if (V == 1 && R == 2) return one ? ell_pick<T, 1, 2, kSpmv, 1>(inst) : ell_pick<T, 1, 2, kSpmv, 2>(inst);
  if (V == 4 && R == 1) return one ? ell_pick<T, 4, 1, kSpmv, 1>(inst) : ell_pick<T, 4, 1, kSpmv, 2>(inst);
  if (V == 4 && R == 2) return one ? ell_pick<T, 4, 2, kSpmv, 1>(inst) : ell_pick<T, 4, 2, kSpmv, 2>(inst);
  return {};
}

template <typename T>
KernelRef bro_ell_ref_impl(int V, int R, int inst, int mode) {
  if (V == 1 && R == 1) return ell_pick_mode<T, 1, 1>(inst, mode);
  if (V == 1 && R == 2) return ell_pick_mode<T, 1, 2>(inst, mode);
  if (V == 4 && R == 1) return ell_pick_mode<T, 4, 1>(inst, mode);
  if (V == 4 && R == 2) return ell_pick_mode<T, 4, 2>(inst, mode);
  return {};
}

}  // namespace bro
