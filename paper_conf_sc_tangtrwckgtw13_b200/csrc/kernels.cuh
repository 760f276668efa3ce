// sm_100a SpMV kernels for BRO-ELL, BRO-COO (+ carry fix-up) and the
// uncompressed ELLPACK / COO baselines.
//
// Mapping (B200-first; the paper's Fermi/Kepler mapping of one 256-thread
// block per slice, is prior art):
//   * BRO-ELL (bro_ell_spmv_od): one WARP per 32-row slice, one lane per row
//     (h = 32), persistent warps.  Widths are warp-uniform, so every
//     column's bit offset is uniform too: a SHFL scan of the widths gives the
//     offsets of a 32-column block, the block's symbols are staged in a
//     per-warp shared window, and each delta is a branch-free funnel-shift
//     extraction, fused with the x gather and the FMA (the load-decode-compute
//     cycle of Alg. 1 without its per-column branch).
//   * BRO-COO (coo_spmv<kBro=true>): one warp per interval of 32*T entries
//     (P:L140); rows decoded per (step, lane), then a transposed 256-entry
//     batch per iteration (lane owns 8 consecutive entries), sequential lane
//     reduction + one warp segmented scan (the "parallel scan primitive",
//     P:L343) and a deterministic fix-up kernel for rows crossing intervals
//     (the "extra kernel invocation for data reduction").
//   * Uncompressed baselines: ell_spmv (thread per row, column-major ELLPACK)
//     and coo_spmv<kBro=false> (same COO traversal, explicit rows).
//   * Streamed arrays (symbols, values) are read with 16-byte
//     ld.global.nc.L1::no_allocate loads; x is gathered through the
//     read-only path.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include <type_traits>

namespace bro {
namespace dev {

constexpr int kWarp = 32;

// ------------------------------------------------------------------ loads
// BRO_L2_PF: L2 prefetch-size qualifier of the streamed loads.  Measured
// (profiles/r01/s4/ab_l2_256B.txt, A/B in one session): neutral for every
// BRO kernel (C5 f64 343.1 vs 343.8 us, f32 250.4 vs 250.3, C4 111.7 vs
// 111.7, C2 18.5 vs 18.5) and up to 3% faster for the uncompressed ELLPACK
// baseline (C2 27.9 -> 27.0 us), so it is on for both: the speedups are
// quoted against the faster baseline.  -DBRO_L2_PF='""' turns it off.
#ifndef BRO_L2_PF
#define BRO_L2_PF ".L2::256B"
#endif
// Streamed arrays (values, symbols, COO col/row) are read with non-volatile
// inline asm ld.global.nc.L1::no_allocate.  The compiler treats these as pure
// and may issue a guarded load (cond ? ld(p) : 0, or the full-chunk path of
// a partial group) speculatively and select the result — that is what makes
// the tail code branch-free.  The library therefore pads every device array
// by kStreamPad zeroed bytes: the farthest speculated address (a COO tail,
// < 1024 entries past nnz) stays inside the allocation, so compute-sanitizer
// memcheck is clean.  Measured on C5: real-load builtins (__ldg / __ldcs)
// for the guarded loads cost 10-14% on fp32 (per-element branches).
constexpr int kStreamPad = 16384;

__device__ __forceinline__ uint4 ld_stream_u4(const uint32_t* p) {
  uint4 r;
  asm("ld.global.nc.L1::no_allocate" BRO_L2_PF ".v4.u32 {%0,%1,%2,%3}, [%4];"
      : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ uint32_t ld_stream_u32(const uint32_t* p) {
  uint32_t r;
  asm("ld.global.nc.L1::no_allocate" BRO_L2_PF ".u32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ int32_t ld_stream_s32(const int32_t* p) {
  int32_t r;
  asm("ld.global.nc.L1::no_allocate" BRO_L2_PF ".s32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ double ld_stream(const double* p) {
  double r;
  asm("ld.global.nc.L1::no_allocate" BRO_L2_PF ".f64 %0, [%1];" : "=d"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ float ld_stream(const float* p) {
  float r;
  asm("ld.global.nc.L1::no_allocate" BRO_L2_PF ".f32 %0, [%1];" : "=f"(r) : "l"(p));
  return r;
}

// 16-byte value chunk: 2 doubles or 4 floats
template <typename T> struct Chunk;
template <> struct Chunk<double> {
  double v[2];
  static constexpr int N = 2;
  __device__ __forceinline__ void load(const double* p) {
    asm("ld.global.nc.L1::no_allocate" BRO_L2_PF ".v2.f64 {%0,%1}, [%2];" : "=d"(v[0]), "=d"(v[1]) : "l"(p));
  }
};
template <> struct Chunk<float> {
  float v[4];
  static constexpr int N = 4;
  __device__ __forceinline__ void load(const float* p) {
    asm("ld.global.nc.L1::no_allocate" BRO_L2_PF ".v4.f32 {%0,%1,%2,%3}, [%4];"
        : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]) : "l"(p));
  }
};

template <typename T>
__device__ __forceinline__ T ldg_x(const T* p) { return __ldg(p); }

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// ------------------------------------------------------------------ y destinations
// Where an ELL kernel stores y[row].  n = 1 is plain SpMV.  n > 1 is the
// fused exchange of the row-block iteration: the same
// value is also stored into the x replica of every peer GPU (P2P stores
// through NVLink, p[i] = peer-mapped symmetric-memory pointers), so the
// allgather of y overlaps the SpMV row by row instead of following it.
// mc != nullptr: one multimem.st to an NVLS multicast address writes every
// bound replica (the local one included) through the NVSwitch, and p[] is
// unused.  Indices are static (unrolled) so the table stays in the
// kernel-parameter bank.
constexpr int kMaxDst = 8;
template <typename T>
struct YOut {
  T* p[kMaxDst];
  T* mc;
  int n;
};

__device__ __forceinline__ void multimem_st(double* a, double v) {
  asm volatile("multimem.st.relaxed.sys.global.f64 [%0], %1;" :: "l"(a), "d"(v) : "memory");
}
__device__ __forceinline__ void multimem_st(float* a, float v) {
  asm volatile("multimem.st.relaxed.sys.global.f32 [%0], %1;" :: "l"(a), "f"(v) : "memory");
}

template <bool kMulti, typename T>
__device__ __forceinline__ void store_y(const YOut<T>& o, int64_t row, T v) {
  if constexpr (!kMulti) {  // plain SpMV: one store, no destination table
    o.p[0][row] = v;
    return;
  }
  if (o.mc != nullptr) {
    multimem_st(o.mc + row, v);
    return;
  }
  o.p[0][row] = v;
#pragma unroll
  for (int i = 1; i < kMaxDst; ++i)
    if (i < o.n) o.p[i][row] = v;
}

// cp.async (LDGSTS) helpers
__device__ __forceinline__ void cp_async4(uint32_t* dst, const uint32_t* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" :: "r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" :: "n"(N) : "memory"); }

// shl with the PTX clamp (shift >= 32 gives 0)
__device__ __forceinline__ uint32_t shl_clamp(uint32_t v, uint32_t s) {
  uint32_t r;
  asm("shl.b32 %0, %1, %2;" : "=r"(r) : "r"(v), "r"(s));
  return r;
}

__device__ __forceinline__ int64_t place(int64_t r, int64_t q, int64_t S, int64_t V) {
  const int64_t F = S / V;
  const int64_t c = q / V;
  if (c < F) return kWarp * V * c + r * V + (q - c * V);
  return kWarp * V * F + r * (S - V * F) + (q - V * F);
}

// ------------------------------------------------------------------ lane bit stream
// One lane's multiplexed symbol stream read MSB-first through a 64-bit
// window.  Invariant: before every get(b) (1 <= b <= 32) the window holds at
// least 32 valid bits unless the stream is exhausted.  All branches depend
// only on S and on widths, which are warp-uniform.
template <int V>
struct LaneStream {
  const uint32_t* base;  // slice / interval word block
  int S;                 // symbols per lane
  int q;                 // symbols consumed so far
  int avail;             // valid bits in hi:lo
  uint32_t hi, lo;
  uint32_t buf[8];       // symbols q .. (q | 7) of this lane

  __device__ __forceinline__ void fetch8(int lane) {
    if constexpr (V == 4) {
      const int F = S >> 2;
      const int Vp = S - 4 * F;
#pragma unroll
      for (int h2 = 0; h2 < 2; ++h2) {
        const int c = (q >> 2) + h2;
        if (c < F) {
          uint4 v = ld_stream_u4(base + 128 * c + 4 * lane);
          buf[4 * h2 + 0] = v.x; buf[4 * h2 + 1] = v.y;
          buf[4 * h2 + 2] = v.z; buf[4 * h2 + 3] = v.w;
        } else {
#pragma unroll
          for (int k = 0; k < 4; ++k)
            buf[4 * h2 + k] = (c == F && k < Vp) ? ld_stream_u32(base + 128 * F + Vp * lane + k) : 0u;
        }
      }
    } else {
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const int qq = q + k;
        buf[k] = qq < S ? ld_stream_u32(base + place(lane, qq, S, V)) : 0u;
      }
    }
  }
  __device__ __forceinline__ uint32_t pop(int lane) {
    if ((q & 7) == 0) fetch8(lane);
    const uint32_t r = buf[0];
#pragma unroll
    for (int k = 0; k < 7; ++k) buf[k] = buf[k + 1];
    ++q;
    return r;
  }
  __device__ __forceinline__ void init(const uint32_t* b, int S_, int lane) {
    base = b; S = S_; q = 0;
    hi = 0; lo = 0; avail = 0;
    if (S > 0) { hi = pop(lane); avail = 32; }
  }
  __device__ __forceinline__ uint32_t get(int b, int lane) {  // 1 <= b <= 32
    const uint32_t v = hi >> (32 - b);
    hi = __funnelshift_lc(lo, hi, b);
    lo = shl_clamp(lo, b);
    avail -= b;
    if (avail < 32 && q < S) {
      const uint32_t w = pop(lane);
      hi |= w >> avail;
      lo = shl_clamp(w, 32 - avail);
      avail += 32;
    }
    return v;
  }
};

// Values of 8 consecutive slice columns j .. j+7 of this lane (16-byte
// chunks where the chunk is full, scalar loads in the tail chunk, 0 past l).
template <typename T, int G>
__device__ __forceinline__ void load_group_vals(T* v, const T* vs, int j, int l, int lfull, int lane) {
  constexpr int VV = Chunk<T>::N;
#pragma unroll
  for (int u = 0; u < G / VV; ++u) {
    const int jj = j + u * VV;
    if (jj + VV <= lfull) {
      Chunk<T> c;
      c.load(vs + 32 * jj + lane * VV);
#pragma unroll
      for (int k = 0; k < VV; ++k) v[u * VV + k] = c.v[k];
    } else {
      const int tw = l - lfull;  // tail slots per lane (< VV), contiguous per lane
#pragma unroll
      for (int k = 0; k < VV; ++k)
        v[u * VV + k] = (jj + k < l) ? ld_stream(vs + 32 * lfull + lane * tw + (jj + k - lfull)) : T(0);
    }
  }
}

// Group values: straight 16-byte loads when the whole group lies in full
// chunks (the common case), else the tail-aware path.
template <typename T, int G>
__device__ __forceinline__ void load_vals(T* v, const T* vs, int j, int l, int lfull, int lane) {
  constexpr int VV = Chunk<T>::N;
  if (j + G <= lfull) {
#pragma unroll
    for (int u = 0; u < G / VV; ++u) {
      Chunk<T> c;
      c.load(vs + 32 * (j + u * VV) + lane * VV);
#pragma unroll
      for (int q = 0; q < VV; ++q) v[u * VV + q] = c.v[q];
    }
  } else {
    load_group_vals<T, G>(v, vs, j, l, lfull, lane);
  }
}

// ------------------------------------------------------------------ BRO-ELL, offset decode
// Widths are warp-uniform (one per slice column), so the bit offset
// of column j inside every row stream is the same for all 32 lanes:
// o_j = sum_{i<j} b_i.  Per block of up to 32 columns the warp computes the
// offsets with one SHFL scan, stages the block's symbols (<= 33 per lane) in
// a per-warp shared window as [row][lane] (conflict-free), and then each
// column's delta is a branch-free extraction
//     delta = funnelshift(w[q+1], w[q], o mod 32) >> (32 - b),   q = o / 32
// fused with the x gather and the FMA (8 columns in flight per group).
// Bulk (TMA engine) prefetch of [p, p + bytes) into L2; p and bytes multiples of 16.
__device__ __forceinline__ void prefetch_l2(const void* p, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" :: "l"(p), "r"(bytes) : "memory");
}

__device__ __forceinline__ void prefetch_l2_line(const void* p) {
  asm volatile("prefetch.global.L2 [%0];" :: "l"(p));
}

__device__ __forceinline__ uint32_t shr_clamp(uint32_t v, uint32_t s) {
  uint32_t r;
  asm("shr.b32 %0, %1, %2;" : "=r"(r) : "r"(v), "r"(s));
  return r;
}

// Copy symbol rows [qa, qa + nrows) of this lane into win[(q - qa) * 32 + lane]
// (zeros past S) plus one zero guard row.
template <int V>
__device__ __forceinline__ void stage_symbols(uint32_t* win, const uint32_t* __restrict__ wb, int S, int qa,
                                              int nrows, int lane) {
  if constexpr (V == 1) {
    for (int r = 0; r < nrows; ++r) {
      const int q = qa + r;
      win[r * 32 + lane] = q < S ? __ldg(wb + 32 * q + lane) : 0u;
    }
  } else if constexpr (V == 4) {
    const int F = S >> 2;
    const int c_lo = qa >> 2, c_hi = (qa + nrows - 1) >> 2;
    for (int c = c_lo; c <= c_hi; ++c) {
      uint32_t w4[4];
      if (c < F) {
        const uint4 v = ld_stream_u4(wb + 128 * c + 4 * lane);
        w4[0] = v.x; w4[1] = v.y; w4[2] = v.z; w4[3] = v.w;
      } else {
        const int Vp = S - 4 * F;
#pragma unroll
        for (int k = 0; k < 4; ++k) w4[k] = (c == F && k < Vp) ? ld_stream_u32(wb + 128 * F + Vp * lane + k) : 0u;
      }
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const int r = 4 * c + k - qa;
        if (r >= 0 && r < nrows) win[r * 32 + lane] = w4[k];
      }
    }
  } else {
    for (int r = 0; r < nrows; ++r) {
      const int q = qa + r;
      win[r * 32 + lane] = q < S ? ld_stream_u32(wb + place(lane, q, S, V)) : 0u;
    }
  }
  win[nrows * 32 + lane] = 0u;
}

// G columns per group; kRows window rows per warp (34 holds any 32-column
// block: <= 33 symbol rows + a zero guard row).  The short-slice instance
// (G = 4, kRows = 6, 48 warps/SM) serves matrices whose slices all have
// l <= 4 columns (<= 4 symbols per row): less shared memory and fewer
// registers buy 1.5x the resident warps for the latency-bound short rows.
//
// kPf > 0: values move by cp.async (LDGSTS, no registers while in flight)
// into a per-warp ring of kPf + 1 group slots laid out exactly like the
// global chunks; groups 0 .. kPf-1 of a slice are issued before its widths
// and symbols are staged, so the value stream overlaps that round trip, and
// group g + kPf is issued while group g is decoded.
template <typename T, int G>
__device__ __forceinline__ void cp_async_group_vals(T* slot, const T* vs, int j, int l, int lfull, int lane) {
  constexpr int VV = Chunk<T>::N;
#pragma unroll
  for (int u = 0; u < G / VV; ++u) {
    const int jj = j + u * VV;
    T* d = slot + u * 32 * VV + lane * VV;
    if (jj + VV <= lfull) {
      asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" :: "r"(smem_u32(d)), "l"(vs + 32 * jj + lane * VV)
                   : "memory");
    } else if (jj < l) {
      const int tw = l - lfull;  // tail slots per lane (< VV), contiguous per lane
#pragma unroll
      for (int k = 0; k < VV; ++k)
        if (jj + k < l)
          asm volatile("cp.async.ca.shared.global [%0], [%1], %2;"
                       :: "r"(smem_u32(d + k)), "l"(vs + 32 * lfull + lane * tw + (jj + k - lfull)), "n"(sizeof(T))
                       : "memory");
    }
  }
}

template <typename T, int V, int kWarps, int kMinBlocks, int G = 8, int kRows = 34, bool kMulti = false, int kPf = 0>
__global__ void __launch_bounds__(kWarps * 32, kMinBlocks)
bro_ell_spmv_od(int64_t m, int64_t s, const uint32_t* __restrict__ words,
                const uint8_t* __restrict__ bit_alloc, const uint64_t* __restrict__ colptr,
                const uint64_t* __restrict__ symptr, const T* __restrict__ vals,
                const T* __restrict__ x, const YOut<T> y) {
  struct Meta { uint64_t c0, q0; int l, S; };
  constexpr int kNV = kPf + 1;
  __shared__ __align__(16) T vring[kPf ? kWarps : 1][kPf ? kNV * G * 32 : 1];
  __shared__ uint32_t window[kWarps][kRows * 32];
  __shared__ uint2 colmeta[kWarps][32];  // per column of the block: {byte offset of its word row, r | (32-b) << 8}
  __shared__ Meta metas[kWarps][32];     // metadata of this warp's next 32 slices
  const int lane = threadIdx.x & 31;
  const int w = threadIdx.x >> 5;
  uint32_t* win = window[w];
  const uint2* cm = colmeta[w];
  const char* win_lane = reinterpret_cast<const char*>(win + lane);
  const int64_t stride = int64_t(gridDim.x) * kWarps;
  int k32 = 0;
  for (int64_t t = int64_t(blockIdx.x) * kWarps + w; t < s; t += stride, k32 = (k32 + 1) & 31) {
    __syncwarp();
    if (k32 == 0) {  // one round trip fetches the metadata of the next 32 slices
      const int64_t tl = t + lane * stride;
      if (tl < s) {
        const uint64_t c0l = __ldg(colptr + tl), q0l = __ldg(symptr + tl);
        metas[w][lane] = Meta{c0l, q0l, int(__ldg(colptr + tl + 1) - c0l), int(__ldg(symptr + tl + 1) - q0l)};
      }
      __syncwarp();
    }
    const Meta mt = metas[w][k32];
    const uint64_t c0 = mt.c0;
    const int l = mt.l;
    const int S = mt.S;
    const uint32_t* wb = words + 32 * mt.q0;
    const T* vs = vals + 32 * c0;
    const uint8_t* ba = bit_alloc + c0;
    const int lfull = (l / Chunk<T>::N) * Chunk<T>::N;
    T sum = T(0);
    int col = -1;
    int obase = 0;  // bit offset of the current block inside every row stream
    if constexpr (kPf > 0) {  // first groups' values in flight before the staging round trip
#pragma unroll
      for (int p = 0; p < kPf; ++p) {
        if (p * G < l) cp_async_group_vals<T, G>(vring[w] + (p % kNV) * G * 32, vs, p * G, l, lfull, lane);
        cp_async_commit();
      }
    }
    for (int jb = 0; jb < l; jb += 32) {
      const int nb = min(32, l - jb);
      const int b = lane < nb ? int(__ldg(ba + jb + lane)) : 0;
      if (jb == 0) {  // first block starts at symbol 0: stage without waiting for the scan
        __syncwarp();
        stage_symbols<V>(win, wb, S, 0, min(S, kRows - 1), lane);
      }
      int incl = b;  // inclusive scan of the widths over the block
#pragma unroll
      for (int off = 1; off < 32; off <<= 1) {
        const int o = __shfl_up_sync(0xffffffffu, incl, off);
        if (lane >= off) incl += o;
      }
      const int tot = __shfl_sync(0xffffffffu, incl, 31);
      const int qa = jb == 0 ? 0 : obase >> 5;
      const int nrows = tot > 0 ? ((obase + tot - 1) >> 5) - qa + 1 : 0;
      if (jb > 0) {
        __syncwarp();
        stage_symbols<V>(win, wb, S, qa, nrows, lane);
      }
      {
        const int rel = b ? obase + incl - b - 32 * qa : 0;  // column jb+lane inside the window
        colmeta[w][lane] = make_uint2(uint32_t(rel >> 5) * 128u, uint32_t(rel & 31) | ((32u - uint32_t(b)) << 8));
      }
      __syncwarp();
      for (int g = 0; g < nb; g += G) {
        T v[G];
        if constexpr (kPf > 0) {
          const int gi = (jb + g) / G;  // group index within the slice
          const int jn = jb + g + kPf * G;
          if (jn < l) cp_async_group_vals<T, G>(vring[w] + ((gi + kPf) % kNV) * G * 32, vs, jn, l, lfull, lane);
          cp_async_commit();
          cp_async_wait<kPf>();
          const T* sl = vring[w] + (gi % kNV) * G * 32 + lane * Chunk<T>::N;
#pragma unroll
          for (int u = 0; u < G / Chunk<T>::N; ++u) {
            if constexpr (sizeof(T) == 8) {
              const double2 c2 = *reinterpret_cast<const double2*>(sl + u * 32 * Chunk<T>::N);
              v[2 * u] = c2.x; v[2 * u + 1] = c2.y;
            } else {
              const float4 c4 = *reinterpret_cast<const float4*>(sl + u * 32 * Chunk<T>::N);
              v[4 * u] = c4.x; v[4 * u + 1] = c4.y; v[4 * u + 2] = c4.z; v[4 * u + 3] = c4.w;
            }
          }
        } else {
          load_vals<T, G>(v, vs, jb + g, l, lfull, lane);
        }
        int cidx[G];
        bool ok[G];
#pragma unroll
        for (int k = 0; k < G; ++k) {
          const uint2 mm = cm[g + k];  // broadcast
          const uint32_t* wp = reinterpret_cast<const uint32_t*>(win_lane + mm.x);
          // funnelshift_l uses the low 5 bits of mm.y (= r); bits 8.. hold 32-b
          const uint32_t d = shr_clamp(__funnelshift_l(wp[32], wp[0], mm.y), mm.y >> 8);
          col += int(d);
          cidx[k] = col;
          ok[k] = d != 0u;
        }
        T xv[G];
#pragma unroll
        for (int k = 0; k < G; ++k)
          if (ok[k]) xv[k] = ldg_x(x + cidx[k]);
#pragma unroll
        for (int k = 0; k < G; ++k)
          if (ok[k]) sum = fma(v[k], xv[k], sum);  // padding slots (delta 0) are skipped, Alg. 1 line 17
      }
      obase += tot;
    }
    const int64_t row = 32 * t + lane;
    if (row < m) store_y<kMulti>(y, row, sum);
  }
}

// ------------------------------------------------------------------ BRO-ELL, tiny slices
// Every slice has l <= 4 columns (e.g. the ELL part of C3's BRO-HYB, K = 2),
// so a row stream has S <= 4 symbols (<= 4 fields of <= 32 bits): each lane
// keeps its <= 4 words in registers — no shared-memory window, no width
// scan, no column records.  Per slice one round trip fetches the widths
// (broadcast), the lane's words and its values together, then one fetches
// the x gathers; kSl slices are processed interleaved per warp iteration so
// their round trips overlap.  Field j starts at the warp-uniform offset
// o_j = b_0 + ... + b_{j-1}, so q = o_j / 32 selects the word pair uniformly.
template <typename T, int V, int kWarps, int kMinBlocks, int kSl>
__global__ void __launch_bounds__(kWarps * 32, kMinBlocks)
bro_ell_spmv_tiny(int64_t m, int64_t s, const uint32_t* __restrict__ words,
                  const uint8_t* __restrict__ bit_alloc, const uint64_t* __restrict__ colptr,
                  const uint64_t* __restrict__ symptr, const T* __restrict__ vals,
                  const T* __restrict__ x, const YOut<T> y) {
  struct Meta { uint64_t c0, q0; int l, S; };
  __shared__ Meta metas[kWarps][32];  // metadata of this warp's next 32 slices
  const int lane = threadIdx.x & 31;
  const int w = threadIdx.x >> 5;
  const int64_t stride = int64_t(gridDim.x) * kWarps;
  int k32 = 0;
  for (int64_t t0 = int64_t(blockIdx.x) * kWarps + w; t0 < s; t0 += kSl * stride) {
    int l[kSl], S[kSl];
    uint32_t wd[kSl][5];
    T v[kSl][4];
    int bw[kSl][4];
    bool live[kSl];
#pragma unroll
    for (int u = 0; u < kSl; ++u) {
      const int64_t t = t0 + u * stride;
      live[u] = t < s;
      if (k32 == 0) {  // one round trip fetches the metadata of the next 32 slices
        __syncwarp();
        const int64_t tl = t + lane * stride;
        if (tl < s) {
          const uint64_t c0l = __ldg(colptr + tl), q0l = __ldg(symptr + tl);
          metas[w][lane] = Meta{c0l, q0l, int(__ldg(colptr + tl + 1) - c0l), int(__ldg(symptr + tl + 1) - q0l)};
        }
        __syncwarp();
      }
      const Meta mt = metas[w][k32];
      k32 = (k32 + 1) & 31;
      l[u] = live[u] ? mt.l : 0;
      S[u] = live[u] ? mt.S : 0;
      const uint32_t* wb = words + 32 * mt.q0;
      const uint8_t* ba = bit_alloc + mt.c0;
#pragma unroll
      for (int j = 0; j < 4; ++j) bw[u][j] = j < l[u] ? int(__ldg(ba + j)) : 0;
#pragma unroll
      for (int q = 0; q < 4; ++q) wd[u][q] = q < S[u] ? __ldg(wb + place(lane, q, S[u], V)) : 0u;
      wd[u][4] = 0u;
      const int lfull = (l[u] / Chunk<T>::N) * Chunk<T>::N;
      if (l[u] > 0) load_group_vals<T, 4>(v[u], vals + 32 * mt.c0, 0, l[u], lfull, lane);
    }
    int cidx[kSl][4];
    bool ok[kSl][4];
#pragma unroll
    for (int u = 0; u < kSl; ++u) {
      int col = -1, o = 0;
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int b = bw[u][j];
        const int q = o >> 5;
        const uint32_t hi = q == 0 ? wd[u][0] : q == 1 ? wd[u][1] : q == 2 ? wd[u][2] : wd[u][3];
        const uint32_t lo = q == 0 ? wd[u][1] : q == 1 ? wd[u][2] : q == 2 ? wd[u][3] : wd[u][4];
        const uint32_t d = shr_clamp(__funnelshift_l(lo, hi, uint32_t(o & 31)), uint32_t(32 - b));
        col += int(d);
        cidx[u][j] = col;
        ok[u][j] = d != 0u;  // padding (and j >= l: b = 0) is skipped, Alg. 1 line 17
        o += b;
      }
    }
    T xv[kSl][4];
#pragma unroll
    for (int u = 0; u < kSl; ++u)
#pragma unroll
      for (int j = 0; j < 4; ++j)
        if (ok[u][j]) xv[u][j] = ldg_x(x + cidx[u][j]);
#pragma unroll
    for (int u = 0; u < kSl; ++u) {
      T sum = T(0);
#pragma unroll
      for (int j = 0; j < 4; ++j)
        if (ok[u][j]) sum = fma(v[u][j], xv[u][j], sum);
      const int64_t row = 32 * (t0 + u * stride) + lane;
      if (live[u] && row < m) store_y<false>(y, row, sum);
    }
  }
}

// ------------------------------------------------------------------ BRO-ELL, bulk-staged
// Same offset decode, but every byte of a slice (its values, its symbol
// stream in the paper's V = 1 multiplexing comp_str[q*h + tid], and
// its widths) is moved into shared memory by the TMA engine
// (cp.async.bulk, completion on an mbarrier) while the warp works on an
// earlier slice.  Each warp owns a ring of `nslot` slots (one slice each);
// with nslot - 1 slices in flight per warp the bytes in flight no longer
// depend on registers, and the register budget goes to x gathers instead
// (G per group).  V = 1 is what makes staging free: symbol row q of the
// slice is the 128-byte row [q][lane] of the window (conflict-free), so the
// slot IS the decode window (no copy), and each delta is
//     delta = funnelshift(w[q+1], w[q], o mod 32) >> (32 - b),  q = o / 32.
// Metadata of 32 upcoming slices is fetched per round trip (one per lane).
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n"
      "WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n}\n" :: "r"(smem_u32(bar)), "r"(parity) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar,
                                         uint64_t policy) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;"
      :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(policy) : "memory");
}
__device__ __forceinline__ uint64_t policy_evict_first() {
  uint64_t p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
constexpr int kBulkMaxSlots = 8;
constexpr int kBulkMetaRing = 64;
struct BulkMeta { uint64_t c0, q0; int l, S; };

// Bytes of one staged slice (host and device agree on this).
__host__ __device__ __forceinline__ uint32_t bulk_unit_bytes(uint64_t c0, int l, int S, int vsize) {
  const uint64_t ba_lo = c0 & ~uint64_t(15);
  const uint64_t ba_hi = (c0 + uint64_t(l) + 15) & ~uint64_t(15);
  return uint32_t(32 * l * vsize + 128 * S + (ba_hi - ba_lo));
}

// Dynamic shared memory layout of one block (per warp: slot barriers, meta
// ring, column metadata; then the warps' slot rings; 128 bytes of slack so
// the decode's w[q+1] read of the last symbol row stays inside).
template <int kWarps>
struct BulkSmem {
  static constexpr int kBarOff = 0;
  static constexpr int kMetaOff = kBarOff + kWarps * kBulkMaxSlots * 8;
  static constexpr int kColOff = kMetaOff + kWarps * kBulkMetaRing * int(sizeof(BulkMeta));
  static constexpr int kRingOff = ((kColOff + kWarps * 32 * 8) + 127) / 128 * 128;
  static __host__ __device__ int bytes(int nslot, int slot_bytes) {
    return kRingOff + kWarps * nslot * slot_bytes + 128;
  }
};

template <typename T, int kWarps, int G, int kMinBlocks>
__global__ void __launch_bounds__(kWarps * 32, kMinBlocks)
bro_ell_spmv_bulk(int64_t m, int64_t s, const uint32_t* __restrict__ words,
                  const uint8_t* __restrict__ bit_alloc, const uint64_t* __restrict__ colptr,
                  const uint64_t* __restrict__ symptr, const T* __restrict__ vals,
                  const T* __restrict__ x, const YOut<T> y, int nslot, int slot_bytes) {
  using L = BulkSmem<kWarps>;
  constexpr int VV = Chunk<T>::N;
  extern __shared__ __align__(128) uint8_t smem[];
  const int lane = threadIdx.x & 31;
  const int w = threadIdx.x / 32;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + L::kBarOff) + w * kBulkMaxSlots;
  BulkMeta* metas = reinterpret_cast<BulkMeta*>(smem + L::kMetaOff) + w * kBulkMetaRing;
  uint2* cm = reinterpret_cast<uint2*>(smem + L::kColOff) + w * 32;
  uint8_t* ring = smem + L::kRingOff + size_t(w) * nslot * slot_bytes;

  const int64_t stride = int64_t(gridDim.x) * kWarps;
  const int64_t t0 = int64_t(blockIdx.x) * kWarps + w;
  const int nk = t0 < s ? int((s - t0 + stride - 1) / stride) : 0;
  if (lane == 0) {
    for (int i = 0; i < nslot; ++i) mbar_init(bars + i, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
  const uint64_t pol = policy_evict_first();

  // metadata of units [kb, kb + 32) into the meta ring (all lanes); the
  // next batch's lines are prefetched into L2 half a batch ahead.
  auto load_metas = [&](int kb) {
    const int k = kb + lane;
    if (k < nk) {
      const int64_t t = t0 + k * stride;
      const uint64_t c0 = __ldg(colptr + t), q0 = __ldg(symptr + t);
      metas[k & (kBulkMetaRing - 1)] =
          BulkMeta{c0, q0, int(__ldg(colptr + t + 1) - c0), int(__ldg(symptr + t + 1) - q0)};
    }
    __syncwarp();
  };
  auto issue = [&](int k, int slot) {  // uniform across the warp
    if ((k & 31) == 0) load_metas(k);
    if ((k & 31) == 16) {
      const int kn = (k & ~31) + 32 + lane;
      if (kn < nk) {
        const int64_t t = t0 + kn * stride;
        prefetch_l2_line(colptr + t);
        prefetch_l2_line(symptr + t);
      }
    }
    if (lane == 0) {
      const BulkMeta mt = metas[k & (kBulkMetaRing - 1)];
      uint8_t* dst = ring + size_t(slot) * slot_bytes;
      const uint32_t vb = uint32_t(32 * mt.l * int(sizeof(T)));
      const uint32_t sb = uint32_t(128 * mt.S);
      const uint64_t ba_lo = mt.c0 & ~uint64_t(15);
      const uint32_t bb = uint32_t(((mt.c0 + uint64_t(mt.l) + 15) & ~uint64_t(15)) - ba_lo);
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      mbar_arrive_expect_tx(bars + slot, vb + sb + bb);
      if (vb) bulk_g2s(dst, vals + 32 * mt.c0, vb, bars + slot, pol);
      if (sb) bulk_g2s(dst + vb, words + 32 * mt.q0, sb, bars + slot, pol);
      if (bb) bulk_g2s(dst + vb + sb, bit_alloc + ba_lo, bb, bars + slot, pol);
    }
  };

  const int npre = min(nslot - 1, nk);
  for (int k = 0; k < npre; ++k) issue(k, k);
  int slot = 0, phase = 0;           // consumer position
  int islot = nslot - 1;             // slot of unit k + nslot - 1 (= slot of unit k - 1)
  for (int k = 0; k < nk; ++k) {
    if (k + nslot - 1 < nk) issue(k + nslot - 1, islot);  // into the slot freed by unit k - 1
    islot = slot;
    mbar_wait(bars + slot, uint32_t(phase));
    const BulkMeta mt = metas[k & (kBulkMetaRing - 1)];
    const int l = mt.l;
    const uint8_t* base = ring + size_t(slot) * slot_bytes;
    const T* sv = reinterpret_cast<const T*>(base);
    const char* sw_lane = reinterpret_cast<const char*>(base + 32 * l * sizeof(T)) + 4 * lane;
    const uint8_t* sb = base + 32 * l * sizeof(T) + 128 * mt.S + (mt.c0 & 15);
    const int lfull = (l / VV) * VV;
    const int tw = l - lfull;
    T sum = T(0);
    int col = -1;
    int obase = 0;
    for (int jb = 0; jb < l; jb += 32) {
      const int nb = min(32, l - jb);
      const int b = lane < nb ? int(sb[jb + lane]) : 0;
      int incl = b;
#pragma unroll
      for (int off = 1; off < 32; off <<= 1) {
        const int o = __shfl_up_sync(0xffffffffu, incl, off);
        if (lane >= off) incl += o;
      }
      const int tot = __shfl_sync(0xffffffffu, incl, 31);
      {
        const int rel = b ? obase + incl - b : 0;  // bit offset of column jb+lane in every row stream
        cm[lane] = make_uint2(uint32_t(rel >> 5) * 128u, uint32_t(rel & 31) | ((32u - uint32_t(b)) << 8));
      }
      __syncwarp();
      for (int g = 0; g < nb; g += G) {
        int cidx[G];
        bool ok[G];
#pragma unroll
        for (int k2 = 0; k2 < G; ++k2) {
          const uint2 mm = cm[g + k2];  // broadcast
          const uint32_t* wp = reinterpret_cast<const uint32_t*>(sw_lane + mm.x);
          const uint32_t d = shr_clamp(__funnelshift_l(wp[32], wp[0], mm.y), mm.y >> 8);
          col += int(d);
          cidx[k2] = col;
          ok[k2] = d != 0u;
        }
        T xv[G];
#pragma unroll
        for (int k2 = 0; k2 < G; ++k2) xv[k2] = ok[k2] ? ldg_x(x + cidx[k2]) : T(0);
        const int j0 = jb + g;
#pragma unroll
        for (int u = 0; u < G / VV; ++u) {
          const int jj = j0 + u * VV;
          T v[VV];
          if (jj + VV <= lfull) {
            if constexpr (VV == 2) {
              const double2 c2 = *reinterpret_cast<const double2*>(sv + 32 * jj + lane * VV);
              v[0] = c2.x; v[1] = c2.y;
            } else {
              const float4 c4 = *reinterpret_cast<const float4*>(sv + 32 * jj + lane * VV);
              v[0] = c4.x; v[1] = c4.y; v[2] = c4.z; v[3] = c4.w;
            }
          } else {
#pragma unroll
            for (int q = 0; q < VV; ++q)
              v[q] = (jj + q < l) ? sv[32 * lfull + lane * tw + (jj + q - lfull)] : T(0);
          }
#pragma unroll
          for (int q = 0; q < VV; ++q) sum = fma(v[q], xv[u * VV + q], sum);  // padding: v = 0, x = 0
        }
      }
      obase += tot;
      __syncwarp();
    }
    const int64_t row = 32 * (t0 + int64_t(k) * stride) + lane;
    if (row < m) store_y<false>(y, row, sum);
    if (++slot == nslot) { slot = 0; phase ^= 1; }
  }
}

// Decode-only variant: decoded column (or -1) per slot in V=1 slot order.
template <int V>
__global__ void bro_ell_decode(int64_t s, const uint32_t* __restrict__ words,
                               const uint8_t* __restrict__ bit_alloc,
                               const uint64_t* __restrict__ colptr,
                               const uint64_t* __restrict__ symptr, int32_t* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const int64_t t = int64_t(blockIdx.x) * (blockDim.x / 32) + (threadIdx.x >> 5);
  if (t >= s) return;
  const uint64_t c0 = colptr[t];
  const int l = int(colptr[t + 1] - c0);
  const uint64_t q0 = symptr[t];
  LaneStream<V> ls;
  ls.init(words + 32 * q0, int(symptr[t + 1] - q0), lane);
  int col = -1;
  for (int j = 0; j < l; ++j) {
    const uint32_t d = ls.get(bit_alloc[c0 + j], lane);
    col += int(d);
    out[32 * c0 + 32 * j + lane] = d ? col : -1;
  }
}

// ------------------------------------------------------------------ plain ELLPACK
template <typename T, int kThreads, bool kMulti = false>
__global__ void __launch_bounds__(kThreads)
ell_spmv(int64_t m, int64_t K, int64_t pitch, const int32_t* __restrict__ col,
         const T* __restrict__ vals, const T* __restrict__ x, const YOut<T> y) {
  constexpr int G = 8;
  const int64_t row = int64_t(blockIdx.x) * kThreads + threadIdx.x;
  if (row >= m) return;
  T sum = T(0);
  int64_t j = 0;
  for (; j + G <= K; j += G) {
    int c[G];
    T v[G];
#pragma unroll
    for (int k = 0; k < G; ++k) {
      c[k] = ld_stream_s32(col + (j + k) * pitch + row);
      v[k] = ld_stream(vals + (j + k) * pitch + row);
    }
    T xv[G];
#pragma unroll
    for (int k = 0; k < G; ++k) xv[k] = c[k] >= 0 ? ldg_x(x + c[k]) : T(0);
#pragma unroll
    for (int k = 0; k < G; ++k) sum = fma(v[k], xv[k], sum);
  }
  for (; j < K; ++j) {
    const int c = ld_stream_s32(col + j * pitch + row);
    const T v = ld_stream(vals + j * pitch + row);
    if (c >= 0) sum = fma(v, ldg_x(x + c), sum);
  }
  store_y<kMulti>(y, row, sum);
}

__global__ void ell_decode(int64_t m, int64_t K, int64_t pitch, const int32_t* __restrict__ col,
                           int32_t* __restrict__ out) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= K * pitch) return;
  out[i] = col[i];
  (void)m;
}

// ------------------------------------------------------------------ (BRO-)COO
// One warp per interval of 32*T entries.  BRO row deltas are laid
// out per (step t, lane) (element (t, lane) = entry e0 + 32t + lane), so each
// lane first decodes its rows for 8 steps into a per-warp shared buffer.  The
// multiply is then done TRANSPOSED: lane l owns the 8 consecutive entries
// 8l .. 8l+7 of the 256-entry batch (16-byte loads of col / vals, which are in
// plain COO order), reduces them sequentially, and one warp-level segmented
// scan over the lanes' trailing partials (the "parallel scan primitive" of
// P:L343) links segments that cross lanes.  Complete segments of rows other
// than the interval's first row are added into y directly (each such row
// lives in exactly one interval); the first and last rows' partials go to
// carry arrays for the deterministic fix-up kernel.
template <typename T>
struct Vec8 {  // 8 consecutive values of one lane, loaded as 16-byte chunks
  T v[8];
  __device__ __forceinline__ void load(const T* p) {
#pragma unroll
    for (int u = 0; u < 8 / Chunk<T>::N; ++u) {
      Chunk<T> c;
      c.load(p + u * Chunk<T>::N);
#pragma unroll
      for (int q = 0; q < Chunk<T>::N; ++q) v[u * Chunk<T>::N + q] = c.v[q];
    }
  }
};

__device__ __forceinline__ void load8_s32(int* d, const int32_t* p) {
  const uint4 a = ld_stream_u4(reinterpret_cast<const uint32_t*>(p));
  const uint4 b = ld_stream_u4(reinterpret_cast<const uint32_t*>(p) + 4);
  d[0] = int(a.x); d[1] = int(a.y); d[2] = int(a.z); d[3] = int(a.w);
  d[4] = int(b.x); d[5] = int(b.y); d[6] = int(b.z); d[7] = int(b.w);
}

// delta of step t in a lane stream of b-bit fields staged as [row][lane]
// (wl points at the lane's word of row 0); 0 when b = 0 (empty stream).
__device__ __forceinline__ int coo_delta(const uint32_t* wl, int t, int b) {
  const int o = t * b;
  const uint32_t* p = wl + 32 * (o >> 5);
  return int(shr_clamp(__funnelshift_l(p[32], p[0], uint32_t(o & 31)), uint32_t(32 - b)));
}

// One transposed batch of 8*32 entries (lane owns entries 8*lane .. 8*lane+7,
// rows r[] non-decreasing across the batch): gathers x, reduces each lane's
// entries sequentially and links segments across lanes with one warp
// segmented scan; complete segments go to emit(row, partial), the batch's
// trailing partial is carried (crow, carry) into the next batch.
template <typename T, typename Emit>
__device__ __forceinline__ void coo_segments(const int* r, const int* c, const T* v, const T* __restrict__ x,
                                             int lane, int& crow, T& carry, Emit&& emit) {
  constexpr int TB = 8;
  T xv[TB];
#pragma unroll
  for (int k = 0; k < TB; ++k) xv[k] = c[k] >= 0 ? ldg_x(x + c[k]) : T(0);
  // sequential pass over the lane's 8 entries
  const int f = r[0];
  T A = T(0), cur = T(0);
  bool one = true;
  int cr = f;
#pragma unroll
  for (int k = 0; k < TB; ++k) {
    const T p = v[k] * xv[k];
    if (r[k] != cr) {           // the segment of row cr ends inside this lane
      if (one) { A = cur; one = false; }
      else emit(cr, cur);       // interior segment: complete, row unique to this lane
      cr = r[k];
      cur = p;
    } else {
      cur += p;
    }
  }
  if (one) A = cur;
  const int L = cr;             // trailing segment: row L, partial cur
  // carry-in from earlier lanes (or earlier batches for lane 0)
  const int Lprev = __shfl_up_sync(0xffffffffu, L, 1);
  const bool link = lane == 0 ? (crow == f) : (Lprev == f);
  // C_out(l) = B_l + [one_l && link_l] * C_out(l-1): segmented scan
  T co = cur;
  bool open = one && link;      // this lane's partial continues an earlier one
  if (lane == 0 && open) co += carry;
#pragma unroll
  for (int off = 1; off < 32; off <<= 1) {
    const T o = __shfl_up_sync(0xffffffffu, co, off);
    const int op = __shfl_up_sync(0xffffffffu, int(open), off);
    if (lane >= off && open) co += o;
    if (lane >= off) open = open && op;
  }
  // C_in = C_out(l-1) if linked; lane 0 takes the batch carry
  T cin = __shfl_up_sync(0xffffffffu, co, 1);
  if (lane == 0) cin = carry;
  if (!link) cin = T(0);
  if (lane == 0 && !link && crow != f) {
    // the carried row ended before this batch
    emit(crow, carry);
  }
  if (!one) emit(f, A + cin);   // first segment complete inside this lane
  const int fnext = __shfl_down_sync(0xffffffffu, f, 1);
  if (lane < 31 && fnext != L) emit(L, co);  // trailing segment complete at this lane
  carry = __shfl_sync(0xffffffffu, co, 31);
  crow = __shfl_sync(0xffffffffu, L, 31);
}

template <typename T, int V, bool kBro, int kThreads, int kMinBlocks = 0>
__global__ void __launch_bounds__(kThreads, kMinBlocks)
coo_spmv(int64_t nnz, int64_t nI, int T_steps, int upi_log2, const uint32_t* __restrict__ words,
         const uint32_t* __restrict__ base_row, const uint8_t* __restrict__ width,
         const uint64_t* __restrict__ symptr, const int32_t* __restrict__ rows,
         const int32_t* __restrict__ col, const T* __restrict__ vals, const T* __restrict__ x,
         T* __restrict__ y, T* __restrict__ carry_first, T* __restrict__ carry_last,
         int32_t* __restrict__ first_row, int32_t* __restrict__ last_row, int l2_prefetch) {
  constexpr int TB = 8;
  __shared__ __align__(16) int32_t rowbuf[kThreads / 32][TB * 32];
  __shared__ uint32_t cwin[kThreads / 32][kBro ? 33 * 32 : 1];  // lane word rows (+ zero guard row)
  const int lane = threadIdx.x & 31;
  const int w = threadIdx.x >> 5;
  // work unit = steps [ts, ts + T_steps / upi) of interval i (upi = 2^upi_log2
  // units per interval; shifts, not 64-bit divisions)
  const int64_t u = int64_t(blockIdx.x) * (kThreads / 32) + w;
  const int64_t i = u >> upi_log2;
  if (i >= nI) return;
  const int steps = T_steps >> upi_log2;
  const int ts = int(u & ((int64_t(1) << upi_log2) - 1)) * steps;
  int32_t* rb = rowbuf[w];
  const int64_t e0 = i * 32 * T_steps;
  // optional L2 prefetch (TMA engine) of the unit's batches after the first
  // one (BRO_COO_L2PF=1): measured slower, C4 BRO-HYB f64 115.2 vs 111.2 us
  // (profiles/r01/s3/coo_l2pf.txt), so off by default
  if (l2_prefetch && lane == 0) {
    const int64_t p0 = e0 + 32 * (ts + TB);
    const int64_t p1 = min(e0 + 32 * int64_t(ts + steps), nnz) & ~int64_t(3);
    if (p1 > p0) {
      prefetch_l2(col + p0, uint32_t((p1 - p0) * 4));
      prefetch_l2(vals + p0, uint32_t((p1 - p0) * sizeof(T)));
      if constexpr (!kBro) prefetch_l2(rows + p0, uint32_t((p1 - p0) * 4));
    }
  }
  int row = (int)base_row[i];
  const int b = kBro ? int(width[i]) : 0;
  const uint32_t* wn = cwin[w] + lane;
  // row of the unit's first entry (element (ts, 0))
  int first = 0;
  if constexpr (!kBro) first = rows[min(e0 + 32 * ts, nnz - 1)];
  bool first_pending = kBro;  // kBro: lane 0's row at step ts is known only after the first decode
  T carry = T(0);   // partial of row crow carried from earlier batches (not yet written)
  int crow = first;
  // A complete segment of row r.  Every row other than the unit's first and
  // last rows is complete in exactly one place of the whole launch, so it
  // receives exactly one addition: a fire-and-forget RED (atomicAdd with the
  // result unused) is as deterministic as y[r] += v but does not serialize
  // the warp on a load -> store chain per segment.
  auto emit = [&](int r, T v) {
    if (r == first) carry_first[u] = v;
    else atomicAdd(y + r, v);
  };
  for (int t0 = ts; t0 < ts + steps; t0 += TB) {
    const int64_t eb = e0 + 32 * t0;            // first entry of the batch
    const int64_t el = eb + TB * lane;          // this lane's first entry (transposed)
    int r[TB], c[TB];
    T v[TB];
    // col / vals (and plain rows) of the batch first: they do not depend on
    // the row decode, so their round trip overlaps it
    if (el + TB <= nnz) {
      if constexpr (!kBro) load8_s32(r, rows + el);
      load8_s32(c, col + el);
      Vec8<T> vv;
      vv.load(vals + el);
#pragma unroll
      for (int k = 0; k < TB; ++k) v[k] = vv.v[k];
    } else {  // tail of the last interval: entries past nnz repeat the last row with value 0
#pragma unroll
      for (int k = 0; k < TB; ++k) {
        const bool ok = el + k < nnz;
        if constexpr (!kBro) r[k] = ld_stream_s32(rows + (ok ? el + k : nnz - 1));
        c[k] = ok ? ld_stream_s32(col + el + k) : -1;
        v[k] = ok ? ld_stream(vals + el + k) : T(0);
      }
    }
    if constexpr (kBro) {
      if (t0 == ts) {
        // One width per interval, so the bit offset of step t is t*b
        // in every lane stream: stage the words the unit needs (rows
        // [0, q_hi]) in a per-warp [row][lane] window and extract each delta
        // branch-free: delta_t = funnelshift(w[q+1], w[q], o mod 32) >> (32 - b), o = t*b.
        const uint64_t q0 = symptr[i];
        const int S = int(symptr[i + 1] - q0);
        const int nrows = b ? min(S, (((ts + steps) * b - 1) >> 5) + 1) : 0;
        stage_symbols<V>(cwin[w], words + 32 * q0, S, 0, nrows, lane);
        __syncwarp();
        for (int t = 0; t < ts; ++t) row += coo_delta(wn, t, b);  // rows of the steps before the unit
      }
#pragma unroll
      for (int k = 0; k < TB; ++k) {  // decode rows of steps t0..t0+7 for (t, lane)
        row += coo_delta(wn, t0 + k, b);
        rb[k * 32 + lane] = row;
      }
      __syncwarp();
      const int4 ra = *reinterpret_cast<const int4*>(rb + TB * lane);
      const int4 rc = *reinterpret_cast<const int4*>(rb + TB * lane + 4);
      r[0] = ra.x; r[1] = ra.y; r[2] = ra.z; r[3] = ra.w;
      r[4] = rc.x; r[5] = rc.y; r[6] = rc.z; r[7] = rc.w;
      if (first_pending) {
        first = rb[0];
        crow = first;
        first_pending = false;
      }
      __syncwarp();
    }
    coo_segments<T>(r, c, v, x, lane, crow, carry, emit);
  }
  if (lane == 0) {
    first_row[u] = first;
    last_row[u] = crow;
    if (crow == first) {
      carry_first[u] = carry;
      carry_last[u] = T(0);
    } else {
      carry_last[u] = carry;
    }
  }
}

// ------------------------------------------------------------------ (BRO-)COO, persistent pipeline
// Same entry order, decode and segment logic as coo_spmv, but a persistent
// warp walks a CONTIGUOUS range of whole intervals batch by batch (8 steps =
// 256 entries) with a one-batch software pipeline: while batch k is decoded,
// gathered and reduced, batch k+1's col / vals (rows for plain COO) are
// already in flight into registers and its row-stream words are copied into
// the other half of a double-buffered per-warp window by cp.async (no
// registers).  A batch at step t0 of an interval with width b needs word rows
// (t0*b)>>5 .. ((t0+8)*b-1)>>5 only (<= 9 rows, S = b words per lane for
// T = 32), so staging is per batch and never skips.  Interval metadata
// (base row, width, first word) of the warp's next 32 intervals is fetched
// lane-parallel into shared memory.  One work unit (carry pair) per warp:
// rows continue across the warp's intervals, so the fix-up sees nW units.

constexpr int kCooPipeRows = 10;  // window rows per batch buffer (<= 9 used)

template <typename T, int V, bool kBro, int kWarps, int kMinBlocks>
__global__ void __launch_bounds__(kWarps * 32, kMinBlocks)
coo_spmv_pipe(int64_t nnz, int64_t nI, const uint32_t* __restrict__ words,
              const uint32_t* __restrict__ base_row, const uint8_t* __restrict__ width,
              const uint64_t* __restrict__ symptr, const int32_t* __restrict__ rows,
              const int32_t* __restrict__ col, const T* __restrict__ vals, const T* __restrict__ x,
              T* __restrict__ y, T* __restrict__ carry_first, T* __restrict__ carry_last,
              int32_t* __restrict__ first_row, int32_t* __restrict__ last_row) {
  constexpr int TB = 8;          // steps per batch
  constexpr int BPI = 32 / TB;   // batches per interval (T = 32)
  struct IMeta { uint64_t q0; uint32_t base; int b; };
  __shared__ __align__(16) int32_t rowbuf[kWarps][TB * 32];
  __shared__ uint32_t cwin[kWarps][kBro ? 2 * kCooPipeRows * 32 : 1];
  __shared__ IMeta metas[kWarps][kBro ? 32 : 1];
  const int lane = threadIdx.x & 31;
  const int w = threadIdx.x >> 5;
  const int64_t nW = int64_t(gridDim.x) * kWarps;
  const int64_t u = int64_t(blockIdx.x) * kWarps + w;  // this warp = one work unit
  const int64_t iA = u * nI / nW, iB = (u + 1) * nI / nW;
  const int64_t nbat = (iB - iA) * BPI;
  int32_t* rb = rowbuf[w];
  if (nbat == 0) {  // (launcher keeps nW <= nI; kept for safety) an empty unit
    if (lane == 0) { first_row[u] = -1; last_row[u] = -1; carry_first[u] = T(0); carry_last[u] = T(0); }
    return;
  }
  // metadata of intervals [i0, i0 + 32) of this warp into shared memory
  auto fetch_meta = [&](int64_t i0) {
    __syncwarp();
    const int64_t il = i0 + lane;
    if (kBro && il < iB) metas[w][kBro ? lane : 0] = IMeta{symptr[il], base_row[il], int(width[il])};
    __syncwarp();
  };
  // cp.async the word rows of batch (interval i, step t0) into buffer buf
  auto stage = [&](int64_t i, int t0, int buf) {
    if constexpr (kBro) {
      const IMeta mt = metas[w][(i - iA) & 31];
      const int b = mt.b;
      if (b == 0) return;
      const int S = b;  // T = 32 steps of b bits = b words per lane
      const int qa = (t0 * b) >> 5, qb = ((t0 + TB) * b - 1) >> 5;
      const uint32_t* wb = words + 32 * mt.q0;
      uint32_t* dst = cwin[w] + buf * kCooPipeRows * 32 + lane;
      for (int q = qa; q <= qb; ++q) cp_async4(dst + 32 * (q - qa), wb + place(lane, q, S, V));
    }
  };
  auto load_batch = [&](int64_t i, int t0, int* r, int* c, T* v) {
    const int64_t el = i * 1024 + 32 * t0 + TB * lane;  // transposed: lane's 8 consecutive entries
    if (el + TB <= nnz) {
      if constexpr (!kBro) load8_s32(r, rows + el);
      load8_s32(c, col + el);
      Vec8<T> vv;
      vv.load(vals + el);
#pragma unroll
      for (int k = 0; k < TB; ++k) v[k] = vv.v[k];
    } else {  // tail of the last interval: entries past nnz repeat the last row with value 0
#pragma unroll
      for (int k = 0; k < TB; ++k) {
        const bool ok = el + k < nnz;
        if constexpr (!kBro) r[k] = ld_stream_s32(rows + (ok ? el + k : nnz - 1));
        c[k] = ok ? ld_stream_s32(col + el + k) : -1;
        v[k] = ok ? ld_stream(vals + el + k) : T(0);
      }
    }
  };

  if constexpr (kBro) fetch_meta(iA);
  int r[TB], c[TB];
  T v[TB];
  stage(iA, 0, 0);
  cp_async_commit();
  load_batch(iA, 0, r, c, v);
  int row = 0, b = 0;
  int first = 0;
  bool first_pending = true;
  T carry = T(0);
  int crow = 0;
  auto emit = [&](int rr, T val) {
    if (rr == first) carry_first[u] = val;
    else atomicAdd(y + rr, val);
  };
  for (int64_t k = 0; k < nbat; ++k) {
    const int64_t i = iA + k / BPI;
    const int t0 = int(k % BPI) * TB;
    if constexpr (kBro) {
      if (t0 == 0) {
        const IMeta mt = metas[w][(i - iA) & 31];
        row = int(mt.base);
        b = mt.b;
      }
    }
    // issue batch k+1: words (cp.async) and col / vals (registers)
    int rn[TB], cn[TB];
    T vn[TB];
    const bool has_next = k + 1 < nbat;
    if (has_next) {
      const int64_t i1 = iA + (k + 1) / BPI;
      const int t1 = int((k + 1) % BPI) * TB;
      if constexpr (kBro) {
        if (t1 == 0 && ((i1 - iA) & 31) == 0) fetch_meta(i1);  // every 32 intervals (current one in registers)
      }
      stage(i1, t1, int((k + 1) & 1));
      cp_async_commit();
      load_batch(i1, t1, rn, cn, vn);
      cp_async_wait<1>();
    } else {
      cp_async_wait<0>();
    }
    __syncwarp();
    if constexpr (kBro) {
      const uint32_t* wl = cwin[w] + int(k & 1) * kCooPipeRows * 32 + lane;
      const int obase = (t0 * b) & ~31;  // bit offset of the window's first row
#pragma unroll
      for (int s = 0; s < TB; ++s) {
        const int o = (t0 + s) * b - obase;
        const uint32_t* pw = wl + 32 * (o >> 5);
        row += int(shr_clamp(__funnelshift_l(pw[32], pw[0], uint32_t(o & 31)), uint32_t(32 - b)));
        rb[s * 32 + lane] = row;
      }
      __syncwarp();
      const int4 ra = *reinterpret_cast<const int4*>(rb + TB * lane);
      const int4 rc = *reinterpret_cast<const int4*>(rb + TB * lane + 4);
      r[0] = ra.x; r[1] = ra.y; r[2] = ra.z; r[3] = ra.w;
      r[4] = rc.x; r[5] = rc.y; r[6] = rc.z; r[7] = rc.w;
      __syncwarp();
    }
    if (first_pending) {
      first = __shfl_sync(0xffffffffu, r[0], 0);
      crow = first;
      first_pending = false;
    }
    coo_segments<T>(r, c, v, x, lane, crow, carry, emit);
    if (has_next) {
#pragma unroll
      for (int q = 0; q < TB; ++q) {
        c[q] = cn[q];
        v[q] = vn[q];
        if constexpr (!kBro) r[q] = rn[q];
      }
    }
  }
  if (lane == 0) {
    first_row[u] = first;
    last_row[u] = crow;
    if (crow == first) {
      carry_first[u] = carry;
      carry_last[u] = T(0);
    } else {
      carry_last[u] = carry;
    }
  }
}

// Exchange of a finished y for formats whose last kernel is not an ELL
// kernel (COO / HYB: the COO part and the fix-up add into y after the ELL
// part stored it, so only the final values may leave the GPU): copy the
// local y (o.p[0]) into the other destinations o.p[1..n-1], or once through
// the multicast address; m * sizeof(T) bytes per peer.
template <typename T>
__global__ void replicate_y(int64_t m, const YOut<T> o) {
  const T* __restrict__ src = o.p[0];
  const int64_t stride = int64_t(gridDim.x) * blockDim.x;
  for (int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x; i < m; i += stride) {
    const T v = src[i];
    if (o.mc != nullptr) {
      multimem_st(o.mc + i, v);
    } else {
#pragma unroll
      for (int k = 1; k < kMaxDst; ++k)
        if (k < o.n) o.p[k][i] = v;
    }
  }
}

// Deterministic application of the units' carries (one thread per unit,
// fixed summation order = unit order).  first[u] / last[u] = rows of the
// unit's first and last entries; cf = partial of the first row (the whole
// unit if first == last), cl = partial of the last row.
// acc += cf[j] for the units j = i+1, i+2, ... that continue row R (first[j]
// == R), stopping after the first of them that ends on another row.  Units
// are read 8 at a time, so a row spanning up to 9 units costs one round trip
// instead of one per unit; the additions stay in unit order.
template <typename T>
__device__ __forceinline__ T chain_sum(int64_t i, int64_t nU, int R, T acc, const int32_t* __restrict__ first,
                                       const int32_t* __restrict__ last_row, const T* __restrict__ cf) {
  constexpr int B = 8;
  for (int64_t j0 = i + 1; j0 < nU; j0 += B) {
    int fj[B], lj[B];
    T cj[B];
#pragma unroll
    for (int k = 0; k < B; ++k) {
      const bool in = j0 + k < nU;
      fj[k] = in ? first[j0 + k] : -1;
      lj[k] = in ? last_row[j0 + k] : -1;
      cj[k] = in ? cf[j0 + k] : T(0);
    }
    bool done = false;
#pragma unroll
    for (int k = 0; k < B; ++k) {
      if (!done) {
        if (fj[k] != R) {
          done = true;
        } else {
          acc += cj[k];
          done = lj[k] != R;
        }
      }
    }
    if (done) break;
  }
  return acc;
}

template <typename T>
__global__ void coo_fixup(int64_t nU, const int32_t* __restrict__ first,
                          const int32_t* __restrict__ last_row, const T* __restrict__ cf,
                          const T* __restrict__ cl, T* __restrict__ y) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= nU) return;
  const int F = first[i];
  const int L = last_row[i];
  if (L != F)  // unit i is the first one holding row L
    y[L] += chain_sum<T>(i, nU, L, cl[i], first, last_row, cf);
  if (i == 0 || last_row[i - 1] != F)  // unit i is the first one holding row F
    y[F] += L == F ? chain_sum<T>(i, nU, F, cf[i], first, last_row, cf) : cf[i];
}

template <int V>
__global__ void bro_coo_decode(int64_t nnz, int64_t nI, int T_steps, const uint32_t* __restrict__ words,
                               const uint32_t* __restrict__ base_row, const uint8_t* __restrict__ width,
                               const uint64_t* __restrict__ symptr, int32_t* __restrict__ out) {
  const int lane = threadIdx.x & 31;
  const int64_t i = int64_t(blockIdx.x) * (blockDim.x / 32) + (threadIdx.x >> 5);
  if (i >= nI) return;
  const int b = width[i];
  LaneStream<V> ls;
  ls.init(words + 32 * symptr[i], int(symptr[i + 1] - symptr[i]), lane);
  int row = (int)base_row[i];
  for (int t = 0; t < T_steps; ++t) {
    if (b) row += (int)ls.get(b, lane);
    const int64_t e = i * 32 * T_steps + 32 * t + lane;
    if (e < nnz) out[e] = row;
  }
}

}  // namespace dev
}  // namespace bro
