// sm_100a SpMV kernels for BRO-ELL, BRO-COO (+ carry fix-up) and the
// uncompressed ELLPACK / COO baselines.
//
// Mapping (B200-first; the paper's Fermi/Kepler mapping of one 256-thread
// block per slice, is prior art):
//   * BRO-ELL (bro_ell_od): one WARP per slice of h = 32*R rows, R rows per
//     lane (R = 1: h = 32; R = 2: h = 64, rows lane and lane + 32),
//     persistent warps.  Widths are shared by the slice's rows, so
//     every column's bit offset is warp-uniform: a SHFL scan of the widths
//     gives the offsets of a 32-column block, the block's symbols are staged
//     in a per-warp shared window [q][lane][R], and each delta is a
//     branch-free funnel-shift extraction fused with the x gather and the FMA
//     (the load-decode-compute cycle of Alg. 1 without its per-column branch,
//     P:L120-122).  R = 2 shares the widths, offsets and column records of a
//     column between two rows and fetches both rows' symbol words with one
//     64-bit shared load.
//   * bro_ell_tiny: slices of <= 4 columns keep their <= 4 symbols per row in
//     registers (no window, no scan).
//   * BRO-COO (coo_spmv<kBro=true>): one warp per interval of 32*T entries
//     (P:L140), lane l owning T consecutive entries (reading R13): the lane
//     decodes its deltas from a staged window, one warp scan of the lane
//     totals gives every lane its start row, the lane reduces its entries
//     sequentially and ONE warp segmented scan per interval links segments
//     that cross lanes (the "parallel scan primitive" of P:L343); a
//     deterministic fix-up kernel adds the partials of rows crossing
//     intervals (the "extra kernel invocation for data reduction").
//   * Uncompressed baselines: ell_spmv (thread per row, column-major
//     ELLPACK) and coo_spmv<kBro=false> (same traversal, explicit rows).
//   * Every kernel takes a Mode: kSpmv (y = A.x), kScatter (y also stored
//     into peer replicas, the fused exchange of dist.py) or kDecode (the SAME
//     decode path, storing the decoded column / row index instead of the
//     FMA: bro_decode_indices checks the hot path bit-exactly).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace bro {
namespace dev {

constexpr int kWarp = 32;
enum Mode { kSpmv = 0, kScatter = 1, kDecode = 2 };

// ------------------------------------------------------------------ loads
// Streamed arrays (values, symbols, COO col/row) are read with
// ld.global.nc.L1::no_allocate.L2::256B (no L1 allocation for data used once,
// 256-byte L2 fetches; profiles/r01/s4/ab_l2_256B.txt).  The asm is
// non-volatile: the compiler may issue a guarded load speculatively and
// select the result, which is what makes the tail code branch-free.  The
// library therefore pads every device array by kStreamPad zeroed bytes, so
// the farthest speculated address stays inside the allocation
// (compute-sanitizer memcheck clean).
constexpr int kStreamPad = 16384;

__device__ __forceinline__ uint4 ld_stream_u4(const void* p) {
  uint4 r;
  asm("ld.global.nc.L1::no_allocate.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];"
      : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ uint32_t ld_stream_u32(const uint32_t* p) {
  uint32_t r;
  asm("ld.global.nc.L1::no_allocate.L2::256B.u32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}
// never speculated: a guarded load stays a predicated load (symbol staging,
// whose guards cut off the words of the NEXT slice)
__device__ __forceinline__ uint32_t ld_stream_u32_g(const uint32_t* p) {
  uint32_t r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::256B.u32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ uint4 ld_stream_u4_g(const void* p) {
  uint4 r;
  asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ int32_t ld_stream_s32(const int32_t* p) {
  int32_t r;
  asm("ld.global.nc.L1::no_allocate.L2::256B.s32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ double ld_stream(const double* p) {
  double r;
  asm("ld.global.nc.L1::no_allocate.L2::256B.f64 %0, [%1];" : "=d"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ float ld_stream(const float* p) {
  float r;
  asm("ld.global.nc.L1::no_allocate.L2::256B.f32 %0, [%1];" : "=f"(r) : "l"(p));
  return r;
}

// 16-byte value chunk: 2 doubles or 4 floats
template <typename T> struct Chunk;
template <> struct Chunk<double> {
  double v[2];
  static constexpr int N = 2;
  __device__ __forceinline__ void load(const double* p) {
    asm("ld.global.nc.L1::no_allocate.L2::256B.v2.f64 {%0,%1}, [%2];" : "=d"(v[0]), "=d"(v[1]) : "l"(p));
  }
};
template <> struct Chunk<float> {
  float v[4];
  static constexpr int N = 4;
  __device__ __forceinline__ void load(const float* p) {
    asm("ld.global.nc.L1::no_allocate.L2::256B.v4.f32 {%0,%1,%2,%3}, [%4];"
        : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]) : "l"(p));
  }
};

template <typename T>
__device__ __forceinline__ T ldg_x(const T* p) { return __ldg(p); }

// A kernel-parameter pointer the compiler must keep in a register: without
// this it re-loads the x base from the constant bank (LDC) before every
// predicated gather of the BRO-ELL loop — one extra instruction per slot.
// (z is a runtime zero: m >> 62 of a row count; an expression of two
// parameters is not worth re-materialising, so the sum stays in a register)
template <typename T>
__device__ __forceinline__ const T* in_reg(const T* p, int64_t z) {
  const T* r;
  asm("add.s64 %0, %1, %2;" : "=l"(r) : "l"(p), "l"(z));
  return r;
}

// shl / shr with the PTX clamp (shift >= 32 gives 0)
__device__ __forceinline__ uint32_t shl_clamp(uint32_t v, uint32_t s) {
  uint32_t r;
  asm("shl.b32 %0, %1, %2;" : "=r"(r) : "r"(v), "r"(s));
  return r;
}
__device__ __forceinline__ uint32_t shr_clamp(uint32_t v, uint32_t s) {
  uint32_t r;
  asm("shr.b32 %0, %1, %2;" : "=r"(r) : "r"(v), "r"(s));
  return r;
}

// item q of row r in a block of H rows x S items in chunks of V (the
// multiplexing of P:L116, reading R11; V = 1 is comp_str_i[q*h + tid])
__device__ __forceinline__ int64_t place(int64_t r, int64_t q, int64_t S, int64_t V, int64_t H) {
  const int64_t F = S / V;
  const int64_t c = q / V;
  if (c < F) return H * V * c + r * V + (q - c * V);
  return H * V * F + r * (S - V * F) + (q - V * F);
}

// ------------------------------------------------------------------ y destinations
// Where a kernel stores y[row].  kSpmv: p[0] only.  kScatter (the fused
// exchange of the row-block iteration): the same value
// also goes into the x replica of every peer GPU (P2P stores through
// NVLink, p[i] = peer-mapped symmetric-memory pointers), or once through an
// NVLS multicast address (mc).  Indices are static (unrolled) so the table
// stays in the kernel-parameter bank.
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

template <int kMode, typename T>
__device__ __forceinline__ void store_y(const YOut<T>& o, int64_t row, T v) {
  if constexpr (kMode != kScatter) {
    o.p[0][row] = v;
  } else {
    if (o.mc != nullptr) {
      multimem_st(o.mc + row, v);
      return;
    }
    o.p[0][row] = v;
#pragma unroll
    for (int i = 1; i < kMaxDst; ++i)
      if (i < o.n) o.p[i][row] = v;
  }
}

// ------------------------------------------------------------------ parameter blocks
template <typename T>
struct EllDev {           // a BRO-ELL part (or a range of its slices)
  int64_t m, s;           // rows (y stores stop at m), slices
  const uint32_t* words;
  const uint8_t* bit_alloc;
  const uint64_t* colptr;
  const uint64_t* symptr;
  const T* vals;
  const T* x;
  const int2* xwin;       // x-staged instances: per block, {first column, columns} of its x window
  const uint8_t* vcodes;  // value-indexed handles (reading R28): codes in the slot layout, 4-byte chunks
  const T* vdict;         // ... and the table of distinct values they index
  uint32_t vpad;          // ... and the code of padding slots (a finite value, reading R28)
};

// ------------------------------------------------------------------ TMA bulk copy + mbarrier
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(count) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n"
      "WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra WAIT_%=;\n}\n" :: "r"(smem_u32(bar)), "r"(parity) : "memory");
}
// bytes (multiple of 16) from global src (16-byte aligned) into shared dst,
// completion counted on bar (which expects them)
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(smem_u32(bar)), "r"(bytes) : "memory");
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               :: "r"(smem_u32(dst)), "l"(src), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}

template <typename T>
struct PellDev {          // plain ELLPACK (column-major, -1 padding)
  int64_t m, K, pitch;
  const int32_t* col;
  const T* vals;
  const T* x;
};

template <typename T>
struct CooDev {           // (BRO-)COO part
  int64_t nnz, nI;
  const uint32_t* words;
  const uint32_t* base_row;
  const uint8_t* width;
  const uint64_t* symptr;
  const int32_t* rows;    // plain COO only
  const int32_t* col;
  const T* vals;
  const T* x;
  T* cf;                  // per interval: partial of its first row (when that row spans intervals)
  T* cl;                  // per interval: partial of its last row (when that row spans intervals)
  const int32_t* end_row; // per interval: row of its last entry (computed at create)
};

// Programmatic dependent launch (PDL): a kernel launched with the
// programmatic-serialization attribute may start while the previous kernel
// of the stream finishes; it must execute griddepcontrol.wait before it
// touches memory that kernel writes.  Without the attribute both are no-ops.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_launch_dependents() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

// ------------------------------------------------------------------ BRO-ELL values
// G values of row r (slot columns j .. j+G-1) of a slice of H rows: 16-byte
// chunks where the chunk is full, scalar loads in the tail chunk, 0 past l.
template <typename T, int G, int H>
__device__ __forceinline__ void load_vals(T* v, const T* vs, int j, int l, int lfull, int r) {
  constexpr int VV = Chunk<T>::N;
  if (j + G <= lfull) {
#pragma unroll
    for (int u = 0; u < G / VV; ++u) {
      Chunk<T> c;
      c.load(vs + H * (j + u * VV) + r * VV);
#pragma unroll
      for (int q = 0; q < VV; ++q) v[u * VV + q] = c.v[q];
    }
  } else {
    const int tw = l - lfull;  // tail slots per row (< VV), contiguous per row
#pragma unroll
    for (int u = 0; u < G / VV; ++u) {
      const int jj = j + u * VV;
      if (jj + VV <= lfull) {
        Chunk<T> c;
        c.load(vs + H * jj + r * VV);
#pragma unroll
        for (int k = 0; k < VV; ++k) v[u * VV + k] = c.v[k];
      } else {
#pragma unroll
        for (int k = 0; k < VV; ++k)
          v[u * VV + k] = (jj + k < l) ? ld_stream(vs + H * lfull + r * tw + (jj + k - lfull)) : T(0);
      }
    }
  }
}

// Value indexing (reading R28, the "value data compression" of P:L416 by the
// value-index method of [16]): the G values of row r are codes of CB bytes in
// 4-byte chunks of 4/CB codes (slot layout, P:L116 multiplexing), looked up in
// the table of distinct values (a few KB at most: L1-resident).
template <int CB>
__device__ __forceinline__ uint32_t ld_code(const uint8_t* p) {
  uint32_t r;
  if constexpr (CB == 1) asm("ld.global.nc.L1::no_allocate.u8 %0, [%1];" : "=r"(r) : "l"(p));
  else asm("ld.global.nc.L1::no_allocate.u16 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}
template <typename T, int G, int H, int CB>
__device__ __forceinline__ void load_vals_vi(T* v, const uint8_t* cs, const T* __restrict__ dict, uint32_t pad,
                                             int j, int l, int r) {
  constexpr int VC = 4 / CB;
  static_assert(G % VC == 0, "a column group holds whole 4-byte code chunks");
  const int lfull = (l / VC) * VC;
  uint32_t code[G];
  auto chunk = [&](int u, int jj) {
    const uint32_t w = ld_stream_u32(reinterpret_cast<const uint32_t*>(cs + CB * (H * jj + r * VC)));
#pragma unroll
    for (int q = 0; q < VC; ++q) code[u * VC + q] = CB == 1 ? (w >> (8 * q)) & 0xffu : (w >> (16 * q)) & 0xffffu;
  };
  if (j + G <= lfull) {
#pragma unroll
    for (int u = 0; u < G / VC; ++u) chunk(u, j + u * VC);
  } else {
    const int tw = l - lfull;  // tail codes per row (< VC), contiguous per row
#pragma unroll
    for (int u = 0; u < G / VC; ++u) {
      const int jj = j + u * VC;
      if (jj + VC <= lfull) {
        chunk(u, jj);
      } else {
#pragma unroll
        for (int k = 0; k < VC; ++k)
          code[u * VC + k] = jj + k < l ? ld_code<CB>(cs + CB * (H * lfull + r * tw + (jj + k - lfull))) : pad;
      }
    }
  }
#pragma unroll
  for (int k = 0; k < G; ++k) v[k] = __ldg(dict + code[k]);
}

// Copy symbol rows [qa, qa + nrows) of this lane's R rows into
// win[((q - qa) * 32 + lane) * R + k] (zeros past S) plus one zero guard row.
// Copy symbol rows [qa, qa + nrows) of this lane's R rows into
// win[((q - qa) * 32 + lane) * R + k] (zeros past S) plus one zero guard row.
// kB rows per batch, every load of a batch issued before its first store, so
// a window of n rows arrives in ceil(n / kB) round trips (the group loop's
// registers are free at this point of the slice).
template <int V, int R, int kB>
__device__ __forceinline__ void stage_symbols(uint32_t* win, const uint32_t* __restrict__ wb, int S, int qa,
                                              int nrows, int lane) {
  constexpr int H = 32 * R;
  if constexpr (V == 1) {
    for (int r0 = 0; r0 < nrows; r0 += kB) {
      uint32_t w[kB][R];
#pragma unroll
      for (int u = 0; u < kB; ++u) {
        const int q = qa + r0 + u;
#pragma unroll
        for (int k = 0; k < R; ++k) w[u][k] = 0u;
        if (r0 + u < nrows && q < S) {
#pragma unroll
          for (int k = 0; k < R; ++k) w[u][k] = ld_stream_u32_g(wb + H * q + 32 * k + lane);
        }
      }
#pragma unroll
      for (int u = 0; u < kB; ++u) {
        if (r0 + u < nrows) {
          if constexpr (R == 1) win[(r0 + u) * 32 + lane] = w[u][0];
          else reinterpret_cast<uint2*>(win)[(r0 + u) * 32 + lane] = make_uint2(w[u][0], w[u][1]);
        }
      }
    }
  } else {
    static_assert(V == 4, "V must be 1 or 4");
    constexpr int kC = (kB + 3) / 4 + 1;  // 16-byte chunks covering kB rows at any alignment
    const int F = S >> 2;
    const int Vp = S - 4 * F;
    const int c_lo = qa >> 2, c_hi = (qa + nrows - 1) >> 2;
    for (int c0 = c_lo; c0 <= c_hi; c0 += kC) {
      uint32_t w4[kC][R][4];
#pragma unroll
      for (int cc = 0; cc < kC; ++cc) {
        const int c = c0 + cc;
#pragma unroll
        for (int k = 0; k < R; ++k) {
          const int row = 32 * k + lane;
#pragma unroll
          for (int e = 0; e < 4; ++e) w4[cc][k][e] = 0u;
          if (c <= c_hi && c < F) {
            const uint4 v = ld_stream_u4_g(wb + H * 4 * c + 4 * row);
            w4[cc][k][0] = v.x; w4[cc][k][1] = v.y; w4[cc][k][2] = v.z; w4[cc][k][3] = v.w;
          } else if (c <= c_hi && c == F) {
#pragma unroll
            for (int e = 0; e < 4; ++e)
              if (e < Vp) w4[cc][k][e] = ld_stream_u32_g(wb + H * 4 * F + Vp * row + e);
          }
        }
      }
#pragma unroll
      for (int cc = 0; cc < kC; ++cc) {
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const int r = 4 * (c0 + cc) + e - qa;
          if (c0 + cc <= c_hi && r >= 0 && r < nrows) {
            if constexpr (R == 1) win[r * 32 + lane] = w4[cc][0][e];
            else reinterpret_cast<uint2*>(win)[r * 32 + lane] = make_uint2(w4[cc][0][e], w4[cc][1][e]);
          }
        }
      }
    }
  }
  if constexpr (R == 1) win[nrows * 32 + lane] = 0u;
  else reinterpret_cast<uint2*>(win)[nrows * 32 + lane] = make_uint2(0u, 0u);
}

// ------------------------------------------------------------------ BRO-ELL, offset decode
// Widths are shared by the slice's rows, so the bit offset of
// column j inside every row stream is the same: o_j = sum_{i<j} b_i.  Per
// block of up to 32 columns the warp computes the offsets with one SHFL scan,
// stages the block's symbols (<= 33 per row) in the per-warp window, and each
// column's delta is the branch-free extraction
//     delta = funnelshift(w[q+1], w[q], o mod 32) >> (32 - b),   q = o / 32.
// G columns per group; kRows window rows per warp (34 holds any 32-column
// block: <= 33 symbol rows + a zero guard row; smaller windows for matrices
// whose row streams are all shorter leave more of the SM's memory to L1).
// L2 prefetch (TMA engine, no registers, no shared memory) of [p, p + bytes);
// p and bytes multiples of 16.
__device__ __forceinline__ void prefetch_l2(const void* p, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" :: "l"(p), "r"(bytes) : "memory");
}

// kPf > 0: at the start of a slice, lane 0 asks the TMA engine to prefetch
// into L2 the values, symbols and widths of the slice this warp handles kPf
// slices later, so its own loads of that slice hit L2 instead of HBM.
// kPipe: software-pipelined column groups (group g+1 issued before group g's FMAs).
// kX: x-window staging (single-pass grids only: block b handles slices
// [b*kWarps, (b+1)*kWarps)): at block start one thread has the TMA engine copy
// the block's x window p.xwin[b] into dynamic shared memory; the gathers then
// read shared memory (north_star: "the x gather ... with TMA or shared-memory
// staging where the slice's column window fits").
// kPfAt: when the prefetch is issued — 0 at the slice start, k (1..3) once the
// warp reaches column k*l/4 of the current slice (a later trigger keeps fewer
// prefetched bytes waiting in L2 per warp, so more warps can prefetch).
// kP > 1 (multiple warps per slice, the "multiple threads per row" of P:L416):
// the kP adjacent warps of a block share one slice, warp `part` owning the
// column range [part*cs, part*cs + cs) (cs = ceil(l / kP) rounded up to G).
// A warp decodes the columns before its range without gathering (the column
// index of a row is the prefix sum of its deltas), then the block adds the kP
// partial sums of each row in part order (deterministic) and stores y.  For
// matrices with few, long slices (C2): kP times more warps stream values.
template <typename T, int V, int R, int kWarps, int kMinBlocks, int G, int kRows, int kMode, int kPf = 0,
          bool kL1 = false, int kPfAt = 0, bool kPipe = false, int kSB = 0, bool kX = false, int kP = 1,
          int kVI = 0>
__global__ void __launch_bounds__(kWarps * 32, kMinBlocks)
bro_ell_od(const EllDev<T> p, const YOut<T> y, int32_t* __restrict__ dec) {
  static_assert(G % Chunk<T>::N == 0, "a column group holds whole 16-byte value chunks");
  static_assert(kWarps % kP == 0 && (kP == 1 || (!kPipe && !kX && kPf == 0)), "split slices: plain groups only");
  constexpr int kSl = kWarps / kP;  // slices per block per pass
  // symbol rows staged per round trip, sized by the instance's register
  // budget (16 / 12 / 8 loads in flight for >= 96 / >= 80 / fewer registers)
  constexpr int kMaxRegs = 65536 / (kWarps * 32 * kMinBlocks);
  constexpr int kLoads = kMaxRegs >= 96 ? 16 : kMaxRegs >= 80 ? 12 : 8;
  constexpr int kStageB = kSB ? kSB : (kRows - 1 < kLoads / R ? kRows - 1 : kLoads / R);
  constexpr int H = 32 * R;
  struct Meta { uint64_t c0, q0; int l, S; };
  __shared__ __align__(16) uint32_t window[kWarps][kRows * H];
  __shared__ uint2 colmeta[kWarps][32];  // per column of the block: {byte offset of its word row, r | (32-b) << 8}
  __shared__ Meta metas[kWarps][32];     // metadata of this warp's next 32 slices
  const int lane = threadIdx.x & 31;
  const int w = threadIdx.x >> 5;
  if constexpr (kMode == kSpmv) pdl_launch_dependents();  // a HYB handle's COO part may be scheduled
  uint32_t* win = window[w];
  const uint2* cm = colmeta[w];
  // x window of this block (kX): columns [xlo, xlo + xn) in shared memory
  extern __shared__ __align__(128) unsigned char dsm[];
  __shared__ uint64_t xbar;
  const T* xs = reinterpret_cast<const T*>(dsm);
  int xlo = 0, xn = 0;
  if constexpr (kX) {
    const int2 wl = p.xwin[blockIdx.x];
    xlo = wl.x;
    xn = wl.y;
    if (threadIdx.x == 0) {
      mbar_init(&xbar, 1);
      if (xn > 0) bulk_g2s(dsm, p.x + xlo, uint32_t(xn * int(sizeof(T))), &xbar);
    }
    __syncthreads();
  }
  bool xready = !kX;
  const char* win_lane = reinterpret_cast<const char*>(win + lane * R);
  const T* __restrict__ xg = in_reg(p.x, p.m >> 62);
  const int part = kP > 1 ? w % kP : 0;
  __shared__ T psum[kP > 1 ? kWarps : 1][kP > 1 ? H : 1];  // split slices: partial sums per part
  const int64_t stride = int64_t(gridDim.x) * kSl;
  int k32 = 0;
  // block-uniform trip count (the split epilogue synchronises the block)
  for (int64_t t0 = int64_t(blockIdx.x) * kSl; t0 < p.s; t0 += stride, k32 = (k32 + 1) & 31) {
    const int64_t t = t0 + w / kP;
    T sum[R];
#pragma unroll
    for (int k = 0; k < R; ++k) sum[k] = T(0);
    if (t < p.s) {
    __syncwarp();
    if (k32 == 0) {  // one round trip fetches the metadata of the next 32 slices
      const int64_t tl = t + lane * stride;
      if (tl < p.s) {
        const uint64_t c0l = __ldg(p.colptr + tl), q0l = __ldg(p.symptr + tl);
        metas[w][lane] = Meta{c0l, q0l, int(__ldg(p.colptr + tl + 1) - c0l), int(__ldg(p.symptr + tl + 1) - q0l)};
      }
      __syncwarp();
    }
    const Meta mt = metas[w][k32];
    // prefetch of the slice this warp handles kPf slices later (lane 0)
    auto prefetch_next = [&]() {
      if (lane == 0 && k32 + kPf < 32 && t + kPf * stride < p.s) {
        const Meta nx = metas[w][k32 + kPf];
        if (nx.l > 0) {
          if constexpr (kVI == 0) prefetch_l2(p.vals + H * nx.c0, uint32_t(H * nx.l * sizeof(T)));
          prefetch_l2(p.words + H * nx.q0, uint32_t(H * nx.S * 4));
          const uint64_t b0 = nx.c0 & ~uint64_t(15), b1 = (nx.c0 + uint64_t(nx.l) + 15) & ~uint64_t(15);
          prefetch_l2(p.bit_alloc + b0, uint32_t(b1 - b0));
          if constexpr (kVI > 0) prefetch_l2(p.vcodes + kVI * H * nx.c0, uint32_t((kVI * H * nx.l + 15) & ~15));
        }
      }
    };
    if constexpr (kPf > 0 && kPfAt == 0 && kMode != kDecode) prefetch_next();
    const int l = mt.l;
    const int S = mt.S;
    const uint32_t* wb = p.words + H * mt.q0;
    const T* vs = p.vals + H * mt.c0;
    const uint8_t* vcs = kVI > 0 ? p.vcodes + kVI * H * mt.c0 : nullptr;
    const uint8_t* ba = p.bit_alloc + mt.c0;
    const int lfull = (l / Chunk<T>::N) * Chunk<T>::N;
    int col[R];
#pragma unroll
    for (int k = 0; k < R; ++k) col[k] = -1;
    // this warp's column range [j0, j1) of the slice (the whole slice if kP = 1)
    int j0 = 0, j1 = l;
    if constexpr (kP > 1) {
      const int cs = ((l + kP - 1) / kP + G - 1) / G * G;
      j0 = min(l, part * cs);
      j1 = min(l, j0 + cs);
    }
    int obase = 0;  // bit offset of the current block inside every row stream
    for (int jb = 0; jb < j1; jb += 32) {
      const int nb = min(32, l - jb);
      const int b = lane < nb ? int(__ldg(ba + jb + lane)) : 0;
      if (jb == 0) {  // first block starts at symbol 0: stage without waiting for the scan
        __syncwarp();
        stage_symbols<V, R, kStageB>(win, wb, S, 0, min(S, kRows - 1), lane);
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
        stage_symbols<V, R, kStageB>(win, wb, S, qa, nrows, lane);
      }
      {
        const int rel = b ? obase + incl - b - 32 * qa : 0;  // column jb+lane inside the window
        colmeta[w][lane] = make_uint2(uint32_t(rel >> 5) * uint32_t(128 * R),
                                      uint32_t(rel & 31) | ((32u - uint32_t(b)) << 8));
      }
      __syncwarp();
      // one group = G columns of the block: its R x G values, decoded columns
      // and x gathers (padding slots: delta 0, no gather, no FMA; Alg. 1 line 17)
      struct Grp {
        T v[R][G];
        T xv[R][G];
        int cidx[R][G];
        bool ok[R][G];
      };
      auto issue = [&](Grp& q, int g) {  // loads of group g: values, decode, gathers
        if constexpr (kPf > 0 && kPfAt > 0 && kMode != kDecode) {
          const int at = (kPfAt * l) >> 2;  // trigger column
          if (jb + g <= at && at < jb + g + G) prefetch_next();
        }
        if constexpr (kMode != kDecode) {
#pragma unroll
          for (int k = 0; k < R; ++k) {
            if constexpr (kVI > 0) load_vals_vi<T, G, H, kVI>(q.v[k], vcs, p.vdict, p.vpad, jb + g, l, 32 * k + lane);
            else load_vals<T, G, H>(q.v[k], vs, jb + g, l, lfull, 32 * k + lane);
          }
        }
#pragma unroll
        for (int kk = 0; kk < G; ++kk) {
          const uint2 mm = cm[g + kk];  // broadcast
          uint32_t hi[R], lo[R];
          if constexpr (R == 1) {
            const uint32_t* wp = reinterpret_cast<const uint32_t*>(win_lane + mm.x);
            hi[0] = wp[0];
            lo[0] = wp[32];
          } else {
            const uint2* wp = reinterpret_cast<const uint2*>(win_lane + mm.x);
            const uint2 a = wp[0], c = wp[32];
            hi[0] = a.x; hi[1] = a.y; lo[0] = c.x; lo[1] = c.y;
          }
          const uint32_t sh = mm.y >> 8;
#pragma unroll
          for (int k = 0; k < R; ++k) {
            // funnelshift_l uses the low 5 bits of mm.y (= r); bits 8.. hold 32-b
            const uint32_t d = shr_clamp(__funnelshift_l(lo[k], hi[k], mm.y), sh);
            col[k] += int(d);
            q.cidx[k][kk] = col[k];
            q.ok[k][kk] = d != 0u;
          }
        }
        if constexpr (kMode == kDecode) {
          // decoded column per slot (V = 1 slot order: h*colptr + h*j + row), -1 = padding
#pragma unroll
          for (int k = 0; k < R; ++k)
#pragma unroll
            for (int kk = 0; kk < G; ++kk)
              if (g + kk < nb) dec[H * (mt.c0 + jb + g + kk) + 32 * k + lane] = q.ok[k][kk] ? q.cidx[k][kk] : -1;
        } else {
          if constexpr (kX) {
            if (!xready) {  // the block's x window has landed in shared memory
              mbar_wait(&xbar, 0);
              xready = true;
            }
          }
#pragma unroll
          for (int k = 0; k < R; ++k)
#pragma unroll
            for (int kk = 0; kk < G; ++kk) {
              q.xv[k][kk] = T(0);  // padding slots: value 0 (stored) times 0 adds +0
              if (q.ok[k][kk]) {
                if constexpr (kX) {
                  const int cx = q.cidx[k][kk] - xlo;  // columns past the staged window (its 16-byte tail) from global
                  q.xv[k][kk] = unsigned(cx) < unsigned(xn) ? xs[cx] : ldg_x(xg + q.cidx[k][kk]);
                } else {
                  q.xv[k][kk] = ldg_x(xg + q.cidx[k][kk]);
                }
              }
            }
        }
      };
      auto consume = [&](const Grp& q) {
        if constexpr (kMode != kDecode) {
#pragma unroll
          for (int k = 0; k < R; ++k)
#pragma unroll
            for (int kk = 0; kk < G; ++kk)
              // stored padding values are 0 and their x is never gathered (0):
              // the FMA adds +0 and needs no select (two FSELs per fp64 slot
              // on this issue-bound loop: C5 fp64 330.6 -> 311.9 us, fp32
              // 202.3 -> 191.4 us; value-indexed C5 fp64 303.7 -> 273.6 us: its
              // padding code is a finite value, reading R28).  The predicate
              // stays in the 51-register mid-window instance (C4 fp64 99.1 vs
              // 110.0 us) and the fp32 few-slice instance with 32-column groups
              // (C2 fp32 16.7 vs 18.6 us).
              if constexpr (kMaxRegs >= 56 && !(sizeof(T) == 4 && G >= 32)) sum[k] = fma(q.v[k][kk], q.xv[k][kk], sum[k]);
              else if (q.ok[k][kk]) sum[k] = fma(q.v[k][kk], q.xv[k][kk], sum[k]);
        }
      };
      if constexpr (!kPipe) {
        for (int g = 0; g < nb; g += G) {
          if constexpr (kP > 1) {
            if (jb + g >= j1) break;
            if (jb + g < j0) {  // before this warp's range: advance the column indices only
#pragma unroll
              for (int kk = 0; kk < G; ++kk) {
                const uint2 mm = cm[g + kk];
                const uint32_t* wp = reinterpret_cast<const uint32_t*>(win_lane + mm.x);
#pragma unroll
                for (int k = 0; k < R; ++k)
                  col[k] += int(shr_clamp(__funnelshift_l(wp[32 * R + k], wp[k], mm.y), mm.y >> 8));
              }
              continue;
            }
          }
          Grp q;
          issue(q, g);
          consume(q);
        }
      } else {
        // software pipeline: group g+G's values and gathers are in flight
        // while group g's FMAs wait for theirs
        Grp qa, qb;
        issue(qa, 0);
        for (int g = 0; g < nb; g += 2 * G) {
          if (g + G < nb) issue(qb, g + G);
          consume(qa);
          if (g + G >= nb) break;
          if (g + 2 * G < nb) issue(qa, g + 2 * G);
          consume(qb);
        }
      }
      obase += tot;
    }
    }  // t < p.s
    if constexpr (kMode != kDecode) {
      if constexpr (kP > 1) {  // partials of the slice's kP warps, added in part order
#pragma unroll
        for (int k = 0; k < R; ++k) psum[w][32 * k + lane] = sum[k];
        __syncthreads();
        if (part == 0 && t < p.s) {
#pragma unroll
          for (int k = 0; k < R; ++k) {
            T s = psum[w][32 * k + lane];
#pragma unroll
            for (int q = 1; q < kP; ++q) s += psum[w + q][32 * k + lane];
            const int64_t row = H * t + 32 * k + lane;
            if (row < p.m) store_y<kMode>(y, row, s);
          }
        }
        __syncthreads();
      } else if (t < p.s) {
#pragma unroll
        for (int k = 0; k < R; ++k) {
          const int64_t row = H * t + 32 * k + lane;
          if (row < p.m) store_y<kMode>(y, row, sum[k]);
        }
      }
    }
  }
}

// ------------------------------------------------------------------ BRO-ELL, tiny slices
// Every slice has l <= 4 columns (e.g. the ELL part of C3's BRO-HYB, K = 2),
// so a row stream has S <= 4 symbols: each lane keeps its rows' <= 4 words in
// registers — no shared window, no width scan, no column records.  Per slice
// one round trip fetches the widths (broadcast), the words and the values
// together, then one fetches the x gathers.  Field j starts at the
// warp-uniform offset o_j = b_0 + ... + b_{j-1}, so q = o_j / 32 selects the
// word pair uniformly.
template <typename T, int V, int R, int kWarps, int kMinBlocks, int kMode, int kVI = 0>
__global__ void __launch_bounds__(kWarps * 32, kMinBlocks)
bro_ell_tiny(const EllDev<T> p, const YOut<T> y, int32_t* __restrict__ dec) {
  constexpr int H = 32 * R;
  struct Meta { uint64_t c0, q0; int l, S; };
  __shared__ Meta metas[kWarps][32];  // metadata of this warp's next 32 slices
  const int lane = threadIdx.x & 31;
  const int w = threadIdx.x >> 5;
  if constexpr (kMode == kSpmv) pdl_launch_dependents();  // a HYB handle's COO part may be scheduled
  const int64_t stride = int64_t(gridDim.x) * kWarps;
  int k32 = 0;
  for (int64_t t = int64_t(blockIdx.x) * kWarps + w; t < p.s; t += stride, k32 = (k32 + 1) & 31) {
    __syncwarp();
    if (k32 == 0) {
      const int64_t tl = t + lane * stride;
      if (tl < p.s) {
        const uint64_t c0l = __ldg(p.colptr + tl), q0l = __ldg(p.symptr + tl);
        metas[w][lane] = Meta{c0l, q0l, int(__ldg(p.colptr + tl + 1) - c0l), int(__ldg(p.symptr + tl + 1) - q0l)};
      }
      __syncwarp();
    }
    const Meta mt = metas[w][k32];
    const int l = mt.l, S = mt.S;
    const uint32_t* wb = p.words + H * mt.q0;
    const uint8_t* ba = p.bit_alloc + mt.c0;
    int bw[4];
#pragma unroll
    for (int j = 0; j < 4; ++j) bw[j] = j < l ? int(__ldg(ba + j)) : 0;
    uint32_t wd[R][5];
    T v[R][4];
    const int lfull = (l / Chunk<T>::N) * Chunk<T>::N;
#pragma unroll
    for (int k = 0; k < R; ++k) {
      const int row = 32 * k + lane;
#pragma unroll
      for (int q = 0; q < 4; ++q) wd[k][q] = q < S ? ld_stream_u32(wb + place(row, q, S, V, H)) : 0u;
      wd[k][4] = 0u;
      if constexpr (kMode != kDecode) {
        if (l > 0) {
          if constexpr (kVI > 0) load_vals_vi<T, 4, H, kVI>(v[k], p.vcodes + kVI * H * mt.c0, p.vdict, p.vpad, 0, l, row);
          else load_vals<T, 4, H>(v[k], p.vals + H * mt.c0, 0, l, lfull, row);
        } else {
#pragma unroll
          for (int q = 0; q < 4; ++q) v[k][q] = T(0);
        }
      }
    }
    int cidx[R][4];
    bool ok[R][4];
#pragma unroll
    for (int k = 0; k < R; ++k) {
      int c = -1, o = 0;
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const int b = bw[j];
        const int q = o >> 5;
        const uint32_t hi = q == 0 ? wd[k][0] : q == 1 ? wd[k][1] : q == 2 ? wd[k][2] : wd[k][3];
        const uint32_t lo = q == 0 ? wd[k][1] : q == 1 ? wd[k][2] : q == 2 ? wd[k][3] : wd[k][4];
        const uint32_t d = shr_clamp(__funnelshift_l(lo, hi, uint32_t(o & 31)), uint32_t(32 - b));
        c += int(d);
        cidx[k][j] = c;
        ok[k][j] = d != 0u;  // padding (and j >= l: b = 0) is skipped, Alg. 1 line 17
        o += b;
      }
    }
    if constexpr (kMode == kDecode) {
#pragma unroll
      for (int k = 0; k < R; ++k)
#pragma unroll
        for (int j = 0; j < 4; ++j)
          if (j < l) dec[H * (mt.c0 + j) + 32 * k + lane] = ok[k][j] ? cidx[k][j] : -1;
    } else {
      const T* __restrict__ xg = in_reg(p.x, p.m >> 62);
      T xv[R][4];
#pragma unroll
      for (int k = 0; k < R; ++k)
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          xv[k][j] = T(0);
          if (ok[k][j]) xv[k][j] = ldg_x(xg + cidx[k][j]);
        }
#pragma unroll
      for (int k = 0; k < R; ++k) {
        T sum = T(0);
#pragma unroll
        for (int j = 0; j < 4; ++j) {  // padding (and j >= l): stored value 0 times x = 0 (as in bro_ell_od)
          sum = fma(v[k][j], xv[k][j], sum);
        }
        const int64_t row = H * t + 32 * k + lane;
        if (row < p.m) store_y<kMode>(y, row, sum);
      }
    }
  }
}

// ------------------------------------------------------------------ plain ELLPACK
template <typename T, int kThreads, int kMode>
__global__ void __launch_bounds__(kThreads)
ell_spmv(const PellDev<T> p, const YOut<T> y, int32_t* __restrict__ dec) {
  constexpr int G = 8;
  const int64_t row = int64_t(blockIdx.x) * kThreads + threadIdx.x;
  if constexpr (kMode == kSpmv) pdl_launch_dependents();  // a HYB handle's COO part may be scheduled
  if (row >= p.m) return;
  if constexpr (kMode == kDecode) {
    for (int64_t j = 0; j < p.K; ++j) dec[j * p.pitch + row] = ld_stream_s32(p.col + j * p.pitch + row);
    return;
  }
  T sum = T(0);
  int64_t j = 0;
  for (; j + G <= p.K; j += G) {
    int c[G];
    T v[G];
#pragma unroll
    for (int k = 0; k < G; ++k) {
      c[k] = ld_stream_s32(p.col + (j + k) * p.pitch + row);
      v[k] = ld_stream(p.vals + (j + k) * p.pitch + row);
    }
    T xv[G];
#pragma unroll
    for (int k = 0; k < G; ++k) xv[k] = c[k] >= 0 ? ldg_x(p.x + c[k]) : T(0);
#pragma unroll
    for (int k = 0; k < G; ++k) sum = fma(v[k], xv[k], sum);
  }
  for (; j < p.K; ++j) {
    const int c = ld_stream_s32(p.col + j * p.pitch + row);
    const T v = ld_stream(p.vals + j * p.pitch + row);
    if (c >= 0) sum = fma(v, ldg_x(p.x + c), sum);
  }
  store_y<kMode>(y, row, sum);
}

// ------------------------------------------------------------------ (BRO-)COO
// One warp per interval of 32*T entries; lane l owns the T
// consecutive entries e = i*32T + T*l + t (reading R13), stored
// lane-contiguously in 16-byte chunks (reading R26: entry (l, t) at
// i*32T + place(l, t, T, chunk)), processed in batches of 8.
//
// Rows (BRO): deltas follow entry order (row(e) - row(e-1)), one width b per
// interval.  The lane's T fields sit at the warp-uniform offsets t*b of its
// stream, staged as a [q][lane] window: pass 1 sums the lane's fields, one
// warp scan of the lane sums gives each lane its start row, pass 2 decodes
// the rows batch by batch.
//
// Multiply: each lane reduces its entries sequentially (segments of equal
// rows); ONE warp segmented scan per interval links the lanes' trailing and
// leading partials.  A row complete inside the interval and other than its
// first row receives exactly one fire-and-forget RED into y (each such row
// lives in exactly one interval, so the sum is deterministic); the first and
// last rows' partials go to carry arrays for the deterministic fix-up.
template <typename T>
struct Vec8 {  // 8 consecutive entries of one lane: 16-byte chunks
  T v[8];
  __device__ __forceinline__ void load(const T* base, int t0, int lane) {
    constexpr int N = Chunk<T>::N;
#pragma unroll
    for (int u = 0; u < 8 / N; ++u) {
      Chunk<T> c;
      c.load(base + 32 * (t0 + u * N) + N * lane);
#pragma unroll
      for (int q = 0; q < N; ++q) v[u * N + q] = c.v[q];
    }
  }
};

__device__ __forceinline__ void load8_s32(int* d, const int32_t* base, int t0, int lane) {
  const uint4 a = ld_stream_u4(base + 32 * t0 + 4 * lane);
  const uint4 b = ld_stream_u4(base + 32 * (t0 + 4) + 4 * lane);
  d[0] = int(a.x); d[1] = int(a.y); d[2] = int(a.z); d[3] = int(a.w);
  d[4] = int(b.x); d[5] = int(b.y); d[6] = int(b.z); d[7] = int(b.w);
}

// field t of this lane's stream of b-bit fields staged as [q][lane] (wl
// points at the lane's word of row 0); b >= 1.
__device__ __forceinline__ int coo_field(const uint32_t* wl, int t, int b) {
  const int o = t * b;
  const uint32_t* p = wl + 32 * (o >> 5);
  return int(shr_clamp(__funnelshift_l(p[32], p[0], uint32_t(o & 31)), uint32_t(32 - b)));
}

__device__ __forceinline__ void cp_async4(uint32_t* dst, const uint32_t* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(static_cast<uint32_t>(__cvta_generic_to_shared(dst))),
               "l"(src) : "memory");
}

template <typename T, bool kBro, int TT, int kWarps, int kMinBlocks, int kMode>
__global__ void __launch_bounds__(kWarps * 32, kMinBlocks)
coo_spmv(const CooDev<T> p, T* __restrict__ y, int32_t* __restrict__ dec) {
  constexpr int I = 32 * TT;
  constexpr int CH = TT < 16 ? TT : 16;  // entries per lane loaded at once (one chunk)
  constexpr int NC = TT / CH;
  __shared__ uint32_t cwin[kWarps][kBro ? (TT + 1) * 32 : 1];  // <= T symbol rows + a zero guard row
  const int lane = threadIdx.x & 31;
  const int w = threadIdx.x >> 5;
  const int64_t i = int64_t(blockIdx.x) * kWarps + w;
  if constexpr (kMode != kDecode) pdl_launch_dependents();  // the fix-up may be scheduled
  if (i >= p.nI) return;
  const int64_t e0 = i * I;
  const int32_t* cb = p.col + e0;
  const T* vb = p.vals + e0;
  const T* __restrict__ xg = in_reg(p.x, p.nnz >> 62);  // x base in a register (see in_reg)
  // per-lane segment state: f = row of the lane's first entry, A = partial of
  // its first segment, cr / cur = current (trailing) segment
  int f = 0, cr = 0;
  T A = T(0), cur = T(0);
  bool one = true;
  int b = 0, S = 0, row = 0, first = 0, lim = 0, prev_end = -1, next_first = -1;
  uint32_t w0 = 0, w1 = 0;
  const uint32_t* wl = cwin[w] + lane;
#pragma unroll
  for (int ch = 0; ch < NC; ++ch) {
    // the chunk's col / vals (and plain rows) first: nothing they need
    // depends on the interval header, so their round trip overlaps the
    // header -> word staging chain below
    int r[CH], c[CH];
    T v[CH];
    if constexpr (kMode != kDecode) {
#pragma unroll
      for (int u = 0; u < CH / 8; ++u) {
        load8_s32(c + 8 * u, cb, CH * ch + 8 * u, lane);
        Vec8<T> vv;
        vv.load(vb, CH * ch + 8 * u, lane);
#pragma unroll
        for (int k = 0; k < 8; ++k) v[8 * u + k] = vv.v[k];
      }
    }
    if constexpr (!kBro) {
#pragma unroll
      for (int u = 0; u < CH / 8; ++u) load8_s32(r + 8 * u, p.rows + e0, CH * ch + 8 * u, lane);
    }
    if (ch == 0) {
      lim = int(min(int64_t(I), p.nnz - e0));  // valid entries of the interval
      // the whole header at once, unconditionally: the words' address must not
      // wait for the width (width -> symptr -> words would be 3 round trips)
      first = int(p.base_row[i]);              // row of the interval's first entry
      row = first;
      // boundary rows for the epilogue: does the first row continue from
      // interval i-1, does the next interval start on this one's last row
      prev_end = i > 0 ? p.end_row[i - 1] : -1;
      next_first = i + 1 < p.nI ? int(p.base_row[i + 1]) : -1;
      if constexpr (kBro) {
        b = int(p.width[i]);
        const uint64_t q0 = p.symptr[i];
        S = int(p.symptr[i + 1] - q0);
        if (b > 0) {  // b = 0: one row for the whole interval, empty stream
          const uint32_t* wb = p.words + 32 * q0 + lane;  // V = 1: word q of lane l at 32q + l
          if (S <= 2) {
            // short streams (T*b <= 64 bits; C3/C4 intervals have small row
            // gaps): the lane's <= 2 words in registers, no window
            w0 = ld_stream_u32(wb);
            w1 = S > 1 ? ld_stream_u32(wb + 32) : 0u;
          } else {  // the lane words -> [q][lane] window by cp.async
            uint32_t* win = cwin[w] + lane;
            for (int q = 0; q < S; ++q) cp_async4(win + 32 * q, wb + 32 * q);
            asm volatile("cp.async.commit_group;" ::: "memory");
            win[32 * S] = 0u;
          }
        }
      }
    }
    T xv[CH];
    if constexpr (kMode != kDecode) {
#pragma unroll
      for (int k = 0; k < CH; ++k)  // slots past nnz hold col 0 / value 0: no gather
        xv[k] = TT * lane + CH * ch + k < lim ? ldg_x(xg + c[k]) : T(0);
    }
    if constexpr (kBro) {
      if (b > 0 && S <= 2) {
        // field t = bits [t*b, t*b + b) of the 64-bit stream w0:w1, MSB first
        const uint64_t W = (uint64_t(w0) << 32) | w1;
        int d[CH];
#pragma unroll
        for (int k = 0; k < CH; ++k) d[k] = int((W << ((CH * ch + k) * b)) >> (64 - b));
        if (ch == 0) {
          int tot = 0;  // sum of this lane's deltas (all T fields)
          if constexpr (NC == 1) {
#pragma unroll
            for (int k = 0; k < CH; ++k) tot += d[k];  // the chunk is the whole lane stream
          } else {
#pragma unroll
            for (int t = 0; t < TT; ++t) tot += int((W << (t * b)) >> (64 - b));
          }
          int incl = tot;
#pragma unroll
          for (int off = 1; off < 32; off <<= 1) {
            const int o = __shfl_up_sync(0xffffffffu, incl, off);
            if (lane >= off) incl += o;
          }
          row = first + incl - tot;  // row of the entry before this lane's first
        }
#pragma unroll
        for (int k = 0; k < CH; ++k) {
          row += d[k];
          r[k] = row;
        }
      } else {
        if (ch == 0 && b > 0) {
          asm volatile("cp.async.wait_group 0;" ::: "memory");
          __syncwarp();
          int tot = 0;  // pass 1: sum of this lane's deltas
#pragma unroll 8
          for (int t = 0; t < TT; ++t) tot += coo_field(wl, t, b);
          int incl = tot;
#pragma unroll
          for (int off = 1; off < 32; off <<= 1) {
            const int o = __shfl_up_sync(0xffffffffu, incl, off);
            if (lane >= off) incl += o;
          }
          row = first + incl - tot;  // row of the entry before this lane's first (its deltas follow)
        }
#pragma unroll
        for (int k = 0; k < CH; ++k) {
          if (b > 0) row += coo_field(wl, CH * ch + k, b);
          r[k] = row;
        }
      }
    }
    if constexpr (kMode == kDecode) {
#pragma unroll
      for (int k = 0; k < CH; ++k)
        if (TT * lane + CH * ch + k < lim) dec[e0 + TT * lane + CH * ch + k] = r[k];
    } else {
      // everything above only read constant inputs; y (stored by the ELL
      // part of a HYB handle) is updated from here on
      if (ch == 0) pdl_wait();
#pragma unroll
      for (int k = 0; k < CH; ++k) {
        const T prod = v[k] * xv[k];
        if (ch == 0 && k == 0) {
          f = r[0];
          cr = r[0];
          cur = prod;
        } else if (r[k] != cr) {  // the segment of row cr ends inside this lane
          if (one) { A = cur; one = false; }
          else atomicAdd(y + cr, cur);  // interior segment (row > first): complete, unique to this lane
          cr = r[k];
          cur = prod;
        } else {
          cur += prod;
        }
      }
    }
  }
  if constexpr (kMode == kDecode) return;
  if (one) A = cur;
  // segmented scan over the lanes: C_out(l) = cur_l + [one_l && link_l] C_out(l-1)
  const int L = cr;
  const int Lprev = __shfl_up_sync(0xffffffffu, L, 1);
  const bool link = lane > 0 && Lprev == f;  // this lane's first row continues the previous lane's last
  T co = cur;
  bool open = one && link;
#pragma unroll
  for (int off = 1; off < 32; off <<= 1) {
    const T o = __shfl_up_sync(0xffffffffu, co, off);
    const int op = __shfl_up_sync(0xffffffffu, int(open), off);
    if (lane >= off && open) co += o;
    if (lane >= off) open = open && op;
  }
  T cin = __shfl_up_sync(0xffffffffu, co, 1);
  if (!link) cin = T(0);
  // Complete segments of rows other than the interval's first row go straight
  // to y.  The first row F and the last row L go to y directly too unless they
  // span intervals (known statically: F spans if the previous interval ends
  // on F, L spans if the next one starts on L); then their partials are
  // carried for the fix-up, which adds each spanning row once, in interval
  // order.
  T fpart = T(0);
  bool hasF = false;
  auto emit = [&](int rr, T val) {
    if (rr == first) { fpart = val; hasF = true; }
    else atomicAdd(y + rr, val);
  };
  if (!one) emit(f, A + cin);  // first segment complete inside this lane
  const int fnext = __shfl_down_sync(0xffffffffu, f, 1);
  if (lane < 31 && fnext != L) emit(L, co);  // trailing segment complete at this lane
  const unsigned mF = __ballot_sync(0xffffffffu, hasF);
  const T Fp = mF ? __shfl_sync(0xffffffffu, fpart, __ffs(mF) - 1) : T(0);
  if (lane == 31) {
    const bool f_spans = prev_end == first;
    const bool l_spans = next_first == L;
    if (L == first) {  // one row for the whole interval: its partial is co
      if (f_spans || l_spans) p.cf[i] = co;
      else atomicAdd(y + first, co);
    } else {
      if (f_spans) p.cf[i] = Fp;
      else atomicAdd(y + first, Fp);
      if (l_spans) p.cl[i] = co;
      else atomicAdd(y + L, co);
    }
  }
}

// Exchange of a finished y for formats whose last kernel is not an ELL
// kernel (COO / HYB: the COO part and the fix-up add into y after the ELL
// part stored it, so only final values may leave the GPU): copy the local y
// (o.p[0]) into the other destinations, or once through the multicast address.
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

// Deterministic application of the carries of rows that span intervals: one
// thread per such row (precomputed at create: row R, first interval a, last
// interval b, whether R is a's last row or a starts with R), the partials
// summed in interval order: (a's cl or cf) + cf[a+1] + ... + cf[b], added to
// y[R] once.  The static span list is read before griddepcontrol.wait, so
// only the carries are read after the COO kernel completes.
template <typename T>
__global__ void coo_fixup(int64_t nS, const int4* __restrict__ spans, const T* __restrict__ cf,
                          const T* __restrict__ cl, T* __restrict__ y) {
  const int64_t k = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  int4 sp = make_int4(0, 0, -1, 0);
  if (k < nS) sp = spans[k];  // {row, a, b, a_uses_cl}
  pdl_wait();  // the carries come from the COO kernel
  if (k >= nS) return;
  T sum = sp.w ? cl[sp.y] : cf[sp.y];
  constexpr int B = 8;
  for (int j0 = sp.y + 1; j0 <= sp.z; j0 += B) {
    T c[B];
#pragma unroll
    for (int u = 0; u < B; ++u) c[u] = j0 + u <= sp.z ? cf[j0 + u] : T(0);
#pragma unroll
    for (int u = 0; u < B; ++u) sum += c[u];
  }
  y[sp.x] += sum;
}

}  // namespace dev
}  // namespace bro
