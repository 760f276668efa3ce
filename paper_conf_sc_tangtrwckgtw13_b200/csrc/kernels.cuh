// sm_100a SpMV kernels for BRO-ELL, BRO-COO (+ carry fix-up) and the
// uncompressed ELLPACK / COO baselines.
//
// Mapping (B200-first; the paper's Fermi/Kepler mapping of one 256-thread
// block per slice, is prior art):
//   * BRO-ELL: one WARP per 32-row slice, one lane per row (h = 32).  Every
//     per-column quantity of Alg. 1 (b = bit_alloc[c], rb, the refill branch)
//     is warp-uniform, so decode has no divergence.  A lane's
//     symbols are V-interleaved 16-byte chunks -> 128-bit loads; its values
//     are 16-byte chunks too.  The 32 widths of a column block live one per
//     lane and are broadcast with SHFL (replaces constant memory).
//     Decoding uses a 64-bit window (hi:lo) instead of Alg. 1's sym/rb pair
//     (reading R5/R6: no read past the row stream, no shift by sym_len).
//   * BRO-COO: one warp per interval of 32*T entries, a warp-shuffle
//     segmented scan per step (the "parallel scan primitive") with a
//     running carry, and a deterministic fix-up kernel for rows crossing
//     interval boundaries (the "extra kernel invocation for data reduction").
//   * Streamed arrays (symbols, values, COO col/row) are read with
//     ld.global.nc.L1::no_allocate; x is gathered through the read-only path.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace bro {
namespace dev {

constexpr int kWarp = 32;

// ------------------------------------------------------------------ loads
__device__ __forceinline__ uint4 ld_stream_u4(const uint32_t* p) {
  uint4 r;
  asm("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
      : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}
__device__ __forceinline__ uint32_t ld_stream_u32(const uint32_t* p) {
  uint32_t r;
  asm("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ int32_t ld_stream_s32(const int32_t* p) {
  int32_t r;
  asm("ld.global.nc.L1::no_allocate.s32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ double ld_stream(const double* p) {
  double r;
  asm("ld.global.nc.L1::no_allocate.f64 %0, [%1];" : "=d"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ float ld_stream(const float* p) {
  float r;
  asm("ld.global.nc.L1::no_allocate.f32 %0, [%1];" : "=f"(r) : "l"(p));
  return r;
}

// 16-byte value chunk: 2 doubles or 4 floats
template <typename T> struct Chunk;
template <> struct Chunk<double> {
  double v[2];
  static constexpr int N = 2;
  __device__ __forceinline__ void load(const double* p) {
    asm("ld.global.nc.L1::no_allocate.v2.f64 {%0,%1}, [%2];" : "=d"(v[0]), "=d"(v[1]) : "l"(p));
  }
};
template <> struct Chunk<float> {
  float v[4];
  static constexpr int N = 4;
  __device__ __forceinline__ void load(const float* p) {
    asm("ld.global.nc.L1::no_allocate.v4.f32 {%0,%1,%2,%3}, [%4];"
        : "=f"(v[0]), "=f"(v[1]), "=f"(v[2]), "=f"(v[3]) : "l"(p));
  }
};

template <typename T>
__device__ __forceinline__ T ldg_x(const T* p) { return __ldg(p); }

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
  const uint32_t* base;
  int S, lane, next, nbuf, remaining;
  uint32_t buf[8];
  uint32_t hi, lo;
  int avail;

  __device__ __forceinline__ void fetch8() {
    if constexpr (V == 4) {
      const int F = S >> 2;
      const int Vp = S - 4 * F;
#pragma unroll
      for (int h2 = 0; h2 < 2; ++h2) {
        const int c = (next >> 2) + h2;
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
        const int q = next + k;
        buf[k] = q < S ? ld_stream_u32(base + place(lane, q, S, V)) : 0u;
      }
    }
    next += 8;
    nbuf = 8;
  }
  __device__ __forceinline__ uint32_t pop() {
    if (nbuf == 0) fetch8();
    const uint32_t r = buf[0];
#pragma unroll
    for (int k = 0; k < 7; ++k) buf[k] = buf[k + 1];
    --nbuf;
    --remaining;
    return r;
  }
  __device__ __forceinline__ void init(const uint32_t* b, int S_, int lane_) {
    base = b; S = S_; lane = lane_; next = 0; nbuf = 0; remaining = S_;
    hi = 0; lo = 0; avail = 0;
    if (S > 0) { hi = pop(); avail = 32; }
  }
  __device__ __forceinline__ uint32_t get(int b) {  // 1 <= b <= 32
    const uint32_t v = hi >> (32 - b);
    hi = __funnelshift_lc(lo, hi, b);
    lo = shl_clamp(lo, b);
    avail -= b;
    if (avail < 32 && remaining > 0) {
      const uint32_t w = pop();
      hi |= w >> avail;
      lo = shl_clamp(w, 32 - avail);
      avail += 32;
    }
    return v;
  }
};

// ------------------------------------------------------------------ BRO-ELL
// y[32t + lane] = sum_j vals(slot) * x[col_j], Alg. 1.
template <typename T, int V, int kThreads>
__global__ void __launch_bounds__(kThreads)
bro_ell_spmv(int64_t m, int64_t s, const uint32_t* __restrict__ words,
             const uint8_t* __restrict__ bit_alloc, const uint64_t* __restrict__ colptr,
             const uint64_t* __restrict__ symptr, const T* __restrict__ vals,
             const T* __restrict__ x, T* __restrict__ y) {
  constexpr int VV = Chunk<T>::N;
  constexpr int G = 8;  // columns per unrolled group
  const int lane = threadIdx.x & 31;
  const int64_t t = int64_t(blockIdx.x) * (kThreads / 32) + (threadIdx.x >> 5);
  if (t >= s) return;
  const uint64_t c0 = colptr[t];
  const int l = int(colptr[t + 1] - c0);
  const uint64_t q0 = symptr[t];
  const int S = int(symptr[t + 1] - q0);
  LaneStream<V> ls;
  ls.init(words + 32 * q0, S, lane);
  const T* vs = vals + 32 * c0;
  const uint8_t* ba = bit_alloc + c0;
  const int lfull = (l / VV) * VV;
  T sum = T(0);
  int col = -1;
  uint32_t breg = 0;
  int j = 0;
  for (; j + G <= lfull; j += G) {
    if ((j & 31) == 0) breg = lane < l - j ? uint32_t(__ldg(ba + j + lane)) : 0u;
    Chunk<T> v[G / VV];
#pragma unroll
    for (int u = 0; u < G / VV; ++u) v[u].load(vs + 32 * (j + u * VV) + lane * VV);
    int cidx[G];
    bool ok[G];
#pragma unroll
    for (int k = 0; k < G; ++k) {
      const int b = (int)__shfl_sync(0xffffffffu, breg, (j + k) & 31);
      const uint32_t d = ls.get(b);
      col += int(d);
      cidx[k] = col;
      ok[k] = d != 0u;
    }
    T xv[G];
#pragma unroll
    for (int k = 0; k < G; ++k) xv[k] = ok[k] ? ldg_x(x + cidx[k]) : T(0);
#pragma unroll
    for (int k = 0; k < G; ++k) sum = fma(v[k / VV].v[k % VV], xv[k], sum);
  }
  for (; j < l; ++j) {
    if ((j & 31) == 0) breg = lane < l - j ? uint32_t(__ldg(ba + j + lane)) : 0u;
    const int b = (int)__shfl_sync(0xffffffffu, breg, j & 31);
    const uint32_t d = ls.get(b);
    col += int(d);
    const T* vp = j < lfull ? vs + 32 * (j - j % VV) + lane * VV + j % VV
                            : vs + 32 * lfull + lane * (l - lfull) + (j - lfull);
    const T v = ld_stream(vp);
    if (d != 0u) sum = fma(v, ldg_x(x + col), sum);
  }
  const int64_t row = 32 * t + lane;
  if (row < m) y[row] = sum;
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
    const uint32_t d = ls.get(bit_alloc[c0 + j]);
    col += int(d);
    out[32 * c0 + 32 * j + lane] = d ? col : -1;
  }
}

// ------------------------------------------------------------------ plain ELLPACK
template <typename T, int kThreads>
__global__ void __launch_bounds__(kThreads)
ell_spmv(int64_t m, int64_t K, int64_t pitch, const int32_t* __restrict__ col,
         const T* __restrict__ vals, const T* __restrict__ x, T* __restrict__ y) {
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
  y[row] = sum;
}

__global__ void ell_decode(int64_t m, int64_t K, int64_t pitch, const int32_t* __restrict__ col,
                           int32_t* __restrict__ out) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= K * pitch) return;
  out[i] = col[i];
  (void)m;
}

// ------------------------------------------------------------------ (BRO-)COO
// One warp per interval of 32*T entries.  Entry e0 + 32t + lane is element
// (t, lane).  Rows of fully-contained rows are added into y directly; the
// first row's and last row's partial sums go to carry arrays for the fix-up.
template <typename T, int V, bool kBro, int kThreads>
__global__ void __launch_bounds__(kThreads)
coo_spmv(int64_t nnz, int64_t nI, int T_steps, const uint32_t* __restrict__ words,
         const uint32_t* __restrict__ base_row, const uint8_t* __restrict__ width,
         const uint64_t* __restrict__ symptr, const int32_t* __restrict__ rows,
         const int32_t* __restrict__ col, const T* __restrict__ vals, const T* __restrict__ x,
         T* __restrict__ y, T* __restrict__ carry_first, T* __restrict__ carry_last,
         int32_t* __restrict__ last_row) {
  const int lane = threadIdx.x & 31;
  const int64_t i = int64_t(blockIdx.x) * (kThreads / 32) + (threadIdx.x >> 5);
  if (i >= nI) return;
  const int64_t e0 = i * 32 * T_steps;
  const int first = (int)base_row[i];
  int row = first;
  int b = 0;
  LaneStream<V> ls;
  if constexpr (kBro) {
    b = width[i];
    const uint64_t q0 = symptr[i];
    ls.init(words + 32 * q0, int(symptr[i + 1] - q0), lane);
  }
  T carry = T(0);
  int crow = first;
  for (int t = 0; t < T_steps; ++t) {
    const int64_t e = e0 + 32 * t + lane;
    const bool valid = e < nnz;
    if constexpr (kBro) {
      if (b) row += (int)ls.get(b);
    } else {
      row = ld_stream_s32(rows + (valid ? e : nnz - 1));
    }
    T p = T(0);
    if (valid) p = ld_stream(vals + e) * ldg_x(x + ld_stream_s32(col + e));
    // the carried row ended at the previous step's last lane
    const int row0 = __shfl_sync(0xffffffffu, row, 0);
    if (row0 != crow) {
      if (lane == 0) {
        if (crow == first) carry_first[i] = carry;
        else y[crow] += carry;
      }
      carry = T(0);
      crow = row0;
    }
    // inclusive segmented scan over lanes (rows are non-decreasing)
    T sc = p;
#pragma unroll
    for (int off = 1; off < 32; off <<= 1) {
      const T o = __shfl_up_sync(0xffffffffu, sc, off);
      const int ro = __shfl_up_sync(0xffffffffu, row, off);
      if (lane >= off && ro == row) sc += o;
    }
    if (row == crow) sc += carry;
    const int rn = __shfl_down_sync(0xffffffffu, row, 1);
    if (lane != 31 && rn != row) {
      if (row == first) carry_first[i] = sc;
      else y[row] += sc;
    }
    carry = __shfl_sync(0xffffffffu, sc, 31);
    crow = __shfl_sync(0xffffffffu, row, 31);
  }
  if (lane == 0) {
    last_row[i] = crow;
    if (crow == first) {
      carry_first[i] = carry;
      carry_last[i] = T(0);
    } else {
      carry_last[i] = carry;
    }
  }
}

// Deterministic application of interval carries (one thread per interval,
// fixed summation order = interval order).
template <typename T>
__global__ void coo_fixup(int64_t nI, const uint32_t* __restrict__ first,
                          const int32_t* __restrict__ last_row, const T* __restrict__ cf,
                          const T* __restrict__ cl, T* __restrict__ y) {
  const int64_t i = int64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  if (i >= nI) return;
  const int F = (int)first[i];
  const int L = last_row[i];
  if (L != F) {  // interval i is the first one holding row L
    T acc = cl[i];
    for (int64_t j = i + 1; j < nI && (int)first[j] == L; ++j) {
      acc += cf[j];
      if (last_row[j] != L) break;
    }
    y[L] += acc;
  }
  if (i == 0 || last_row[i - 1] != F) {  // interval i is the first one holding row F
    T acc = cf[i];
    if (L == F) {
      for (int64_t j = i + 1; j < nI && (int)first[j] == F; ++j) {
        acc += cf[j];
        if (last_row[j] != F) break;
      }
    }
    y[F] += acc;
  }
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
    if (b) row += (int)ls.get(b);
    const int64_t e = i * 32 * T_steps + 32 * t + lane;
    if (e < nnz) out[e] = row;
  }
}

}  // namespace dev
}  // namespace bro
