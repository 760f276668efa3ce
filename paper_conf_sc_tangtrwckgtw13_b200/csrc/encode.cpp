// Host-side BRO encoder (offline compression on the host CPU).
//
// BRO-ELL: per 32-row slice, per column j the width
// b_j = max Gamma(delta) over the slice's rows, the row streams padded to a
// multiple of 32 bits, then multiplexed so lane r reads its own symbols with
// coalesced 16-byte chunk loads.  BRO-COO: per interval of 32*T
// entries one width for all row deltas.  Multithreaded over slices /
// intervals (layouts are independent per slice).
#include "encode.hpp"

#include <algorithm>
#include <cstring>
#include <numeric>
#include <thread>
#include <unordered_set>

namespace bro {

int num_threads() {
  unsigned n = std::thread::hardware_concurrency();
  if (n == 0) n = 1;
  return (int)std::min(n, 64u);
}

template <class F>
static void parallel_for(int64_t n, F&& fn, int64_t grain = 256) {
  int nt = num_threads();
  if (n <= grain || nt == 1) {
    fn(int64_t(0), n);
    return;
  }
  int64_t chunks = std::min<int64_t>(nt, (n + grain - 1) / grain);
  std::vector<std::thread> th;
  th.reserve(chunks);
  for (int64_t c = 0; c < chunks; ++c) {
    int64_t lo = n * c / chunks, hi = n * (c + 1) / chunks;
    th.emplace_back([&fn, lo, hi] { fn(lo, hi); });
  }
  for (auto& t : th) t.join();
}

static void exclusive_scan(const std::vector<uint64_t>& cnt, std::vector<uint64_t>& ptr) {
  ptr.assign(cnt.size() + 1, 0);
  for (size_t i = 0; i < cnt.size(); ++i) ptr[i + 1] = ptr[i] + cnt[i];
}

std::string check_csr(int64_t m, int64_t n, const int64_t* row_ptr, const int32_t* col) {
  if (m < 0 || n < 0 || m >= (int64_t(1) << 31) || n >= (int64_t(1) << 31))
    return "shape: m and n must be in [0, 2^31)";
  if (!row_ptr) return "row_ptr is NULL";
  if (row_ptr[0] != 0) return "row_ptr[0] != 0";
  for (int64_t i = 0; i < m; ++i)
    if (row_ptr[i + 1] < row_ptr[i]) return "row_ptr is not non-decreasing at row " + std::to_string(i);
  if (row_ptr[m] > 0 && !col) return "col_idx is NULL";
  std::vector<int64_t> bad(num_threads(), -1);
  std::vector<int> kind(num_threads(), 0);
  int nt = num_threads();
  std::vector<std::thread> th;
  for (int c = 0; c < nt; ++c) {
    th.emplace_back([&, c] {
      int64_t lo = m * c / nt, hi = m * (c + 1) / nt;
      for (int64_t i = lo; i < hi && bad[c] < 0; ++i) {
        for (int64_t p = row_ptr[i]; p < row_ptr[i + 1]; ++p) {
          int32_t cc = col[p];
          if (cc < 0 || cc >= n) { bad[c] = i; kind[c] = 1; break; }
          if (p > row_ptr[i] && cc <= col[p - 1]) { bad[c] = i; kind[c] = 2; break; }
        }
      }
    });
  }
  for (auto& t : th) t.join();
  for (int c = 0; c < nt; ++c) {
    if (bad[c] >= 0)
      return (kind[c] == 1 ? "column index out of [0, n) in row " : "columns not strictly increasing in row ") +
             std::to_string(bad[c]);
  }
  return "";
}

std::string check_coo(int64_t m, int64_t n, int64_t nnz, const int32_t* row, const int32_t* col) {
  if (m < 0 || n < 0 || m >= (int64_t(1) << 31) || n >= (int64_t(1) << 31))
    return "shape: m and n must be in [0, 2^31)";
  if (nnz < 0) return "nnz < 0";
  if (nnz > 0 && (!row || !col)) return "row_idx/col_idx is NULL";
  for (int64_t e = 0; e < nnz; ++e) {
    if (row[e] < 0 || row[e] >= m) return "row index out of [0, m) at entry " + std::to_string(e);
    if (col[e] < 0 || col[e] >= n) return "column index out of [0, n) at entry " + std::to_string(e);
    if (e > 0) {
      if (row[e] < row[e - 1]) return "COO entries not sorted by row at entry " + std::to_string(e);
      if (row[e] == row[e - 1] && col[e] <= col[e - 1])
        return "columns not strictly increasing within a row at entry " + std::to_string(e);
    }
  }
  return "";
}

int64_t hyb_K(int64_t m, const int64_t* row_ptr) {
  // K = min{k >= 0 : 3 * #{rows with len > k} < m}   (reading R12)
  if (m <= 0) return 0;
  int64_t maxlen = 0;
  for (int64_t i = 0; i < m; ++i) maxlen = std::max(maxlen, row_ptr[i + 1] - row_ptr[i]);
  std::vector<int64_t> hist(maxlen + 1, 0);
  for (int64_t i = 0; i < m; ++i) hist[row_ptr[i + 1] - row_ptr[i]]++;
  int64_t at_most = 0;
  for (int64_t k = 0; k <= maxlen; ++k) {
    at_most += hist[k];
    if (3 * (m - at_most) < m) return k;
  }
  return maxlen;
}

// ---------------------------------------------------------------------------
// BRO-ELL
// ---------------------------------------------------------------------------

// MSB-first bit writer that emits 32-bit symbols to words[place(lane, q, S, V, h)].
struct SymbolWriter {
  uint32_t* words;
  int64_t lane, S, V, h;
  uint64_t acc = 0;
  int nb = 0;
  int64_t q = 0;
  void put(uint32_t v, int b) {
    if (b == 0) return;
    acc = (acc << b) | v;
    nb += b;
    if (nb >= 32) {
      nb -= 32;
      words[place(lane, q++, S, V, h)] = uint32_t(acc >> nb);
      acc &= (nb ? ((uint64_t(1) << nb) - 1) : 0);
    }
  }
  void flush() {  // append the padding bits b_p (zeros) of P:L114
    if (nb > 0) {
      words[place(lane, q++, S, V, h)] = uint32_t(acc << (32 - nb));
      nb = 0;
      acc = 0;
    }
  }
};

void encode_bro_ell(const RowsView& A, int h, int V, int VV, int min_bits, EllCode& out) {
  const int64_t m = A.m;
  const int64_t s = (m + h - 1) / h;
  out.h = h;
  out.s = s;
  std::vector<uint64_t> ncol(s, 0), nsym(s, 0);
  // num_col: l_t = longest row of the slice (R9)
  parallel_for(s, [&](int64_t lo, int64_t hi) {
    for (int64_t t = lo; t < hi; ++t) {
      int64_t l = 0;
      for (int64_t r = t * h; r < std::min(m, t * h + h); ++r) l = std::max(l, A.len(r));
      ncol[t] = (uint64_t)l;
    }
  });
  exclusive_scan(ncol, out.colptr);
  out.max_l = s ? (int64_t)*std::max_element(ncol.begin(), ncol.end()) : 0;
  out.bit_alloc.assign(out.colptr[s], 0);
  // bit_alloc: b_j = max over rows of Gamma(delta_j)
  parallel_for(s, [&](int64_t lo, int64_t hi) {
    for (int64_t t = lo; t < hi; ++t) {
      uint8_t* ba = out.bit_alloc.data() + out.colptr[t];
      for (int64_t r = t * h; r < std::min(m, t * h + h); ++r) {
        const int32_t* c = A.col + A.row_ptr[r];
        const int64_t len = A.len(r);
        uint32_t prev1 = 0;  // 1-based previous column, c_{-1} = 0
        for (int64_t j = 0; j < len; ++j) {
          uint32_t c1 = uint32_t(c[j]) + 1u;
          int g = gamma_bits(c1 - prev1);
          if (g > ba[j]) ba[j] = (uint8_t)g;
          prev1 = c1;
        }
      }
      uint64_t L = 0;
      for (uint64_t j = 0; j < ncol[t]; ++j) {
        if (ba[j] < min_bits) ba[j] = (uint8_t)min_bits;  // forced widths (Fig. 3)
        L += ba[j];
      }
      nsym[t] = (L + kSym - 1) / kSym;
    }
  });
  exclusive_scan(nsym, out.symptr);
  out.words.assign(size_t(h) * out.symptr[s], 0u);
  out.vals.resize(size_t(h) * out.colptr[s] * A.vsize);
  // pack + multiplex and place values slot-wise
  parallel_for(s, [&](int64_t lo, int64_t hi) {
    for (int64_t t = lo; t < hi; ++t) {
      const uint8_t* ba = out.bit_alloc.data() + out.colptr[t];
      const int64_t l = (int64_t)ncol[t], S = (int64_t)nsym[t];
      uint32_t* wbase = out.words.data() + size_t(h) * out.symptr[t];
      uint8_t* vbase = out.vals.data() + size_t(h) * out.colptr[t] * A.vsize;
      for (int64_t lane = 0; lane < h; ++lane) {
        const int64_t r = t * h + lane;
        const int64_t len = r < m ? A.len(r) : 0;
        const int32_t* c = r < m ? A.col + A.row_ptr[r] : nullptr;
        SymbolWriter w{wbase, lane, S, V, h};
        uint32_t prev1 = 0;
        for (int64_t j = 0; j < l; ++j) {
          uint32_t d = 0;  // 0 = invalid (padding)
          if (j < len) {
            uint32_t c1 = uint32_t(c[j]) + 1u;
            d = c1 - prev1;
            prev1 = c1;
          }
          w.put(d, ba[j]);
        }
        w.flush();
        if (r < m) {
          const uint8_t* src = A.vals + size_t(A.row_ptr[r]) * A.vsize;
          for (int64_t j = 0; j < len; ++j)
            std::memcpy(vbase + size_t(place(lane, j, l, VV, h)) * A.vsize, src + size_t(j) * A.vsize, A.vsize);
        }
      }
    }
  });
}

template <typename U>
static int value_index_impl(const RowsView& A, const EllCode& E, ValueIndexCode& out) {
  constexpr size_t kMaxD = 65536;
  const int64_t m = A.m;
  const int nt = num_threads();
  // distinct bit patterns per thread (early exit past 65,536), then merged
  std::vector<std::unordered_set<U>> sets(nt);
  std::vector<char> over(nt, 0);
  {
    std::vector<std::thread> th;
    for (int c = 0; c < nt; ++c) {
      th.emplace_back([&, c] {
        const int64_t lo = m * c / nt, hi = m * (c + 1) / nt;
        auto& st = sets[c];
        for (int64_t r = lo; r < hi && !over[c]; ++r) {
          const U* v = reinterpret_cast<const U*>(A.vals) + A.row_ptr[r];
          for (int64_t j = 0, len = A.len(r); j < len; ++j) st.insert(v[j]);
          if (st.size() > kMaxD) over[c] = 1;
        }
      });
    }
    for (auto& t : th) t.join();
  }
  std::unordered_set<U> all;
  for (int c = 0; c < nt; ++c) {
    if (over[c]) return 1;
    all.insert(sets[c].begin(), sets[c].end());
    if (all.size() > kMaxD) return 1;
  }
  std::vector<U> D(all.begin(), all.end());
  std::sort(D.begin(), D.end());  // ascending as unsigned integers
  // padding code: the first finite value (exponent field not all ones)
  constexpr U kExp = sizeof(U) == 8 ? U(0x7FF0000000000000ull) : U(0x7F800000u);
  size_t pz = 0;
  while (pz < D.size() && (D[pz] & kExp) == kExp) ++pz;
  if (!D.empty() && pz == D.size()) return 2;
  if (D.empty()) pz = 0;
  const int cb = D.size() <= 256 ? 1 : 2;
  const int64_t VC = 4 / cb;
  const int64_t h = E.h, s = E.s;
  out.cb = cb;
  out.nd = int64_t(D.size());
  out.pz = uint32_t(pz);
  out.dict.resize(D.size() * sizeof(U));
  if (!D.empty()) std::memcpy(out.dict.data(), D.data(), D.size() * sizeof(U));
  out.codes.assign(size_t(cb) * h * E.colptr[s], 0);
  for (size_t i = 0; i < out.codes.size(); i += size_t(cb)) {  // every slot starts as padding
    out.codes[i] = uint8_t(pz);
    if (cb == 2) out.codes[i + 1] = uint8_t(pz >> 8);
  }
  parallel_for(s, [&](int64_t lo, int64_t hi) {
    for (int64_t t = lo; t < hi; ++t) {
      const int64_t l = int64_t(E.colptr[t + 1] - E.colptr[t]);
      uint8_t* base = out.codes.data() + size_t(cb) * h * E.colptr[t];
      for (int64_t lane = 0; lane < h; ++lane) {
        const int64_t r = t * h + lane;
        if (r >= m) break;
        const U* v = reinterpret_cast<const U*>(A.vals) + A.row_ptr[r];
        for (int64_t j = 0, len = A.len(r); j < len; ++j) {
          const uint32_t code = uint32_t(std::lower_bound(D.begin(), D.end(), v[j]) - D.begin());
          uint8_t* dst = base + size_t(cb) * place(lane, j, l, VC, h);
          dst[0] = uint8_t(code);
          if (cb == 2) dst[1] = uint8_t(code >> 8);
        }
      }
    }
  });
  return 0;
}

int encode_value_index(const RowsView& A, const EllCode& E, ValueIndexCode& out) {
  return A.vsize == 8 ? value_index_impl<uint64_t>(A, E, out) : value_index_impl<uint32_t>(A, E, out);
}

void slice_extents(const RowsView& A, int h, int min_bits, int64_t* max_l, int64_t* max_S) {
  const int64_t m = A.m;
  const int64_t s = (m + h - 1) / h;
  const int nt = num_threads();
  std::vector<int64_t> ml(nt, 0), ms(nt, 0);
  std::vector<std::thread> th;
  for (int c = 0; c < nt; ++c) {
    th.emplace_back([&, c] {
      std::vector<uint8_t> ba;
      for (int64_t t = s * c / nt; t < s * (c + 1) / nt; ++t) {
        int64_t l = 0;
        for (int64_t r = t * h; r < std::min(m, t * h + h); ++r) l = std::max(l, A.len(r));
        ba.assign(l, 0);
        for (int64_t r = t * h; r < std::min(m, t * h + h); ++r) {
          const int32_t* col = A.col + A.row_ptr[r];
          uint32_t prev1 = 0;
          for (int64_t j = 0; j < A.len(r); ++j) {
            const uint32_t c1 = uint32_t(col[j]) + 1u;
            ba[j] = std::max<uint8_t>(ba[j], uint8_t(gamma_bits(c1 - prev1)));
            prev1 = c1;
          }
        }
        int64_t L = 0;
        for (int64_t j = 0; j < l; ++j) L += std::max<int>(ba[j], min_bits);
        ml[c] = std::max(ml[c], l);
        ms[c] = std::max(ms[c], (L + kSym - 1) / kSym);
      }
    });
  }
  for (auto& t : th) t.join();
  *max_l = *std::max_element(ml.begin(), ml.end());
  *max_S = *std::max_element(ms.begin(), ms.end());
}

void build_plain_ell(const RowsView& A, int64_t K, PlainEll& out) {
  out.K = K;
  out.pitch = (A.m + kH - 1) / kH * kH;
  out.col.assign(size_t(K) * out.pitch, -1);
  out.vals.resize(size_t(K) * out.pitch * A.vsize);
  parallel_for(A.m, [&](int64_t lo, int64_t hi) {
    for (int64_t r = lo; r < hi; ++r) {
      const int64_t len = std::min<int64_t>(A.len(r), K);
      for (int64_t j = 0; j < len; ++j) {
        const size_t slot = size_t(j) * out.pitch + r;
        out.col[slot] = A.col[A.row_ptr[r] + j];
        std::memcpy(out.vals.data() + slot * A.vsize, A.vals + size_t(A.row_ptr[r] + j) * A.vsize, A.vsize);
      }
    }
  }, 4096);
}

// ---------------------------------------------------------------------------
// BRO-COO (reading R13: lane l of interval i owns the T consecutive entries
// e = i*32T + T*l + t; deltas in entry order, one width per interval)
// ---------------------------------------------------------------------------

// Lane-contiguous, chunk-multiplexed copy of per-entry arrays (reading R26):
// entry (l, t) of interval i at i*32T + place(l, t, T, chunk); `fill` past nnz.
template <class E>
static void arrange(int64_t nnz, int T, int chunk, const E* src, E fill, int esize, uint8_t* dst, int64_t nI) {
  const int64_t I = int64_t(kH) * T;
  parallel_for(nI, [&](int64_t lo, int64_t hi) {
    for (int64_t i = lo; i < hi; ++i)
      for (int lane = 0; lane < kH; ++lane)
        for (int t = 0; t < T; ++t) {
          const int64_t e = i * I + int64_t(T) * lane + t;
          uint8_t* d = dst + size_t(i * I + place(lane, t, T, chunk)) * esize;
          if (e < nnz) std::memcpy(d, reinterpret_cast<const uint8_t*>(src) + size_t(e) * esize, esize);
          else std::memcpy(d, &fill, esize);
        }
  }, 64);
}

static void arrange_col_vals(int64_t nnz, const int32_t* col, const uint8_t* vals, int vsize, int T,
                             CooCode& out) {
  const int64_t slots = out.nI * int64_t(kH) * T;
  out.col.assign(slots, 0);
  out.vals.resize(size_t(slots) * vsize);
  arrange<int32_t>(nnz, T, 4, col, 0, 4, reinterpret_cast<uint8_t*>(out.col.data()), out.nI);
  if (vsize == 8) arrange<double>(nnz, T, 2, reinterpret_cast<const double*>(vals), 0.0, 8, out.vals.data(), out.nI);
  else arrange<float>(nnz, T, 4, reinterpret_cast<const float*>(vals), 0.0f, 4, out.vals.data(), out.nI);
}

void encode_bro_coo(int64_t nnz, const int32_t* row, const int32_t* col, const uint8_t* vals,
                    int vsize, int T, int V, CooCode& out) {
  const int64_t I = int64_t(kH) * T;
  const int64_t nI = (nnz + I - 1) / I;
  out.T = T;
  out.nnz = nnz;
  out.nI = nI;
  out.base_row.assign(nI, 0);
  out.width.assign(nI, 0);
  std::vector<uint64_t> nsym(nI, 0);
  auto at = [&](int64_t e) { return (uint32_t)row[std::min(e, nnz - 1)]; };
  parallel_for(nI, [&](int64_t lo, int64_t hi) {
    for (int64_t i = lo; i < hi; ++i) {
      const uint32_t base = at(i * I);
      uint32_t dmax = 0, prev = base;
      for (int64_t e = i * I; e < (i + 1) * I; ++e) {  // entry order = lane-major
        const uint32_t r = at(e);
        dmax = std::max(dmax, r - prev);
        prev = r;
      }
      out.base_row[i] = base;
      out.width[i] = (uint8_t)gamma_bits(dmax);  // one width per interval
      nsym[i] = (uint64_t(T) * out.width[i] + kSym - 1) / kSym;
    }
  });
  exclusive_scan(nsym, out.symptr);
  out.words.assign(kH * out.symptr[nI], 0u);
  parallel_for(nI, [&](int64_t lo, int64_t hi) {
    for (int64_t i = lo; i < hi; ++i) {
      const int b = out.width[i];
      const int64_t S = (int64_t)nsym[i];
      uint32_t* wbase = out.words.data() + kH * out.symptr[i];
      uint32_t prev = out.base_row[i];
      for (int lane = 0; lane < kH; ++lane) {
        SymbolWriter w{wbase, lane, S, V, kH};
        for (int t = 0; t < T; ++t) {
          const uint32_t r = at(i * I + int64_t(T) * lane + t);
          w.put(r - prev, b);
          prev = r;
        }
        w.flush();
      }
    }
  });
  arrange_col_vals(nnz, col, vals, vsize, T, out);
}

void build_plain_coo(int64_t nnz, const int32_t* row, const int32_t* col, const uint8_t* vals,
                     int vsize, int T, CooCode& out) {
  const int64_t I = int64_t(kH) * T;
  out.T = T;
  out.nnz = nnz;
  out.nI = (nnz + I - 1) / I;
  out.base_row.assign(out.nI, 0);
  for (int64_t i = 0; i < out.nI; ++i) out.base_row[i] = (uint32_t)row[i * I];
  out.row.assign(out.nI * I, 0);
  arrange<int32_t>(nnz, T, 4, row, nnz ? row[nnz - 1] : 0, 4, reinterpret_cast<uint8_t*>(out.row.data()), out.nI);
  arrange_col_vals(nnz, col, vals, vsize, T, out);
}

// ---------------------------------------------------------------------------
// BAR: BRO-aware reordering
// ---------------------------------------------------------------------------

// Method 0 ("signature clustering"): stable order by
// (row length, jump mask, first column, row id), where bit j >= 1 of the
// jump mask is set when Gamma(delta_j) > 2.  Rows with equal length and
// jump positions have equal bit allocation patterns up to the jump widths,
// which is what Eqn (2)'s d(S, j) rewards; ordering by first column inside a
// group keeps x cachelines shared (Eqn (3)'s c(S, j)).
void bar_signature_order(int64_t m, const int64_t* row_ptr, const int32_t* col, int64_t* perm) {
  std::vector<uint64_t> moff(m + 1, 0);
  for (int64_t i = 0; i < m; ++i) moff[i + 1] = moff[i] + uint64_t((row_ptr[i + 1] - row_ptr[i] + 63) / 64);
  std::vector<uint64_t> mask(moff[m], 0);
  parallel_for(m, [&](int64_t lo, int64_t hi) {
    for (int64_t i = lo; i < hi; ++i) {
      uint64_t* mk = mask.data() + moff[i];
      for (int64_t p = row_ptr[i] + 1; p < row_ptr[i + 1]; ++p) {
        int64_t j = p - row_ptr[i];
        uint32_t d = uint32_t(col[p]) - uint32_t(col[p - 1]);
        if (gamma_bits(d) > 2) mk[j / 64] |= uint64_t(1) << (63 - (j % 64));
      }
    }
  }, 4096);
  std::vector<int64_t> idx(m);
  std::iota(idx.begin(), idx.end(), 0);
  auto less = [&](int64_t a, int64_t b) {
    const int64_t la = row_ptr[a + 1] - row_ptr[a], lb = row_ptr[b + 1] - row_ptr[b];
    if (la != lb) return la < lb;
    for (uint64_t w = 0; w < moff[a + 1] - moff[a]; ++w) {
      uint64_t x = mask[moff[a] + w], y = mask[moff[b] + w];
      if (x != y) return x < y;
    }
    const int64_t fa = la ? col[row_ptr[a]] : -1, fb = lb ? col[row_ptr[b]] : -1;
    if (fa != fb) return fa < fb;
    return a < b;
  };
  std::sort(idx.begin(), idx.end(), less);
  std::copy(idx.begin(), idx.end(), perm);
}

// Method 1: Algorithm 2 — greedy clustering on Eqn (1):
//   Phi = sum_i h/w * ( ceil(sum_j d(S_i, j) / alpha) + sum_j c(S_i, j) )
// with h = w = 32 (factor 1, R21), alpha = sym_len = 32, d(S,j) = max Gamma
// of the j-th deltas (Eqn 2), c(S,j) = number of distinct 128-byte lines of x
// touched by the j-th columns (Eqn 3, reading R20).  Adding row r to S_p
// changes only S_p's term, so argmin_p Phi_p = argmin_p DeltaPhi_p; ties go
// to the lowest p and full partitions are skipped (R22).
bool bar_greedy_order(int64_t m, int64_t n, const int64_t* row_ptr, const int32_t* col, int vsize,
                      int64_t* perm, std::string* err) {
  (void)n;
  const int64_t h = kH;
  if (m > 65536) {
    if (err) *err = "Algorithm 2 is O(m^2 k / h); limited to m <= 65536";
    return false;
  }
  if (m == 0) return true;
  const int64_t v = (m + h - 1) / h;
  auto cap = [&](int64_t p) { return p < v - 1 ? h : m - (v - 1) * h; };
  int64_t kmax = 0;
  for (int64_t i = 0; i < m; ++i) kmax = std::max(kmax, row_ptr[i + 1] - row_ptr[i]);
  // per-row deltas' Gamma and x lines
  auto gam = [&](int64_t i, int64_t j) -> int {
    const int64_t p = row_ptr[i] + j;
    uint32_t c1 = uint32_t(col[p]) + 1u;
    uint32_t prev = j ? uint32_t(col[p - 1]) + 1u : 0u;
    return gamma_bits(c1 - prev);
  };
  auto line = [&](int64_t i, int64_t j) -> int64_t { return int64_t(col[row_ptr[i] + j]) * vsize / 128; };
  std::vector<std::vector<uint8_t>> d(v, std::vector<uint8_t>(kmax, 0));
  std::vector<int64_t> dsum(v, 0);
  std::vector<std::vector<std::unordered_set<int64_t>>> lines(v, std::vector<std::unordered_set<int64_t>>(kmax));
  std::vector<std::vector<int64_t>> S(v);
  auto insert = [&](int64_t p, int64_t i) {
    const int64_t len = row_ptr[i + 1] - row_ptr[i];
    for (int64_t j = 0; j < len; ++j) {
      int g = gam(i, j);
      if (g > d[p][j]) { dsum[p] += g - d[p][j]; d[p][j] = (uint8_t)g; }
      lines[p][j].insert(line(i, j));
    }
    S[p].push_back(i);
  };
  // line 2: sort rows by row length (ascending, stable)
  std::vector<int64_t> D(m);
  std::iota(D.begin(), D.end(), 0);
  std::stable_sort(D.begin(), D.end(), [&](int64_t a, int64_t b) {
    return row_ptr[a + 1] - row_ptr[a] < row_ptr[b + 1] - row_ptr[b];
  });
  // lines 3-6: seed S_t with r_{(t-1)h+1}
  std::vector<char> used(m, 0);
  for (int64_t t = 0; t < v; ++t) {
    insert(t, D[t * h]);
    used[t * h] = 1;
  }
  // lines 7-13
  const int64_t alpha = kSym;
  for (int64_t pos = 0; pos < m; ++pos) {
    if (used[pos]) continue;
    const int64_t i = D[pos];
    const int64_t len = row_ptr[i + 1] - row_ptr[i];
    int64_t best = -1, bestc = 0;
    for (int64_t p = 0; p < v; ++p) {
      if ((int64_t)S[p].size() >= cap(p)) continue;
      int64_t nd = dsum[p];
      int64_t dc = 0;
      for (int64_t j = 0; j < len; ++j) {
        int g = gam(i, j);
        if (g > d[p][j]) nd += g - d[p][j];
        if (!lines[p][j].count(line(i, j))) dc++;
      }
      const int64_t delta = (nd + alpha - 1) / alpha - (dsum[p] + alpha - 1) / alpha + dc;
      if (best < 0 || delta < bestc) { best = p; bestc = delta; }
    }
    insert(best, i);
  }
  int64_t k = 0;
  for (int64_t p = 0; p < v; ++p)
    for (int64_t i : S[p]) perm[k++] = i;
  return true;
}

}  // namespace bro

namespace bro {

// Method 2: Algorithm 2 with a candidate window (reading R24), for
// matrices too large for the O(m^2 k / h) exact greedy.  Lines 1-6 as in
// method 1.  For the row at position pos of the sorted sequence D, line 11's
// argmin runs only over the W non-full partitions nearest to the row's own
// partition c = min(pos / h, v - 1) (nearest by |p - c|, equal distance ->
// lower p); cost ties -> lowest p.  With W >= v every non-full partition is a
// candidate and the result is exactly method 1.  Per partition: the column
// widths d(S, j) (Eqn 2) and the distinct x lines of each column (Eqn 3, at
// most h per column), grown to the partition's longest row.  Full partitions
// are skipped with two path-compressed "next non-full" forests.
bool bar_window_order(int64_t m, const int64_t* row_ptr, const int32_t* col, int vsize, int W,
                      int64_t* perm, const int64_t* seed_order) {
  const int64_t h = kH;
  if (m == 0) return true;
  if (W < 1) W = 1;
  const int64_t v = (m + h - 1) / h;
  auto cap = [&](int64_t p) { return p < v - 1 ? h : m - (v - 1) * h; };
  struct Part {
    std::vector<uint8_t> d;      // d(S, j)
    std::vector<uint8_t> nl;     // distinct lines in column j
    std::vector<int32_t> lines;  // column j's lines at [32 j, 32 j + nl[j])
    int64_t dsum = 0;
    int size = 0;
  };
  std::vector<Part> P(v);
  std::vector<std::vector<int64_t>> S(v);
  std::vector<int> g;       // the current row's Gamma(delta_j)
  std::vector<int32_t> ln;  // the current row's x lines
  auto load_row = [&](int64_t i) {
    const int64_t len = row_ptr[i + 1] - row_ptr[i];
    g.resize(len);
    ln.resize(len);
    uint32_t prev = 0;
    for (int64_t j = 0; j < len; ++j) {
      const uint32_t c1 = uint32_t(col[row_ptr[i] + j]) + 1u;
      g[j] = gamma_bits(c1 - prev);
      prev = c1;
      ln[j] = int32_t(int64_t(col[row_ptr[i] + j]) * vsize / 128);
    }
    return len;
  };
  auto has_line = [&](const Part& q, int64_t j, int32_t L) {
    const int32_t* a = q.lines.data() + 32 * j;
    for (int k = 0; k < q.nl[j]; ++k)
      if (a[k] == L) return true;
    return false;
  };
  auto insert = [&](int64_t p, int64_t i) {
    const int64_t len = load_row(i);
    Part& q = P[p];
    if ((int64_t)q.d.size() < len) {
      q.d.resize(len, 0);
      q.nl.resize(len, 0);
      q.lines.resize(32 * len, 0);
    }
    for (int64_t j = 0; j < len; ++j) {
      if (g[j] > q.d[j]) { q.dsum += g[j] - q.d[j]; q.d[j] = (uint8_t)g[j]; }
      if (!has_line(q, j, ln[j])) q.lines[32 * j + q.nl[j]++] = ln[j];
    }
    q.size++;
    S[p].push_back(i);
  };
  // next non-full partition at or right of p (v if none) / at or left of p (-1 if none)
  std::vector<int64_t> rpar(v + 1), lpar(v + 1);
  std::iota(rpar.begin(), rpar.end(), 0);
  std::iota(lpar.begin(), lpar.end(), 0);  // lpar index shifted by one: slot p + 1 <-> partition p
  auto rfind = [&](int64_t p) {
    int64_t r = p;
    while (rpar[r] != r) r = rpar[r];
    while (rpar[p] != r) { int64_t nx = rpar[p]; rpar[p] = r; p = nx; }
    return r;
  };
  auto lfind = [&](int64_t p) {  // p in [-1, v)
    int64_t s = p + 1, r = s;
    while (lpar[r] != r) r = lpar[r];
    while (lpar[s] != r) { int64_t nx = lpar[s]; lpar[s] = r; s = nx; }
    return r - 1;
  };
  auto mark_full = [&](int64_t p) { rpar[p] = p + 1; lpar[p + 1] = p; };
  // line 2 (seed_order: the row sequence to use instead, reading R27)
  std::vector<int64_t> D(m);
  if (seed_order) {
    std::copy(seed_order, seed_order + m, D.begin());
  } else {
    std::iota(D.begin(), D.end(), 0);
    std::stable_sort(D.begin(), D.end(), [&](int64_t a, int64_t b) {
      return row_ptr[a + 1] - row_ptr[a] < row_ptr[b + 1] - row_ptr[b];
    });
  }
  // lines 3-6
  for (int64_t t = 0; t < v; ++t) {
    insert(t, D[t * h]);
    if (P[t].size >= cap(t)) mark_full(t);
  }
  const int64_t alpha = kSym;
  std::vector<int64_t> cand;
  for (int64_t pos = 0; pos < m; ++pos) {
    if (pos % h == 0) continue;  // a seed
    const int64_t i = D[pos];
    const int64_t len = load_row(i);
    const int64_t c = std::min(pos / h, v - 1);
    cand.clear();
    int64_t r = rfind(c), l = lfind(c - 1);
    while ((int64_t)cand.size() < W && (l >= 0 || r < v)) {
      if (l >= 0 && (r >= v || c - l <= r - c)) { cand.push_back(l); l = lfind(l - 1); }
      else { cand.push_back(r); r = rfind(r + 1); }
    }
    int64_t best = -1, bestc = 0;
    for (int64_t p : cand) {
      const Part& q = P[p];
      int64_t nd = q.dsum, dc = 0;
      for (int64_t j = 0; j < len; ++j) {
        const int dj = j < (int64_t)q.d.size() ? q.d[j] : 0;
        if (g[j] > dj) nd += g[j] - dj;
        if (j >= (int64_t)q.d.size() || !has_line(q, j, ln[j])) dc++;
      }
      const int64_t delta = (nd + alpha - 1) / alpha - (q.dsum + alpha - 1) / alpha + dc;
      if (best < 0 || delta < bestc || (delta == bestc && p < best)) { best = p; bestc = delta; }
    }
    insert(best, i);
    if (P[best].size >= cap(best)) mark_full(best);
  }
  int64_t k = 0;
  for (int64_t p = 0; p < v; ++p)
    for (int64_t i : S[p]) perm[k++] = i;
  return true;
}

}  // namespace bro
