// Host-side BRO encoder and layout builder (offline compression).
// Shares no code with oracle/; both follow DESIGN.md "Encoded layout".
#pragma once
#include <cstdint>
#include <string>
#include <vector>

namespace bro {

constexpr int kH = 32;        // warp size: BRO-COO lanes per interval, BAR partition height
constexpr int kSym = 32;      // sym_len in bits
// BRO-ELL slice height h (P:L105 makes it a parameter; reading R10): 32 (one
// row per lane of a warp) or 64 (two rows per lane)

// Bytes of one value type.
struct Bytes {
  std::vector<uint8_t> v;
  void resize(size_t n) { v.assign(n, 0); }
  uint8_t* data() { return v.data(); }
  const uint8_t* data() const { return v.data(); }
  size_t size() const { return v.size(); }
};

// View of the rows that go into an ELL-type part: row i holds the first
// min(len_i, cap) entries of CSR row i.
struct RowsView {
  int64_t m = 0;
  const int64_t* row_ptr = nullptr;
  const int32_t* col = nullptr;
  const uint8_t* vals = nullptr;  // raw value bytes
  int vsize = 8;                  // bytes per value
  int64_t cap = INT64_MAX;        // ELL width bound K
  int64_t len(int64_t i) const {
    int64_t l = row_ptr[i + 1] - row_ptr[i];
    return l < cap ? l : cap;
  }
};

struct EllCode {                  // BRO-ELL
  int h = 32;                     // slice height
  int64_t s = 0;                  // slices
  std::vector<uint64_t> colptr;   // s+1
  std::vector<uint64_t> symptr;   // s+1
  std::vector<uint8_t> bit_alloc; // colptr[s]
  std::vector<uint32_t> words;    // h*symptr[s]
  Bytes vals;                     // h*colptr[s] values
  int64_t max_l = 0;              // max num_col over slices
};

// BRO-COO (reading R13) or plain COO: intervals of 32*T
// entries, lane l owning the T consecutive entries i*32T + T*l + t; col,
// vals (and plain rows) stored lane-contiguously in 16-byte chunks
// (reading R26): entry (l, t) at i*32T + place(l, t, T, chunk).
struct CooCode {
  int T = 32;
  int64_t nnz = 0, nI = 0;
  std::vector<uint32_t> base_row; // nI
  std::vector<uint8_t> width;     // nI
  std::vector<uint64_t> symptr;   // nI+1
  std::vector<uint32_t> words;    // 32*symptr[nI]
  std::vector<int32_t> row;       // plain COO only, nI*32T
  std::vector<int32_t> col;       // nI*32T
  Bytes vals;                     // nI*32T
};

// Value index of a BRO-ELL part (reading R28: the value compression of
// P:L416 by the value-index method of [16]): the distinct bit
// patterns of the stored values, sorted as unsigned integers, and one code of
// cb bytes per slot, slot (r, j) of slice t at h*colptr[t] + place(r, j, l_t,
// 4/cb, h) (padding 0).
struct ValueIndexCode {
  int cb = 0;                     // 1 or 2 bytes per code
  int64_t nd = 0;                 // |D|
  uint32_t pz = 0;                // padding code: the first finite value of D (reading R28)
  Bytes dict;                     // nd values (bit patterns ascending)
  std::vector<uint8_t> codes;     // cb*h*colptr[s] bytes, little-endian codes
};

struct PlainEll {                 // ELLPACK, column-major
  int64_t K = 0, pitch = 0;
  std::vector<int32_t> col;       // K*pitch, -1 = padding
  Bytes vals;                     // K*pitch
};

// Position of item q of row r in a block of h rows x S items grouped in
// chunks of V (tail chunk S - V*floor(S/V)).
inline int64_t place(int64_t r, int64_t q, int64_t S, int64_t V, int64_t h = kH) {
  const int64_t F = S / V;
  const int64_t c = q / V;
  if (c < F) return h * V * c + r * V + (q - c * V);
  return h * V * F + r * (S - V * F) + (q - V * F);
}

inline int gamma_bits(uint32_t u) { return u ? 32 - __builtin_clz(u) : 0; }

// Validation of canonical CSR; returns "" if fine, else a message.
std::string check_csr(int64_t m, int64_t n, const int64_t* row_ptr, const int32_t* col);
std::string check_coo(int64_t m, int64_t n, int64_t nnz, const int32_t* row, const int32_t* col);

int64_t hyb_K(int64_t m, const int64_t* row_ptr);

void encode_bro_ell(const RowsView& A, int h, int V, int value_chunk, int min_bits, EllCode& out);
// Value index of the BRO-ELL part E of A: 0 = done, 1 = more than 65,536
// distinct values, 2 = no finite value (out untouched unless 0).
int encode_value_index(const RowsView& A, const EllCode& E, ValueIndexCode& out);
// Longest slice (columns) and longest row stream (32-bit symbols) of the
// BRO-ELL encoding at slice height h, without packing anything.
void slice_extents(const RowsView& A, int h, int min_bits, int64_t* max_l, int64_t* max_S);
void build_plain_ell(const RowsView& A, int64_t K, PlainEll& out);
// rows: int32 rows of the COO entries (sorted); T steps per interval.
void encode_bro_coo(int64_t nnz, const int32_t* row, const int32_t* col, const uint8_t* vals,
                    int vsize, int T, int V, CooCode& out);
void build_plain_coo(int64_t nnz, const int32_t* row, const int32_t* col, const uint8_t* vals,
                     int vsize, int T, CooCode& out);

// BAR reordering
void bar_signature_order(int64_t m, const int64_t* row_ptr, const int32_t* col, int64_t* perm);
bool bar_window_order(int64_t m, const int64_t* row_ptr, const int32_t* col, int vsize, int W,
                      int64_t* perm, const int64_t* seed_order = nullptr);
bool bar_greedy_order(int64_t m, int64_t n, const int64_t* row_ptr, const int32_t* col, int vsize,
                      int64_t* perm, std::string* err);

int num_threads();

}  // namespace bro
