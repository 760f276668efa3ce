// C ABI of libbro.so (include/bro.h): validation, host encode, upload, launch.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <climits>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <type_traits>

#include "../../include/bro.h"
#include "encode.hpp"
#include "kernels.cuh"

namespace {

thread_local std::string g_err;

bro_status_t fail(bro_status_t s, const std::string& msg) {
  g_err = msg;
  return s;
}

constexpr int kCooThreads = 256;
constexpr int kE2eChunks = 8;  // pieces of the pipelined bro_spmv_host
// below this x size the pieces' launch and event overheads exceed the copy
// time they hide (C1/C2 e2e: 1.3 -> 0.5 and 63 -> 57 GFLOP/s when pipelined)
constexpr size_t kE2eMinBytes = size_t(4) << 20;
constexpr int kBarWindow = 64;  // candidate partitions of BAR method 2 (windowed Algorithm 2)
constexpr int kCooMaxUpi = 4;   // work units per COO interval (8 steps = 256 entries each at 4)
constexpr int kCooUpi = 2;
constexpr int kPlainThreads = 256;

struct DeviceGuard {
  int prev = -1, want = -1;
  explicit DeviceGuard(int d) : want(d) {
    cudaGetDevice(&prev);
    if (prev != d) cudaSetDevice(d);
  }
  ~DeviceGuard() {
    if (prev >= 0 && prev != want) cudaSetDevice(prev);
  }
};

enum Format { FMT_ELL = 0, FMT_COO = 1, FMT_HYB = 2 };

}  // namespace

struct bro_matrix_s {
  int device = -1;
  bool host_only = false;
  bro_dtype_t dtype = BRO_FP64;
  int vsize = 8;
  bro_opts_t opts{};
  int format = FMT_ELL;
  int64_t m = 0, n = 0, nnz = 0, K = 0, nnz_ell = 0, nnz_coo = 0;
  bool has_ell = false, has_coo = false;
  // host encodings (kept only by host-only handles after create)
  bro::EllCode ell;
  bro::PlainEll pell;
  bro::CooCode coo;
  int64_t s = 0, ell_words = 0, ell_slots = 0, pitch = 0, nI = 0, coo_words = 0;
  // device buffers
  uint32_t* d_words = nullptr;
  uint8_t* d_bit_alloc = nullptr;
  uint64_t* d_colptr = nullptr;
  uint64_t* d_symptr = nullptr;
  void* d_ell_vals = nullptr;
  int32_t* d_pell_col = nullptr;
  uint32_t* d_coo_words = nullptr;
  uint32_t* d_coo_base = nullptr;
  uint8_t* d_coo_width = nullptr;
  uint64_t* d_coo_symptr = nullptr;
  int32_t* d_coo_row = nullptr;
  int32_t* d_coo_col = nullptr;
  void* d_coo_vals = nullptr;
  void* d_cf = nullptr;
  void* d_cl = nullptr;
  int32_t* d_last_row = nullptr;
  int32_t* d_first_row = nullptr;
  void* d_xs = nullptr;
  void* d_ys = nullptr;
  int64_t device_bytes = 0;
  uint32_t bulk_unit_max = 0;
  // end-to-end pipeline of ELL-only handles (bro_spmv_host): column range of
  // every 32-row block, side streams and events (created on first use)
  std::vector<int32_t> blk_cmin, blk_cmax;
  cudaStream_t e2e_h2d = nullptr, e2e_d2h = nullptr;
  std::vector<cudaEvent_t> e2e_ev;
  int64_t ell_max_S = 0;       // most 32-bit symbols in one BRO-ELL row stream
  int64_t ell_max_l = 0;       // longest BRO-ELL slice (columns)  // largest staged slice of the bulk BRO-ELL kernel (bytes)
  bro_info_t info{};
};

namespace {

template <typename P>
bro_status_t dev_upload(bro_matrix_s* A, P** dst, const void* src, size_t bytes) {
  *dst = nullptr;
  if (bytes == 0) return BRO_OK;
  void* p = nullptr;
  // every array carries kStreamPad zeroed bytes past its end: the kernels'
  // 16-byte chunk loads may be issued speculatively (see kernels.cuh "loads")
  const size_t pad = bro::dev::kStreamPad;
  cudaError_t e = cudaMalloc(&p, bytes + pad);
  if (e != cudaSuccess) return fail(BRO_ERR_OOM, std::string("cudaMalloc: ") + cudaGetErrorString(e));
  A->device_bytes += (int64_t)(bytes + pad);
  *dst = static_cast<P*>(p);
  if (src) {
    e = cudaMemcpy(p, src, bytes, cudaMemcpyHostToDevice);
    if (e != cudaSuccess) return fail(BRO_ERR_CUDA, std::string("cudaMemcpy H2D: ") + cudaGetErrorString(e));
  }
  e = cudaMemset(static_cast<char*>(p) + bytes, 0, pad);
  if (e != cudaSuccess) return fail(BRO_ERR_CUDA, std::string("cudaMemset: ") + cudaGetErrorString(e));
  return BRO_OK;
}

void free_device(bro_matrix_s* A) {
  if (A->host_only || A->device < 0) return;
  DeviceGuard g(A->device);
  void* ps[] = {A->d_words, A->d_bit_alloc, A->d_colptr, A->d_symptr, A->d_ell_vals, A->d_pell_col,
                A->d_coo_words, A->d_coo_base, A->d_coo_width, A->d_coo_symptr, A->d_coo_row,
                A->d_coo_col, A->d_coo_vals, A->d_cf, A->d_cl, A->d_last_row, A->d_first_row, A->d_xs, A->d_ys};
  for (void* p : ps)
    if (p) cudaFree(p);
  for (cudaEvent_t e : A->e2e_ev) cudaEventDestroy(e);
  if (A->e2e_h2d) cudaStreamDestroy(A->e2e_h2d);
  if (A->e2e_d2h) cudaStreamDestroy(A->e2e_d2h);
}

bro_status_t check_opts(const bro_opts_t& o) {
  if (o.slice_h != 32) return fail(BRO_ERR_UNSUPPORTED, "slice_h must be 32 (one warp per slice)");
  if (o.sym_bits != 32) return fail(BRO_ERR_UNSUPPORTED, "sym_bits must be 32");
  if (o.vec_words != 1 && o.vec_words != 2 && o.vec_words != 4)
    return fail(BRO_ERR_ARG, "vec_words must be 1, 2 or 4");
  if (o.coo_T != 32) return fail(BRO_ERR_UNSUPPORTED, "coo_T must be 32");
  if (o.codec != 0 && o.codec != 1) return fail(BRO_ERR_ARG, "codec must be 0 or 1");
  if (o.hyb_K < -1) return fail(BRO_ERR_ARG, "hyb_K must be >= -1");
  if (o.min_bits < 0 || o.min_bits > 31) return fail(BRO_ERR_ARG, "min_bits must be in [0, 31]");
  return BRO_OK;
}

void fill_info(bro_matrix_s* A, double secs) {
  bro_info_t& I = A->info;
  std::memset(&I, 0, sizeof(I));
  const int64_t vs = A->vsize;
  I.m = A->m; I.n = A->n; I.nnz = A->nnz;
  I.dtype = A->dtype; I.codec = A->opts.codec; I.format = A->format; I.vec_words = A->opts.vec_words;
  I.K = A->K; I.nnz_ell = A->nnz_ell; I.nnz_coo = A->nnz_coo;
  I.n_slices = A->s; I.ell_pitch = A->pitch; I.n_intervals = A->nI;
  I.encode_seconds = secs;
  int64_t meta = 0, stream = 0, raw_index = 0, values = 0;
  if (A->has_ell) {
    if (A->opts.codec) {
      I.ell_slots = A->ell_slots;
      I.ell_stream_bytes = 4 * A->ell_words;
      meta += 16 * (A->s + 1) + (A->s ? int64_t(A->ell_slots / 32) : 0);  // colptr, symptr, bit_alloc
      stream += I.ell_stream_bytes;
      values += A->ell_slots * vs;
    } else {
      I.ell_slots = A->K * A->pitch;
      raw_index += 4 * A->K * A->pitch;
      values += A->K * A->pitch * vs;
    }
  }
  if (A->has_coo) {
    if (A->opts.codec) {
      I.coo_stream_bytes = 4 * A->coo_words;
      stream += I.coo_stream_bytes;
      meta += A->nI * (4 + 1) + 8 * (A->nI + 1);  // base_row, width, symptr
      raw_index += 4 * A->nnz_coo;                // col
    } else {
      raw_index += 8 * A->nnz_coo;                // row + col
      meta += 4 * A->nI;                          // interval first rows
    }
    values += A->nnz_coo * vs;
  }
  I.meta_bytes = meta;
  I.index_bytes = stream + raw_index + meta;
  I.value_bytes = values;
  I.device_bytes = A->device_bytes;
  I.algorithmic_bytes = I.index_bytes + values + (A->n + A->m) * vs;
  const int64_t O = (A->has_ell ? 4 * A->m * A->K : 0) + 8 * A->nnz_coo;
  I.orig_index_bytes = O;
  const int64_t C = stream + (A->opts.codec ? 4 * A->nnz_coo : raw_index);
  I.eta_stream = O > 0 ? 1.0 - double(C) / double(O) : 0.0;
  I.eta_total = O > 0 ? 1.0 - double(I.index_bytes) / double(O) : 0.0;
}

// Build the handle from validated CSR + a split point K (ELL part = first
// min(len, K) entries of each row; COO part = the rest).
bro_status_t build(int device, bro_dtype_t dtype, int64_t m, int64_t n, const int64_t* row_ptr,
                   const int32_t* col, const void* vals, const bro_opts_t& o, int format,
                   int64_t K, bro_matrix_t* out) {
  auto t0 = std::chrono::steady_clock::now();
  bro_matrix_s* A = new (std::nothrow) bro_matrix_s();
  if (!A) return fail(BRO_ERR_OOM, "host allocation failed");
  A->device = device;
  A->host_only = device == BRO_DEVICE_HOST_ONLY;
  A->dtype = dtype;
  A->vsize = dtype == BRO_FP64 ? 8 : 4;
  A->opts = o;
  A->format = format;
  A->m = m; A->n = n; A->nnz = row_ptr[m];
  A->K = K;
  const uint8_t* v8 = static_cast<const uint8_t*>(vals);
  try {
    // ELL part
    if (format != FMT_COO) {
      A->has_ell = true;
      bro::RowsView rv;
      rv.m = m; rv.row_ptr = row_ptr; rv.col = col; rv.vals = v8; rv.vsize = A->vsize; rv.cap = K;
      int64_t ne = 0;
      for (int64_t i = 0; i < m; ++i) ne += rv.len(i);
      A->nnz_ell = ne;
      if (o.codec) {
        bro::encode_bro_ell(rv, o.vec_words, 16 / A->vsize, o.min_bits, A->ell);
        A->s = A->ell.s;
        A->ell_words = (int64_t)A->ell.words.size();
        A->ell_slots = (int64_t)(A->ell.vals.size() / A->vsize);
        A->ell_max_l = A->ell.max_l;
        for (int64_t t = 0; t < A->s; ++t)
          A->ell_max_S = std::max<int64_t>(A->ell_max_S, int64_t(A->ell.symptr[t + 1] - A->ell.symptr[t]));
        for (int64_t t = 0; t < A->s; ++t)
          A->bulk_unit_max = std::max(A->bulk_unit_max,
              bro::dev::bulk_unit_bytes(A->ell.colptr[t], int(A->ell.colptr[t + 1] - A->ell.colptr[t]),
                                        int(A->ell.symptr[t + 1] - A->ell.symptr[t]), A->vsize));
      } else {
        bro::build_plain_ell(rv, K, A->pell);
        A->pitch = A->pell.pitch;
      }
    }
    // COO part
    A->nnz_coo = A->nnz - A->nnz_ell;
    if (format != FMT_ELL && A->nnz_coo > 0) {
      A->has_coo = true;
      std::vector<int32_t> cr, cc;
      std::vector<uint8_t> cv;
      cr.reserve(A->nnz_coo); cc.reserve(A->nnz_coo); cv.reserve(size_t(A->nnz_coo) * A->vsize);
      const int64_t cap = format == FMT_COO ? 0 : K;
      for (int64_t i = 0; i < m; ++i) {
        for (int64_t p = row_ptr[i] + cap; p < row_ptr[i + 1]; ++p) {
          cr.push_back((int32_t)i);
          cc.push_back(col[p]);
          cv.insert(cv.end(), v8 + size_t(p) * A->vsize, v8 + size_t(p + 1) * A->vsize);
        }
      }
      if (o.codec)
        bro::encode_bro_coo(A->nnz_coo, cr.data(), cc.data(), cv.data(), A->vsize, o.coo_T, o.vec_words, A->coo);
      else
        bro::build_plain_coo(A->nnz_coo, cr.data(), cc.data(), cv.data(), A->vsize, o.coo_T, A->coo);
      A->nI = A->coo.nI;
      A->coo_words = (int64_t)A->coo.words.size();
    }
    // column range of every 32-row block (ELL-only handles): which part of x
    // a block of rows needs, for the pipelined bro_spmv_host
    if (A->has_ell && !A->has_coo) {
      const int64_t nb = (m + 31) / 32;
      A->blk_cmin.assign(nb, INT32_MAX);
      A->blk_cmax.assign(nb, -1);
      for (int64_t i = 0; i < m; ++i) {
        if (row_ptr[i + 1] == row_ptr[i]) continue;
        const int64_t bi = i / 32;
        A->blk_cmin[bi] = std::min(A->blk_cmin[bi], col[row_ptr[i]]);
        A->blk_cmax[bi] = std::max(A->blk_cmax[bi], col[row_ptr[i + 1] - 1]);
      }
    }
  } catch (const std::bad_alloc&) {
    delete A;
    return fail(BRO_ERR_OOM, "host allocation failed during encode");
  }
  double secs = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
  if (!A->host_only) {
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || device < 0 || device >= ndev) {
      delete A;
      return fail(BRO_ERR_CUDA, "no such CUDA device: " + std::to_string(device));
    }
    DeviceGuard g(device);
    bro_status_t st = BRO_OK;
#define UP(dst, vec) \
  if (st == BRO_OK) st = dev_upload(A, &(dst), (vec).data(), (vec).size() * sizeof(*(vec).data()))
    if (A->has_ell && o.codec) {
      UP(A->d_words, A->ell.words);
      UP(A->d_bit_alloc, A->ell.bit_alloc);
      UP(A->d_colptr, A->ell.colptr);
      UP(A->d_symptr, A->ell.symptr);
      if (st == BRO_OK) st = dev_upload(A, &A->d_ell_vals, A->ell.vals.data(), A->ell.vals.size());
    }
    if (A->has_ell && !o.codec) {
      UP(A->d_pell_col, A->pell.col);
      if (st == BRO_OK) st = dev_upload(A, &A->d_ell_vals, A->pell.vals.data(), A->pell.vals.size());
    }
    if (A->has_coo) {
      UP(A->d_coo_base, A->coo.base_row);
      UP(A->d_coo_col, A->coo.col);
      if (st == BRO_OK) st = dev_upload(A, &A->d_coo_vals, A->coo.vals.data(), A->coo.vals.size());
      if (o.codec) {
        UP(A->d_coo_words, A->coo.words);
        UP(A->d_coo_width, A->coo.width);
        UP(A->d_coo_symptr, A->coo.symptr);
      } else {
        UP(A->d_coo_row, A->coo.row);
      }
      // per-work-unit carries (up to kCooMaxUpi units per interval)
      const size_t nU = size_t(A->nI) * kCooMaxUpi;
      if (st == BRO_OK) st = dev_upload(A, &A->d_cf, nullptr, nU * A->vsize);
      if (st == BRO_OK) st = dev_upload(A, &A->d_cl, nullptr, nU * A->vsize);
      if (st == BRO_OK) st = dev_upload(A, &A->d_last_row, nullptr, nU * 4);
      if (st == BRO_OK) st = dev_upload(A, &A->d_first_row, nullptr, nU * 4);
    }
#undef UP
    if (st != BRO_OK) {
      std::string msg = g_err;
      free_device(A);
      delete A;
      return fail(st, msg);
    }
    // host copies are not needed any more (export reads the device copy)
    fill_info(A, secs);
    A->ell = bro::EllCode();
    A->pell = bro::PlainEll();
    A->coo = bro::CooCode();
  } else {
    fill_info(A, secs);
  }
  *out = A;
  return BRO_OK;
}

bro_status_t common_checks(bro_dtype_t dtype, const bro_opts_t* opts, bro_opts_t* o, bro_matrix_t* out) {
  if (!out) return fail(BRO_ERR_ARG, "out is NULL");
  *out = nullptr;
  if (dtype != BRO_FP32 && dtype != BRO_FP64) return fail(BRO_ERR_ARG, "dtype must be BRO_FP32 or BRO_FP64");
  if (opts) *o = *opts; else bro_opts_default(o);
  // vec_words 0 = auto: the layout measured fastest for the dtype on B200
  // (fp64: V = 1, the paper's multiplexing; fp32: V = 4, 16-byte lane chunks)
  if (o->vec_words == 0) o->vec_words = dtype == BRO_FP64 ? 1 : 4;
  return check_opts(*o);
}

// Persistent grid: as many resident blocks as the SMs hold (queried once per
// instantiation), capped by the number of slices.
template <typename T, int V, int kWarps, int kMinBlocks, int G, int kRows, bool kMulti, int kPf = 0>
void launch_bro_ell_od_k(bro_matrix_s* A, const T* x, const bro::dev::YOut<T>& y, cudaStream_t st) {
  using namespace bro::dev;
  auto kern = bro_ell_spmv_od<T, V, kWarps, kMinBlocks, G, kRows, kMulti, kPf>;
  static int resident = 0;
  if (resident == 0) {
    int per_sm = 0, sms = 0, dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kWarps * 32, 0);
    resident = std::max(1, per_sm) * std::max(1, sms);
  }
  const int64_t need = (A->s + kWarps - 1) / kWarps;
  const unsigned grid = (unsigned)std::min<int64_t>(need, resident);
  kern<<<grid, kWarps * 32, 0, st>>>(A->m, A->s, A->d_words, A->d_bit_alloc, A->d_colptr, A->d_symptr,
                                     (const T*)A->d_ell_vals, x, y);
}

// single-destination instance unless the call scatters (bro_spmv_scatter)
template <typename T, int V, int kWarps, int kMinBlocks, int G = 8, int kRows = 34, int kPf = 0>
void launch_bro_ell_od(bro_matrix_s* A, const T* x, const bro::dev::YOut<T>& y, cudaStream_t st) {
  if (y.n > 1 || y.mc != nullptr) launch_bro_ell_od_k<T, V, kWarps, kMinBlocks, G, kRows, true, kPf>(A, x, y, st);
  else launch_bro_ell_od_k<T, V, kWarps, kMinBlocks, G, kRows, false, kPf>(A, x, y, st);
}

constexpr int kEllWarps = 8;      // slices per block
constexpr int kEllMinBlocks = 4;  // 32 resident warps per SM (64 registers)
constexpr int kEllMinBlocksShort = 6;  // fp32: 48 resident warps per SM (40 registers), slices of <= 4 columns; fp64: 40 (48 registers)

// Bulk-staged BRO-ELL (V = 1 only): per-warp ring of nslot slots, each
// holding one whole slice.  Ring bytes per warp: BRO_RING_KB (tuning; default
// kBulkRingKB).  Returns false when a slice does not fit twice in the ring
// (then the register-staged kernel runs).
constexpr int kBulkWarps = 4;
constexpr int kBulkRingKB = 16;
constexpr int kBulkG = 32;
constexpr int kMaxSmemPerBlock = 227 * 1024;

int env_int(const char* name, int dflt) {
  const char* v = std::getenv(name);
  return v && *v ? std::atoi(v) : dflt;
}

template <typename T, int G>
bool launch_bro_ell_bulk_g(bro_matrix_s* A, const T* x, const bro::dev::YOut<T>& y, cudaStream_t st) {
  using namespace bro::dev;
  using L = BulkSmem<kBulkWarps>;
  const int unit = int((A->bulk_unit_max + 127) / 128 * 128);
  if (unit == 0) return false;
  // at least two slots per warp (one in flight while one is consumed)
  const int ring = std::max(env_int("BRO_RING_KB", kBulkRingKB) * 1024, 2 * unit);
  const int fit = (kMaxSmemPerBlock - L::bytes(0, unit)) / (kBulkWarps * unit);  // slots the block can hold
  const int nslot = std::min({kBulkMaxSlots, ring / unit, fit});
  if (nslot < 2) return false;
  const int smem = L::bytes(nslot, unit);
  auto kern = bro_ell_spmv_bulk<T, kBulkWarps, G, 1>;
  static int configured = 0;
  if (smem > configured) {
    if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem) != cudaSuccess) return false;
    configured = smem;
  }
  int per_sm = 0, sms = 0, dev = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kBulkWarps * 32, smem);
  if (per_sm < 1) return false;
  const int64_t need = (A->s + kBulkWarps - 1) / kBulkWarps;
  const unsigned grid = (unsigned)std::min<int64_t>(need, int64_t(per_sm) * sms);
  kern<<<grid, kBulkWarps * 32, smem, st>>>(A->m, A->s, A->d_words, A->d_bit_alloc, A->d_colptr, A->d_symptr,
                                            (const T*)A->d_ell_vals, x, y, nslot, unit);
  return true;
}

template <typename T>
bool launch_bro_ell_bulk(bro_matrix_s* A, const T* x, const bro::dev::YOut<T>& y, cudaStream_t st) {
  if (env_int("BRO_BULK_G", kBulkG) == 16) return launch_bro_ell_bulk_g<T, 16>(A, x, y, st);
  return launch_bro_ell_bulk_g<T, 32>(A, x, y, st);
}

// Tiny slices (every slice <= 4 columns): register-resident decode, kSl
// slices interleaved per warp iteration.  Default (BRO_ELL_TINY = 1, one
// slice per iteration at 40-48 warps/SM): C3's ELL part, BRO-HYB f64 42.0 ->
// 35.9 us (profiles/r01/s3/tiny.txt); 2 = two slices interleaved (slower:
// 40.0 us); 0 = the short-slice instance of the offset-decode kernel.
template <typename T, int V, int kMinBlocks, int kSl>
void launch_bro_ell_tiny(bro_matrix_s* A, const T* x, const bro::dev::YOut<T>& y, cudaStream_t st) {
  using namespace bro::dev;
  constexpr int kW = 8;
  auto kern = bro_ell_spmv_tiny<T, V, kW, kMinBlocks, kSl>;
  static int resident = 0;
  if (resident == 0) {
    int per_sm = 0, sms = 0, dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kW * 32, 0);
    resident = std::max(1, per_sm) * std::max(1, sms);
  }
  const int64_t need = (A->s + kW * kSl - 1) / (kW * kSl);
  const unsigned grid = (unsigned)std::min<int64_t>(need, resident);
  kern<<<grid, kW * 32, 0, st>>>(A->m, A->s, A->d_words, A->d_bit_alloc, A->d_colptr, A->d_symptr,
                                 (const T*)A->d_ell_vals, x, y);
}

// Few slices (fewer than the 32 warps/SM of the general instance can hold,
// e.g. C2: 1,951 slices of up to 81 columns): every warp is resident anyway,
// so spend registers on more columns in flight per warp instead: G = 16 at
// 16 warps/SM for fp64 (127 registers), G = 32 at 8 warps/SM for fp32 (128
// registers) — measured best on C2 (profiles/r01/s3/few_slices.txt: fp64
// 22.5 -> 18.5 us, fp32 20.5 -> 16.4 us).  BRO_ELL_FEW_G = 0 disables.
template <typename T>
constexpr int kEllFewG = sizeof(T) == 8 ? 16 : 32;
// Window rows of the small-window instances: every row stream fits in
// kRows - 1 symbols (C5: S <= 7), so the per-warp symbol window shrinks from
// 34 rows (4.3 KB) to 10 (1.3 KB) or 18: up to 24 KB less shared memory per
// block, which the SM gives back to L1 for the x gather (C5 fp64 349 -> 345
// us, profiles/r01/s3/smallwin.txt).
constexpr int kEllSmallRows = 10;
constexpr int kEllMidRows = 18;  // S <= 17
inline int64_t few_slices(bro_matrix_s* A) {
  static int64_t sms = 0;
  if (sms == 0) {
    int n = 0, dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    sms = std::max(1, n);
  }
  (void)A;
  return sms * kEllWarps * kEllMinBlocks;
}

template <typename T, int V>
void launch_bro_ell(bro_matrix_s* A, const T* x, const bro::dev::YOut<T>& y, cudaStream_t st) {
  // BRO_ELL_KERNEL=2 selects the bulk-staged kernel (V = 1 only; measured
  // slower than the register-staged one on C3-C5)
  if (V == 1 && y.n == 1 && y.mc == nullptr && env_int("BRO_ELL_KERNEL", 0) == 2 && launch_bro_ell_bulk<T>(A, x, y, st))
    return;
  const int variant = env_int("BRO_ELL_VARIANT", 0);  // tuning sweeps only
  if (variant == 1)
    launch_bro_ell_od<T, V, kEllWarps, 5, 4, 34>(A, x, y, st);
  else if (variant == 2)
    launch_bro_ell_od<T, V, kEllWarps, 3, 8, 34>(A, x, y, st);
  else if (variant == 3)  // 16 columns in flight per warp (few, long slices: C2)
    launch_bro_ell_od<T, V, kEllWarps, 2, 16, 34>(A, x, y, st);
  else if (variant == 4)
    launch_bro_ell_od<T, V, 4, 4, 16, 34>(A, x, y, st);
  else if (variant == 5)
    launch_bro_ell_od<T, V, 4, 2, 32, 34>(A, x, y, st);
  else if (variant == 6 && A->ell_max_S < kEllSmallRows)  // 4-warp blocks, 10-row window
    launch_bro_ell_od<T, V, 4, 8, 8, kEllSmallRows>(A, x, y, st);
  else if (variant == 7 && A->ell_max_S < kEllSmallRows)  // 8-warp blocks, 10-row window (the previous default)
    launch_bro_ell_od<T, V, kEllWarps, kEllMinBlocks, 8, kEllSmallRows>(A, x, y, st);
  else if (A->ell_max_l <= 4 && y.n == 1 && y.mc == nullptr && env_int("BRO_ELL_TINY", 1) == 1)
    launch_bro_ell_tiny<T, V, sizeof(T) == 8 ? 5 : 6, 1>(A, x, y, st);
  else if (A->ell_max_l <= 4 && y.n == 1 && y.mc == nullptr && env_int("BRO_ELL_TINY", 1) == 2)
    launch_bro_ell_tiny<T, V, sizeof(T) == 8 ? 3 : 4, 2>(A, x, y, st);
  else if (A->ell_max_l <= 4 && env_int("BRO_ELL_SHORT", 1))
    launch_bro_ell_od<T, V, kEllWarps, sizeof(T) == 8 ? kEllMinBlocksShort - 1 : kEllMinBlocksShort, 4, 6>(A, x, y, st);
  else if (A->s < few_slices(A) && env_int("BRO_ELL_FEW_G", kEllFewG<T>) == 32)
    launch_bro_ell_od<T, V, 4, 2, 32, 34>(A, x, y, st);
  else if (A->s < few_slices(A) && env_int("BRO_ELL_FEW_G", kEllFewG<T>) == 16)
    launch_bro_ell_od<T, V, kEllWarps, 2, 16, 34>(A, x, y, st);
  else if (A->ell_max_S < kEllSmallRows && env_int("BRO_ELL_SMALLWIN", 1) && env_int("BRO_ELL_CPV", 0) == 1)
    launch_bro_ell_od<T, V, 4, 8, 8, kEllSmallRows, 1>(A, x, y, st);
  else if (A->ell_max_S < kEllSmallRows && env_int("BRO_ELL_SMALLWIN", 1) && env_int("BRO_ELL_CPV", 0) == 2)
    launch_bro_ell_od<T, V, 4, 6, 8, kEllSmallRows, 2>(A, x, y, st);
  else if (A->ell_max_S < kEllSmallRows && env_int("BRO_ELL_SMALLWIN", 1))
    launch_bro_ell_od<T, V, 16, 2, 8, kEllSmallRows>(A, x, y, st);  // 16-warp blocks: C5 f32 255.4 -> 250.4 us
  else if (A->ell_max_S < kEllMidRows && env_int("BRO_ELL_SMALLWIN", 1))
    launch_bro_ell_od<T, V, kEllWarps, kEllMinBlocks, 8, kEllMidRows>(A, x, y, st);
  else
    launch_bro_ell_od<T, V, kEllWarps, kEllMinBlocks>(A, x, y, st);
}

// Persistent pipelined COO kernel: kCooPipeWarps warps per block, as many
// blocks as are resident; one work unit per warp (contiguous intervals).
// Register budget: MB = 2 (<= 128 registers, 16 warps/SM) or 3 (<= 80, 24
// warps/SM); BRO_COO_PIPE_MINB selects (tuning), default kCooPipeMinBlocks.
constexpr int kCooPipeWarps = 8;
constexpr int kCooPipeMinBlocks = 2;

template <typename T, int V, bool kBro, int MB>
int64_t coo_pipe_resident() {
  static int64_t resident = 0;
  if (resident == 0) {
    int per_sm = 0, sms = 0, dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(
        &per_sm, bro::dev::coo_spmv_pipe<T, V, kBro, kCooPipeWarps, MB>, kCooPipeWarps * 32, 0);
    resident = int64_t(std::max(1, per_sm)) * std::max(1, sms) * kCooPipeWarps;
  }
  return resident;
}

template <typename T, int MB>
int64_t coo_pipe_warps_mb(bro_matrix_s* A, int V) {
  if (!A->opts.codec) return coo_pipe_resident<T, 4, false, MB>();
  return V == 4 ? coo_pipe_resident<T, 4, true, MB>() : coo_pipe_resident<T, 1, true, MB>();
}

template <typename T>
int64_t coo_pipe_warps(bro_matrix_s* A, int V) {
  return env_int("BRO_COO_PIPE_MINB", kCooPipeMinBlocks) == 3 ? coo_pipe_warps_mb<T, 3>(A, V)
                                                               : coo_pipe_warps_mb<T, 2>(A, V);
}

template <typename T, int MB>
int64_t launch_coo_pipe_mb(bro_matrix_s* A, int V, const T* x, T* y, cudaStream_t st) {
  using namespace bro::dev;
  const int64_t nW = std::max<int64_t>(
      kCooPipeWarps, std::min(coo_pipe_warps_mb<T, MB>(A, V), A->nI) / kCooPipeWarps * kCooPipeWarps);
  const unsigned grid = (unsigned)(nW / kCooPipeWarps);
  auto go = [&](auto kern) {
    kern<<<grid, kCooPipeWarps * 32, 0, st>>>(A->nnz_coo, A->nI, A->d_coo_words, A->d_coo_base, A->d_coo_width,
                                              A->d_coo_symptr, A->d_coo_row, A->d_coo_col, (const T*)A->d_coo_vals,
                                              x, y, (T*)A->d_cf, (T*)A->d_cl, A->d_first_row, A->d_last_row);
  };
  if (!A->opts.codec) go(coo_spmv_pipe<T, 4, false, kCooPipeWarps, MB>);
  else if (V == 4) go(coo_spmv_pipe<T, 4, true, kCooPipeWarps, MB>);
  else go(coo_spmv_pipe<T, 1, true, kCooPipeWarps, MB>);
  return nW;
}

// returns the number of work units (warps) for the fix-up
template <typename T>
int64_t launch_coo_pipe(bro_matrix_s* A, int V, const T* x, T* y, cudaStream_t st) {
  return env_int("BRO_COO_PIPE_MINB", kCooPipeMinBlocks) == 3 ? launch_coo_pipe_mb<T, 3>(A, V, x, y, st)
                                                               : launch_coo_pipe_mb<T, 2>(A, V, x, y, st);
}

template <typename T>
bro::dev::YOut<T> make_yout(T* y) {
  bro::dev::YOut<T> o{};
  o.p[0] = y;
  o.n = 1;
  return o;
}

// y = A.x stored into every destination of yo (yo.p[0] = the local y on A's
// device).  ELL-only handles store all destinations from the ELL kernel's
// epilogue (fused exchange); handles with a COO part finish y locally and
// then replicate it (the COO part and the fix-up add into y).
template <typename T>
bro_status_t launch_spmv(bro_matrix_s* A, const T* x, const bro::dev::YOut<T>& yo, cudaStream_t st) {
  using namespace bro::dev;
  const int V = A->opts.vec_words;
  T* y = yo.p[0];
  const bool fused = !(A->has_coo && A->nI > 0);
  const YOut<T> ye = fused ? yo : make_yout(y);
  if (A->has_ell) {
    if (A->opts.codec) {
      if (A->s > 0) {
        if (V == 4) launch_bro_ell<T, 4>(A, x, ye, st);
        else if (V == 2) launch_bro_ell<T, 2>(A, x, ye, st);
        else launch_bro_ell<T, 1>(A, x, ye, st);
      }
    } else if (A->m > 0) {
      dim3 grid((unsigned)((A->m + kPlainThreads - 1) / kPlainThreads));
      if (ye.n > 1 || ye.mc != nullptr)
        ell_spmv<T, kPlainThreads, true><<<grid, kPlainThreads, 0, st>>>(A->m, A->K, A->pitch, A->d_pell_col,
                                                                        (const T*)A->d_ell_vals, x, ye);
      else
        ell_spmv<T, kPlainThreads, false><<<grid, kPlainThreads, 0, st>>>(A->m, A->K, A->pitch, A->d_pell_col,
                                                                         (const T*)A->d_ell_vals, x, ye);
    }
  } else if (A->m > 0) {
    cudaMemsetAsync(y, 0, size_t(A->m) * sizeof(T), st);
  }
  if (A->has_coo && A->nI > 0) {
    const int warps = kCooThreads / 32;
    int upi = std::max(1, std::min(kCooMaxUpi, env_int("BRO_COO_UPI", kCooUpi)));
    const int upi_log2 = upi >= 4 ? 2 : upi >= 2 ? 1 : 0;
    upi = 1 << upi_log2;
    int64_t nU = A->nI * upi;
    // BRO_COO_KERNEL: 1 (default) per-unit kernel; 2 persistent pipelined
    // kernel (opt-in: measured no faster); 0 auto =
    // pipelined when there are at least as many intervals as resident warps
    const int ck = env_int("BRO_COO_KERNEL", 1);
    const int64_t pipe_w = (V == 2 || ck == 1) ? 0 : coo_pipe_warps<T>(A, V);
    if (pipe_w > 0 && A->nI >= kCooPipeWarps && (ck == 2 || (ck == 0 && A->nI >= pipe_w))) {
      nU = launch_coo_pipe<T>(A, V, x, y, st);
      upi = 0;
    }
    dim3 grid((unsigned)((nU + warps - 1) / warps));
    const int T_ = A->opts.coo_T;
    if (upi > 0) {
    auto args = [&](auto kern) {
      kern<<<grid, kCooThreads, 0, st>>>(A->nnz_coo, A->nI, T_, upi_log2, A->d_coo_words, A->d_coo_base,
                                         A->d_coo_width, A->d_coo_symptr, A->d_coo_row, A->d_coo_col,
                                         (const T*)A->d_coo_vals, x, y, (T*)A->d_cf, (T*)A->d_cl,
                                         A->d_first_row, A->d_last_row, env_int("BRO_COO_L2PF", 0));
    };
    // BRO_COO_MINB=4: 64-register instances (32 resident warps/SM; tuning sweeps)
    const bool minb4 = env_int("BRO_COO_MINB", 0) == 4;
    if (A->opts.codec) {
      if (V == 4) minb4 ? args(coo_spmv<T, 4, true, kCooThreads, 4>) : args(coo_spmv<T, 4, true, kCooThreads>);
      else if (V == 2) args(coo_spmv<T, 2, true, kCooThreads>);
      else minb4 ? args(coo_spmv<T, 1, true, kCooThreads, 4>) : args(coo_spmv<T, 1, true, kCooThreads>);
    } else {
      minb4 ? args(coo_spmv<T, 4, false, kCooThreads, 4>) : args(coo_spmv<T, 4, false, kCooThreads>);
    }
    }
    dim3 g2((unsigned)((nU + 255) / 256));
    coo_fixup<T><<<g2, 256, 0, st>>>(nU, A->d_first_row, A->d_last_row, (const T*)A->d_cf,
                                     (const T*)A->d_cl, y);
  }
  if (!fused && A->m > 0 && (yo.n > 1 || yo.mc != nullptr)) {
    const unsigned g3 = (unsigned)std::min<int64_t>((A->m + 255) / 256, 148 * 8);
    replicate_y<T><<<g3, 256, 0, st>>>(A->m, yo);
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(BRO_ERR_CUDA, std::string("kernel launch: ") + cudaGetErrorString(e));
  return BRO_OK;
}

struct PartView {
  const void* host = nullptr;
  const void* dev = nullptr;
  size_t bytes = 0;
};

PartView part_view(bro_matrix_s* A, int32_t part) {
  PartView v;
  const bool bro_ell = A->has_ell && A->opts.codec;
  const bool plain_ell = A->has_ell && !A->opts.codec;
  const bool coo = A->has_coo;
  const bool bro_coo = coo && A->opts.codec;
  const size_t vs = A->vsize;
  auto set = [&](const void* h, const void* d, size_t b) { v.host = h; v.dev = d; v.bytes = b; };
  switch (part) {
    case BRO_PART_ELL_WORDS: if (bro_ell) set(A->ell.words.data(), A->d_words, 4 * size_t(A->ell_words)); break;
    case BRO_PART_ELL_BIT_ALLOC: if (bro_ell) set(A->ell.bit_alloc.data(), A->d_bit_alloc, size_t(A->ell_slots / 32)); break;
    case BRO_PART_ELL_COLPTR: if (bro_ell) set(A->ell.colptr.data(), A->d_colptr, 8 * size_t(A->s + 1)); break;
    case BRO_PART_ELL_SYMPTR: if (bro_ell) set(A->ell.symptr.data(), A->d_symptr, 8 * size_t(A->s + 1)); break;
    case BRO_PART_ELL_VALS: if (bro_ell) set(A->ell.vals.data(), A->d_ell_vals, vs * size_t(A->ell_slots)); break;
    case BRO_PART_COO_WORDS: if (bro_coo) set(A->coo.words.data(), A->d_coo_words, 4 * size_t(A->coo_words)); break;
    case BRO_PART_COO_BASE_ROW: if (bro_coo) set(A->coo.base_row.data(), A->d_coo_base, 4 * size_t(A->nI)); break;
    case BRO_PART_COO_WIDTH: if (bro_coo) set(A->coo.width.data(), A->d_coo_width, size_t(A->nI)); break;
    case BRO_PART_COO_SYMPTR: if (bro_coo) set(A->coo.symptr.data(), A->d_coo_symptr, 8 * size_t(A->nI + 1)); break;
    case BRO_PART_COO_COL: if (coo) set(A->coo.col.data(), A->d_coo_col, 4 * size_t(A->nnz_coo)); break;
    case BRO_PART_COO_VALS: if (coo) set(A->coo.vals.data(), A->d_coo_vals, vs * size_t(A->nnz_coo)); break;
    case BRO_PART_COO_ROW: if (coo && !A->opts.codec) set(A->coo.row.data(), A->d_coo_row, 4 * size_t(A->nnz_coo)); break;
    case BRO_PART_PELL_COL: if (plain_ell) set(A->pell.col.data(), A->d_pell_col, 4 * size_t(A->K * A->pitch)); break;
    case BRO_PART_PELL_VALS: if (plain_ell) set(A->pell.vals.data(), A->d_ell_vals, vs * size_t(A->K * A->pitch)); break;
    default: v.bytes = SIZE_MAX;
  }
  return v;
}

}  // namespace

namespace {

// y = A.x over 32-row blocks [b0, b1) only: the ELL arrays are addressed
// through the block range (slice metadata / plain ELL rows offset by b0, y
// offset by 32*b0), the kernels are unchanged.  ELL-only handles.
template <typename T>
bro_status_t launch_spmv_blocks(bro_matrix_s* A, const T* x, T* y, int64_t b0, int64_t b1, cudaStream_t st) {
  const int64_t m0 = A->m, s0 = A->s;
  uint64_t* const cp0 = A->d_colptr;
  uint64_t* const sp0 = A->d_symptr;
  int32_t* const pc0 = A->d_pell_col;
  void* const pv0 = A->d_ell_vals;
  A->m = std::min(m0, 32 * b1) - 32 * b0;
  if (A->opts.codec) {
    A->s = b1 - b0;
    A->d_colptr = cp0 + b0;
    A->d_symptr = sp0 + b0;
  } else {
    A->d_pell_col = pc0 + 32 * b0;
    A->d_ell_vals = static_cast<char*>(pv0) + size_t(32 * b0) * A->vsize;
  }
  const bro_status_t r = launch_spmv<T>(A, x, make_yout(y + 32 * b0), st);
  A->m = m0; A->s = s0; A->d_colptr = cp0; A->d_symptr = sp0; A->d_pell_col = pc0; A->d_ell_vals = pv0;
  return r;
}

// Pipelined end-to-end SpMV of an ELL-only handle: x goes up in K pieces on
// one stream, each block of rows runs as soon as the pieces covering its
// columns (blk_cmin/blk_cmax) have arrived, and its y goes down on a third
// stream while later blocks compute — H2D, compute and D2H overlap (PCIe is
// full duplex).  Same kernels and per-row arithmetic as bro_spmv.
bro_status_t spmv_host_pipelined(bro_matrix_s* A, const void* x_host, void* y_host, cudaStream_t st, int K) {
  const int64_t nb = (A->m + 31) / 32;
  const size_t vs = size_t(A->vsize);
  cudaError_t e = cudaSuccess;
  if (!A->e2e_h2d) {
    if ((e = cudaStreamCreateWithFlags(&A->e2e_h2d, cudaStreamNonBlocking)) != cudaSuccess ||
        (e = cudaStreamCreateWithFlags(&A->e2e_d2h, cudaStreamNonBlocking)) != cudaSuccess)
      return fail(BRO_ERR_CUDA, std::string("stream create: ") + cudaGetErrorString(e));
  }
  while ((int)A->e2e_ev.size() < 2 * K + 1) {
    cudaEvent_t ev;
    if ((e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming)) != cudaSuccess)
      return fail(BRO_ERR_CUDA, std::string("event create: ") + cudaGetErrorString(e));
    A->e2e_ev.push_back(ev);
  }
  cudaEvent_t* evx = A->e2e_ev.data();
  cudaEvent_t* evy = evx + K;
  cudaEvent_t start = evx[2 * K];
  auto xa = [&](int i) { return A->n * i / K; };
  // the side streams start after earlier work on the caller's stream
  cudaEventRecord(start, st);
  cudaStreamWaitEvent(A->e2e_h2d, start, 0);
  cudaStreamWaitEvent(A->e2e_d2h, start, 0);
  for (int i = 0; i < K; ++i) {
    const int64_t a = xa(i), b = xa(i + 1);
    if (b > a)
      e = cudaMemcpyAsync(static_cast<char*>(A->d_xs) + a * vs, static_cast<const char*>(x_host) + a * vs,
                          size_t(b - a) * vs, cudaMemcpyHostToDevice, A->e2e_h2d);
    if (e != cudaSuccess) return fail(BRO_ERR_CUDA, std::string("H2D x: ") + cudaGetErrorString(e));
    cudaEventRecord(evx[i], A->e2e_h2d);
  }
  for (int c = 0; c < K; ++c) {
    const int64_t b0 = nb * c / K, b1 = nb * (c + 1) / K;
    if (b1 <= b0) {
      cudaEventRecord(evy[c], st);
      continue;
    }
    int32_t hi = -1;
    for (int64_t bi = b0; bi < b1; ++bi) hi = std::max(hi, A->blk_cmax[bi]);
    // wait for the piece holding column hi (pieces arrive in order)
    int p = K - 1;
    if (hi < 0) p = -1;
    else
      while (p > 0 && xa(p) > hi) --p;
    if (p >= 0) cudaStreamWaitEvent(st, evx[p], 0);
    bro_status_t r = A->dtype == BRO_FP64
        ? launch_spmv_blocks<double>(A, (const double*)A->d_xs, (double*)A->d_ys, b0, b1, st)
        : launch_spmv_blocks<float>(A, (const float*)A->d_xs, (float*)A->d_ys, b0, b1, st);
    if (r != BRO_OK) return r;
    cudaEventRecord(evy[c], st);
    cudaStreamWaitEvent(A->e2e_d2h, evy[c], 0);
    const int64_t r0 = 32 * b0, r1 = std::min(A->m, 32 * b1);
    e = cudaMemcpyAsync(static_cast<char*>(y_host) + r0 * vs, static_cast<const char*>(A->d_ys) + r0 * vs,
                        size_t(r1 - r0) * vs, cudaMemcpyDeviceToHost, A->e2e_d2h);
    if (e != cudaSuccess) return fail(BRO_ERR_CUDA, std::string("D2H y: ") + cudaGetErrorString(e));
  }
  if ((e = cudaStreamSynchronize(A->e2e_d2h)) != cudaSuccess || (e = cudaStreamSynchronize(st)) != cudaSuccess ||
      (e = cudaStreamSynchronize(A->e2e_h2d)) != cudaSuccess)
    return fail(BRO_ERR_CUDA, std::string("sync: ") + cudaGetErrorString(e));
  return BRO_OK;
}

}  // namespace

extern "C" {

void bro_opts_default(bro_opts_t* o) {
  if (!o) return;
  o->slice_h = 32;
  o->sym_bits = 32;
  o->vec_words = 0;
  o->coo_T = 32;
  o->hyb_K = -1;
  o->codec = 1;
  o->min_bits = 0;
}

bro_status_t bro_create_ell(int device, bro_dtype_t dtype, int64_t m, int64_t n, const int64_t* row_ptr,
                            const int32_t* col_idx, const void* vals, const bro_opts_t* opts,
                            bro_matrix_t* out) {
  g_err.clear();
  bro_opts_t o;
  bro_status_t st = common_checks(dtype, opts, &o, out);
  if (st) return st;
  std::string msg = bro::check_csr(m, n, row_ptr, col_idx);
  if (!msg.empty()) return fail(msg.rfind("shape", 0) == 0 ? BRO_ERR_SHAPE : (row_ptr ? BRO_ERR_INDEX : BRO_ERR_ARG), msg);
  if (row_ptr[m] > 0 && !vals) return fail(BRO_ERR_ARG, "vals is NULL");
  int64_t K = 0;
  for (int64_t i = 0; i < m; ++i) K = std::max(K, row_ptr[i + 1] - row_ptr[i]);
  return build(device, dtype, m, n, row_ptr, col_idx, vals, o, FMT_ELL, K, out);
}

bro_status_t bro_create_hyb(int device, bro_dtype_t dtype, int64_t m, int64_t n, const int64_t* row_ptr,
                            const int32_t* col_idx, const void* vals, const bro_opts_t* opts,
                            bro_matrix_t* out) {
  g_err.clear();
  bro_opts_t o;
  bro_status_t st = common_checks(dtype, opts, &o, out);
  if (st) return st;
  std::string msg = bro::check_csr(m, n, row_ptr, col_idx);
  if (!msg.empty()) return fail(msg.rfind("shape", 0) == 0 ? BRO_ERR_SHAPE : (row_ptr ? BRO_ERR_INDEX : BRO_ERR_ARG), msg);
  if (row_ptr[m] > 0 && !vals) return fail(BRO_ERR_ARG, "vals is NULL");
  const int64_t K = o.hyb_K >= 0 ? o.hyb_K : bro::hyb_K(m, row_ptr);
  return build(device, dtype, m, n, row_ptr, col_idx, vals, o, FMT_HYB, K, out);
}

bro_status_t bro_create_coo(int device, bro_dtype_t dtype, int64_t m, int64_t n, int64_t nnz,
                            const int32_t* row_idx, const int32_t* col_idx, const void* vals,
                            const bro_opts_t* opts, bro_matrix_t* out) {
  g_err.clear();
  bro_opts_t o;
  bro_status_t st = common_checks(dtype, opts, &o, out);
  if (st) return st;
  std::string msg = bro::check_coo(m, n, nnz, row_idx, col_idx);
  if (!msg.empty()) return fail(msg.rfind("shape", 0) == 0 ? BRO_ERR_SHAPE : BRO_ERR_INDEX, msg);
  if (nnz > 0 && !vals) return fail(BRO_ERR_ARG, "vals is NULL");
  std::vector<int64_t> rp(m + 1, 0);
  for (int64_t e = 0; e < nnz; ++e) rp[row_idx[e] + 1]++;
  for (int64_t i = 0; i < m; ++i) rp[i + 1] += rp[i];
  return build(device, dtype, m, n, rp.data(), col_idx, vals, o, FMT_COO, 0, out);
}

bro_status_t bro_spmv(bro_matrix_t A, const void* x, void* y, bro_stream_t stream) {
  if (!A) return fail(BRO_ERR_ARG, "matrix is NULL");
  if (A->host_only) return fail(BRO_ERR_UNSUPPORTED, "host-only handle: no device copy (there is no CPU SpMV path)");
  if ((!x && A->n > 0) || (!y && A->m > 0)) return fail(BRO_ERR_ARG, "x or y is NULL");
  if (x == y && A->m > 0) return fail(BRO_ERR_ARG, "x and y must not alias");
  DeviceGuard g(A->device);
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  if (A->dtype == BRO_FP64) return launch_spmv<double>(A, (const double*)x, make_yout((double*)y), st);
  return launch_spmv<float>(A, (const float*)x, make_yout((float*)y), st);
}

bro_status_t bro_spmv_scatter(bro_matrix_t A, const void* x, void* const* y_dsts, int32_t n_dst,
                              void* y_mc, bro_stream_t stream) {
  if (!A) return fail(BRO_ERR_ARG, "matrix is NULL");
  if (A->host_only) return fail(BRO_ERR_UNSUPPORTED, "host-only handle: no device copy (there is no CPU SpMV path)");
  if (!y_dsts || n_dst < 1 || n_dst > bro::dev::kMaxDst)
    return fail(BRO_ERR_ARG, "y_dsts must hold 1.." + std::to_string(bro::dev::kMaxDst) + " pointers");
  if (!x && A->n > 0) return fail(BRO_ERR_ARG, "x is NULL");
  for (int i = 0; i < n_dst; ++i) {
    if (!y_dsts[i] && A->m > 0) return fail(BRO_ERR_ARG, "y_dsts[" + std::to_string(i) + "] is NULL");
    if (y_dsts[i] == x && A->m > 0) return fail(BRO_ERR_ARG, "x and a y destination must not alias");
  }
  if (y_mc && y_mc == x && A->m > 0) return fail(BRO_ERR_ARG, "x and the multicast y must not alias");
  DeviceGuard g(A->device);
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  auto run = [&](auto* tag) {
    using T = std::remove_pointer_t<decltype(tag)>;
    bro::dev::YOut<T> o{};
    for (int i = 0; i < n_dst; ++i) o.p[i] = static_cast<T*>(y_dsts[i]);
    o.n = n_dst;
    o.mc = static_cast<T*>(y_mc);
    return launch_spmv<T>(A, static_cast<const T*>(x), o, st);
  };
  if (A->dtype == BRO_FP64) return run((double*)nullptr);
  return run((float*)nullptr);
}

bro_status_t bro_spmv_host(bro_matrix_t A, const void* x_host, void* y_host, bro_stream_t stream) {
  if (!A) return fail(BRO_ERR_ARG, "matrix is NULL");
  if (A->host_only) return fail(BRO_ERR_UNSUPPORTED, "host-only handle: no device copy (there is no CPU SpMV path)");
  if ((!x_host && A->n > 0) || (!y_host && A->m > 0)) return fail(BRO_ERR_ARG, "x or y is NULL");
  DeviceGuard g(A->device);
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  const size_t xb = size_t(A->n) * A->vsize, yb = size_t(A->m) * A->vsize;
  bro_status_t s = BRO_OK;
  if (!A->d_xs && xb) s = dev_upload(A, &A->d_xs, nullptr, xb);
  if (s == BRO_OK && !A->d_ys && yb) s = dev_upload(A, &A->d_ys, nullptr, yb);
  if (s != BRO_OK) return s;
  // ELL-only handles: pipelined copies and compute (BRO_E2E_CHUNKS pieces, 1 = serial)
  const int K = std::max(1, std::min(64, env_int("BRO_E2E_CHUNKS", kE2eChunks)));
  const size_t min_bytes = size_t(std::max(0, env_int("BRO_E2E_MIN_KB", int(kE2eMinBytes >> 10)))) << 10;
  if (K > 1 && A->has_ell && !A->has_coo && int64_t(A->blk_cmax.size()) >= K && xb >= min_bytes && xb > 0)
    return spmv_host_pipelined(A, x_host, y_host, st, K);
  cudaError_t e = xb ? cudaMemcpyAsync(A->d_xs, x_host, xb, cudaMemcpyHostToDevice, st) : cudaSuccess;
  if (e != cudaSuccess) return fail(BRO_ERR_CUDA, std::string("H2D x: ") + cudaGetErrorString(e));
  s = bro_spmv(A, A->d_xs, A->d_ys, stream);
  if (s != BRO_OK) return s;
  e = yb ? cudaMemcpyAsync(y_host, A->d_ys, yb, cudaMemcpyDeviceToHost, st) : cudaSuccess;
  if (e != cudaSuccess) return fail(BRO_ERR_CUDA, std::string("D2H y: ") + cudaGetErrorString(e));
  e = cudaStreamSynchronize(st);
  if (e != cudaSuccess) return fail(BRO_ERR_CUDA, std::string("sync: ") + cudaGetErrorString(e));
  return BRO_OK;
}

bro_status_t bro_destroy(bro_matrix_t A) {
  if (!A) return BRO_OK;
  free_device(A);
  delete A;
  return BRO_OK;
}

bro_status_t bro_get_info(bro_matrix_t A, bro_info_t* info) {
  if (!A || !info) return fail(BRO_ERR_ARG, "NULL argument");
  A->info.device_bytes = A->device_bytes;
  *info = A->info;
  return BRO_OK;
}

bro_status_t bro_export_encoded(bro_matrix_t A, int32_t part, void* host_buf, size_t* nbytes) {
  if (!A || !nbytes) return fail(BRO_ERR_ARG, "NULL argument");
  PartView v = part_view(A, part);
  if (v.bytes == SIZE_MAX) return fail(BRO_ERR_ARG, "unknown part " + std::to_string(part));
  if (!host_buf) {
    *nbytes = v.bytes;
    return BRO_OK;
  }
  if (*nbytes < v.bytes) return fail(BRO_ERR_ARG, "buffer too small for part " + std::to_string(part));
  *nbytes = v.bytes;
  if (v.bytes == 0) return BRO_OK;
  if (A->host_only) {
    std::memcpy(host_buf, v.host, v.bytes);
    return BRO_OK;
  }
  DeviceGuard g(A->device);
  cudaError_t e = cudaMemcpy(host_buf, v.dev, v.bytes, cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return fail(BRO_ERR_CUDA, std::string("D2H export: ") + cudaGetErrorString(e));
  return BRO_OK;
}

bro_status_t bro_decode_indices(bro_matrix_t A, int32_t* d_ell_cols, int32_t* d_coo_rows, bro_stream_t stream) {
  using namespace bro::dev;
  if (!A) return fail(BRO_ERR_ARG, "matrix is NULL");
  if (A->host_only) return fail(BRO_ERR_UNSUPPORTED, "host-only handle has no device copy");
  DeviceGuard g(A->device);
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  const int V = A->opts.vec_words;
  if (d_ell_cols && A->has_ell) {
    if (A->opts.codec) {
      if (A->s > 0) {
        dim3 grid((unsigned)((A->s + 7) / 8));
        if (V == 4) bro_ell_decode<4><<<grid, 256, 0, st>>>(A->s, A->d_words, A->d_bit_alloc, A->d_colptr, A->d_symptr, d_ell_cols);
        else if (V == 2) bro_ell_decode<2><<<grid, 256, 0, st>>>(A->s, A->d_words, A->d_bit_alloc, A->d_colptr, A->d_symptr, d_ell_cols);
        else bro_ell_decode<1><<<grid, 256, 0, st>>>(A->s, A->d_words, A->d_bit_alloc, A->d_colptr, A->d_symptr, d_ell_cols);
      }
    } else if (A->K * A->pitch > 0) {
      dim3 grid((unsigned)((A->K * A->pitch + 255) / 256));
      ell_decode<<<grid, 256, 0, st>>>(A->m, A->K, A->pitch, A->d_pell_col, d_ell_cols);
    }
  }
  if (d_coo_rows && A->has_coo && A->nI > 0) {
    if (A->opts.codec) {
      dim3 grid((unsigned)((A->nI + 7) / 8));
      if (V == 4) bro_coo_decode<4><<<grid, 256, 0, st>>>(A->nnz_coo, A->nI, A->opts.coo_T, A->d_coo_words, A->d_coo_base, A->d_coo_width, A->d_coo_symptr, d_coo_rows);
      else if (V == 2) bro_coo_decode<2><<<grid, 256, 0, st>>>(A->nnz_coo, A->nI, A->opts.coo_T, A->d_coo_words, A->d_coo_base, A->d_coo_width, A->d_coo_symptr, d_coo_rows);
      else bro_coo_decode<1><<<grid, 256, 0, st>>>(A->nnz_coo, A->nI, A->opts.coo_T, A->d_coo_words, A->d_coo_base, A->d_coo_width, A->d_coo_symptr, d_coo_rows);
    } else {
      cudaMemcpyAsync(d_coo_rows, A->d_coo_row, 4 * size_t(A->nnz_coo), cudaMemcpyDeviceToDevice, st);
    }
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return fail(BRO_ERR_CUDA, std::string("decode launch: ") + cudaGetErrorString(e));
  return BRO_OK;
}

bro_status_t bro_hyb_K(int64_t m, const int64_t* row_ptr, int64_t* K_out) {
  if (!row_ptr || !K_out || m < 0) return fail(BRO_ERR_ARG, "bad argument");
  *K_out = bro::hyb_K(m, row_ptr);
  return BRO_OK;
}

bro_status_t bro_reorder_bar(int64_t m, int64_t n, const int64_t* row_ptr, const int32_t* col_idx,
                             bro_dtype_t dtype, int32_t method, int64_t* perm_out) {
  g_err.clear();
  if (!perm_out) return fail(BRO_ERR_ARG, "perm_out is NULL");
  if (dtype != BRO_FP32 && dtype != BRO_FP64) return fail(BRO_ERR_ARG, "bad dtype");
  std::string msg = bro::check_csr(m, n, row_ptr, col_idx);
  if (!msg.empty()) return fail(msg.rfind("shape", 0) == 0 ? BRO_ERR_SHAPE : BRO_ERR_INDEX, msg);
  try {
    if (method == 0) {
      bro::bar_signature_order(m, row_ptr, col_idx, perm_out);
      return BRO_OK;
    }
    if (method == 2) {
      bro::bar_window_order(m, row_ptr, col_idx, dtype == BRO_FP64 ? 8 : 4, env_int("BRO_BAR_WINDOW", kBarWindow),
                            perm_out);
      return BRO_OK;
    }
    if (method == 1) {
      std::string err;
      if (!bro::bar_greedy_order(m, n, row_ptr, col_idx, dtype == BRO_FP64 ? 8 : 4, perm_out, &err))
        return fail(BRO_ERR_UNSUPPORTED, err);
      return BRO_OK;
    }
  } catch (const std::bad_alloc&) {
    return fail(BRO_ERR_OOM, "host allocation failed");
  }
  return fail(BRO_ERR_ARG, "method must be 0, 1 or 2");
}

const char* bro_status_str(bro_status_t s) {
  switch (s) {
    case BRO_OK: return "BRO_OK";
    case BRO_ERR_ARG: return "BRO_ERR_ARG";
    case BRO_ERR_INDEX: return "BRO_ERR_INDEX";
    case BRO_ERR_SHAPE: return "BRO_ERR_SHAPE";
    case BRO_ERR_OOM: return "BRO_ERR_OOM";
    case BRO_ERR_CUDA: return "BRO_ERR_CUDA";
    case BRO_ERR_UNSUPPORTED: return "BRO_ERR_UNSUPPORTED";
  }
  return "BRO_ERR_UNKNOWN";
}

const char* bro_last_error(void) { return g_err.c_str(); }

int bro_version(void) { return BRO_VERSION; }

}  // extern "C"
