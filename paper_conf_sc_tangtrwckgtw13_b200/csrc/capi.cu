// C ABI of libbro.so (include/bro.h): validation, host encode, upload,
// kernel-instance resolution (once, at create, on the handle's device) and
// launch.  The kernels live in kern_*.cu (launch.hpp is the table).
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <climits>
#include <cstring>
#include <new>
#include <string>
#include <type_traits>

#include "../../include/bro.h"
#include "encode.hpp"
#include "kernels.cuh"
#include "launch.hpp"

namespace {

thread_local std::string g_err;

bro_status_t fail(bro_status_t s, const std::string& msg) {
  g_err = msg;
  return s;
}

constexpr int kE2eChunks = 8;  // pieces of the pipelined bro_spmv_host
// below this x size the pieces' launch and event overheads exceed the copy
// time they hide (C1/C2 e2e: 1.3 -> 0.5 and 63 -> 57 GFLOP/s when pipelined)
constexpr size_t kE2eMinBytes = size_t(4) << 20;
constexpr int kBarWindow = 64;  // candidate partitions of BAR method 2 (windowed Algorithm 2)
// Device-independent thresholds of the automatic layout choices (a B200 has
// 148 SMs; the general BRO-ELL instance keeps 32 warps per SM resident):
constexpr int64_t kB200Warps = 148 * 32;
constexpr int64_t kAutoH64Rows = 64 * kB200Warps;  // slice_h = 64 from 303,104 rows on

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

// A kernel instance of a handle, resolved on the handle's device at create:
// its entry point and how many of its blocks the device keeps resident.
struct Launch {
  bro::KernelRef k;
  int64_t resident_blocks = 0;
};

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
  int h = 32;       // BRO-ELL slice height (rows of a row block of the plain ELL)
  int coo_T = 32;   // COO entries per lane of an interval
  int ell_inst = 0; // BRO-ELL kernel instance (launch.hpp EllInst)
  // value index of the BRO-ELL part (opts.value_codec = 1, reading R28)
  bro::ValueIndexCode vi;
  uint8_t* d_vcodes = nullptr;
  void* d_vdict = nullptr;
  // host encodings (kept only by host-only handles after create)
  bro::EllCode ell;
  bro::PlainEll pell;
  bro::CooCode coo;
  int64_t s = 0, ell_words = 0, ell_slots = 0, pitch = 0, nI = 0, coo_words = 0;
  int64_t ell_max_S = 0;  // most 32-bit symbols in one BRO-ELL row stream
  int64_t ell_max_l = 0;  // longest BRO-ELL slice (columns)
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
  int32_t* d_coo_end = nullptr;  // per interval: row of its last entry
  int4* d_spans = nullptr;       // rows spanning intervals: {row, first interval, last interval, uses cl}
  int64_t n_spans = 0;
  std::vector<int32_t> coo_end_host;
  std::vector<int4> spans_host;
  void* d_xs = nullptr;
  void* d_ys = nullptr;
  int64_t device_bytes = 0;
  // kernel instances (index = mode: 0 spmv, 1 scatter, 2 decode)
  Launch ell_k[3];
  Launch coo_k[3];  // 0 spmv, 2 decode
  Launch fix_k, rep_k;
  // x-window staging of the few-slice instance (row N1): per block {first
  // column, columns} of its x window, the staged instance, its shared bytes
  int2* d_xwin = nullptr;
  std::vector<int2> xwin_host;
  Launch ell_x;
  int xwin_bytes = 0;
  bool xstage = false;
  // end-to-end pipeline of ELL-only handles (bro_spmv_host): column range of
  // every row block (h rows), side streams and events (created on first use)
  std::vector<int32_t> blk_cmin, blk_cmax;
  cudaStream_t e2e_h2d = nullptr, e2e_d2h = nullptr;
  std::vector<cudaEvent_t> e2e_ev;
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
                A->d_coo_col, A->d_coo_vals, A->d_cf, A->d_cl, A->d_coo_end, A->d_spans, A->d_xs, A->d_ys,
                A->d_xwin, A->d_vcodes, A->d_vdict};
  for (void* p : ps)
    if (p) cudaFree(p);
  for (cudaEvent_t e : A->e2e_ev) cudaEventDestroy(e);
  if (A->e2e_h2d) cudaStreamDestroy(A->e2e_h2d);
  if (A->e2e_d2h) cudaStreamDestroy(A->e2e_d2h);
}

bro_status_t check_opts(const bro_opts_t& o) {
  if (o.slice_h != 0 && o.slice_h != 32 && o.slice_h != 64)
    return fail(BRO_ERR_UNSUPPORTED, "slice_h must be 0 (auto), 32 or 64");
  if (o.sym_bits != 32) return fail(BRO_ERR_UNSUPPORTED, "sym_bits must be 32");
  if (o.vec_words != 0 && o.vec_words != 1 && o.vec_words != 4)
    return fail(BRO_ERR_ARG, "vec_words must be 0 (auto), 1 or 4");
  if (o.coo_T != 0 && o.coo_T != 8 && o.coo_T != 16 && o.coo_T != 32)
    return fail(BRO_ERR_UNSUPPORTED, "coo_T must be 0 (auto), 8, 16 or 32");
  if (o.codec != 0 && o.codec != 1) return fail(BRO_ERR_ARG, "codec must be 0 or 1");
  if (o.hyb_K < -1) return fail(BRO_ERR_ARG, "hyb_K must be >= -1");
  if (o.min_bits < 0 || o.min_bits > 31) return fail(BRO_ERR_ARG, "min_bits must be in [0, 31]");
  if (o.pdl < 0 || o.pdl > 2) return fail(BRO_ERR_ARG, "pdl must be 0, 1 or 2");
  if (o.x_stage < 0 || o.x_stage > 1) return fail(BRO_ERR_ARG, "x_stage must be 0 or 1");
  if (o.value_codec < 0 || o.value_codec > 1) return fail(BRO_ERR_ARG, "value_codec must be 0 or 1");
  if (o.value_codec == 1 && o.codec != 1) return fail(BRO_ERR_ARG, "value_codec 1 needs codec 1 (BRO-ELL values)");
  if (o.ell_kernel < 0 || o.ell_kernel > bro::ELL_LAST)
    return fail(BRO_ERR_ARG, "ell_kernel must be in [0, " + std::to_string(bro::ELL_LAST) + "]");
  return BRO_OK;
}

// coo_T = 0: T = 8 (256-entry intervals) — measured fastest for BRO-COO and
// plain COO alike on C3 and C4 (profiles/r02/ab/r02o): both kernels are
// latency-bound, and shorter intervals give more warps in flight
int auto_coo_T(int64_t) { return 8; }

void fill_info(bro_matrix_s* A, double secs) {
  bro_info_t& I = A->info;
  std::memset(&I, 0, sizeof(I));
  const int64_t vs = A->vsize;
  I.m = A->m; I.n = A->n; I.nnz = A->nnz;
  I.dtype = A->dtype; I.codec = A->opts.codec; I.format = A->format; I.vec_words = A->opts.vec_words;
  I.slice_h = A->h; I.coo_T = A->coo_T; I.ell_kernel = A->ell_inst;
  I.x_stage_bytes = A->xstage ? A->xwin_bytes : 0;
  I.K = A->K; I.nnz_ell = A->nnz_ell; I.nnz_coo = A->nnz_coo;
  I.n_slices = A->s; I.ell_pitch = A->pitch; I.n_intervals = A->nI;
  I.encode_seconds = secs;
  int64_t meta = 0, stream = 0, raw_index = 0, values = 0;
  if (A->has_ell) {
    if (A->opts.codec) {
      I.ell_slots = A->ell_slots;
      I.ell_stream_bytes = 4 * A->ell_words;
      meta += 16 * (A->s + 1) + (A->s ? int64_t(A->ell_slots / A->h) : 0);  // colptr, symptr, bit_alloc
      stream += I.ell_stream_bytes;
      if (A->vi.cb) {  // value index: codes per slot + the table
        values += A->ell_slots * A->vi.cb + A->vi.nd * vs;
        I.value_code_bytes = A->vi.cb;
        I.value_dict_size = A->vi.nd;
      } else {
        values += A->ell_slots * vs;
      }
    } else {
      I.ell_slots = A->K * A->pitch;
      raw_index += 4 * A->K * A->pitch;
      values += A->K * A->pitch * vs;
    }
  }
  if (A->has_coo) {
    const int64_t slots = A->nI * 32 * A->coo_T;  // stored (padded) COO slots
    if (A->opts.codec) {
      I.coo_stream_bytes = 4 * A->coo_words;
      stream += I.coo_stream_bytes;
      meta += A->nI * (4 + 1) + 8 * (A->nI + 1);  // base_row, width, symptr
      raw_index += 4 * slots;                     // col
    } else {
      raw_index += 8 * slots;                     // row + col
      meta += 4 * A->nI;                          // interval first rows
    }
    values += slots * vs;
  }
  I.meta_bytes = meta;
  I.index_bytes = stream + raw_index + meta;
  I.value_bytes = values;
  I.device_bytes = A->device_bytes;
  I.algorithmic_bytes = I.index_bytes + values + (A->n + A->m) * vs;
  // eta of P:L246 (reading R19): O = 4*m*K (+ 8 per COO entry), C = streams
  // (+ 4 per COO entry of raw col) — counted per entry, not per padded slot
  const int64_t O = (A->has_ell ? 4 * A->m * A->K : 0) + 8 * A->nnz_coo;
  I.orig_index_bytes = O;
  const int64_t C = A->opts.codec ? stream + 4 * A->nnz_coo
                                  : (A->has_ell ? 4 * A->K * A->pitch : 0) + 8 * A->nnz_coo;
  I.eta_stream = O > 0 ? 1.0 - double(C) / double(O) : 0.0;
  I.eta_total = O > 0 ? 1.0 - double(I.index_bytes) / double(O) : 0.0;
}

// The BRO-ELL instance for this matrix (opts.ell_kernel 0 = auto, first
// match): every slice <= 4 columns -> tiny; h = 32 and fewer slices than the
// general instance keeps resident (32 warps per SM) -> few-slice; every row
// stream < 10 symbols -> small window; < 18 -> mid window; else general.
bro_status_t choose_ell_instance(bro_matrix_s* A, int sms) {
  using namespace bro;
  const int want = A->opts.ell_kernel;
  const bool tiny_ok = A->ell_max_l <= kEllTinyCols;
  const bool small_ok = A->ell_max_S < kEllRowsSmall;
  const bool mid_ok = A->ell_max_S < kEllRowsMid;
  const bool small_family = want == ELL_SMALL;
  const bool mid_family = want == ELL_MID;
  if (want == ELL_AUTO) {
    if (tiny_ok) A->ell_inst = ELL_TINY;
    else if (A->h == 32 && A->s < int64_t(sms) * 32) A->ell_inst = ELL_FEW;
    else if (small_ok) A->ell_inst = ELL_SMALL;
    else if (mid_ok) A->ell_inst = ELL_MID;
    else A->ell_inst = ELL_GEN;
    return BRO_OK;
  }
  if ((want == ELL_TINY && !tiny_ok) || (small_family && !small_ok) || (mid_family && !mid_ok))
    return fail(BRO_ERR_ARG, "ell_kernel " + std::to_string(want) + " does not fit this matrix (longest slice " +
                                 std::to_string(A->ell_max_l) + " columns, longest row stream " +
                                 std::to_string(A->ell_max_S) + " symbols)");
  A->ell_inst = want;
  return BRO_OK;
}

bro_status_t resolve(Launch& L, const bro::KernelRef& k, int sms, const char* what) {
  if (!k.fn) return fail(BRO_ERR_UNSUPPORTED, std::string("no kernel instance for ") + what);
  int per_sm = 0;
  cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k.fn, k.threads, 0);
  if (e != cudaSuccess) return fail(BRO_ERR_CUDA, std::string("occupancy query: ") + cudaGetErrorString(e));
  L.k = k;
  L.resident_blocks = int64_t(std::max(1, per_sm)) * sms;
  return BRO_OK;
}

// The x-staged few-slice instance: dynamic shared memory for the largest
// window, and only if its grid covers every slice in one pass (block b = the
// b-th group of warps-per-block slices, the group its window was cut for).
template <typename T>
bro_status_t resolve_xstage(bro_matrix_s* A, int sms) {
  const bro::KernelRef k = bro::bro_ell_xstage_ref<T>(A->opts.vec_words);
  if (!k.fn) return BRO_OK;
  cudaError_t e = cudaFuncSetAttribute(k.fn, cudaFuncAttributeMaxDynamicSharedMemorySize, A->xwin_bytes);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return BRO_OK;  // no staging on this device
  }
  int per_sm = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k.fn, k.threads, A->xwin_bytes);
  if (e != cudaSuccess || per_sm < 1) {
    cudaGetLastError();
    return BRO_OK;
  }
  const int64_t blocks = (A->s + k.warps_per_block() - 1) / k.warps_per_block();
  if (blocks > int64_t(per_sm) * sms) return BRO_OK;  // would need a second pass
  A->ell_x.k = k;
  A->ell_x.resident_blocks = int64_t(per_sm) * sms;
  A->xstage = true;
  return BRO_OK;
}

// Resolve every kernel instance of the handle on its device (current).
template <typename T>
bro_status_t resolve_kernels(bro_matrix_s* A) {
  int sms = 0;
  cudaError_t e = cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, A->device);
  if (e != cudaSuccess) return fail(BRO_ERR_CUDA, std::string("device attribute: ") + cudaGetErrorString(e));
  sms = std::max(1, sms);
  bro_status_t st = BRO_OK;
  const int V = A->opts.vec_words;
  if (A->has_ell) {
    if (A->opts.codec) {
      if ((st = choose_ell_instance(A, sms))) return st;
      for (int mode = 0; mode < 3 && !st; ++mode) {
        if (A->vi.cb && mode == 1) continue;  // value-indexed handles: no scatter epilogue
        const bro::KernelRef k = A->vi.cb && mode == 0 ? bro::bro_ell_vi_ref<T>(V, A->h / 32, A->ell_inst, A->vi.cb)
                                                        : bro::bro_ell_ref<T>(V, A->h / 32, A->ell_inst, mode);
        st = resolve(A->ell_k[mode], k, sms, "BRO-ELL");
      }
      if (!st && A->xwin_bytes > 0 && A->ell_inst == bro::ELL_FEW && !A->vi.cb) st = resolve_xstage<T>(A, sms);
    } else {
      for (int mode = 0; mode < 3 && !st; ++mode) st = resolve(A->ell_k[mode], bro::plain_ell_ref<T>(mode), sms, "ELL");
    }
  }
  if (A->has_coo && !st) {
    st = resolve(A->coo_k[0], bro::coo_ref<T>(A->opts.codec == 1, A->coo_T, 0), sms, "COO");
    if (!st) st = resolve(A->coo_k[2], bro::coo_ref<T>(A->opts.codec == 1, A->coo_T, 2), sms, "COO decode");
    if (!st) st = resolve(A->fix_k, bro::fixup_ref<T>(), sms, "COO fix-up");
  }
  if (!st) st = resolve(A->rep_k, bro::replicate_ref<T>(), sms, "replicate");
  return st;
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
  if (o.codec && o.slice_h) {
    A->h = o.slice_h;
  } else if (o.codec && m >= kAutoH64Rows && format != FMT_COO) {
    // h = 64 for big matrices whose rows fit the small- or mid-window
    // instance at h = 32 (every row stream < 18 symbols) and are not tiny:
    // two rows per lane then share the widths, offsets and setup (C5 fp32
    // 247 -> 203 us; C4 fp64 99.7 -> 97.3 us since the decode-loop cuts,
    // profiles/r02/s2/c4/)
    bro::RowsView rv;
    rv.m = m; rv.row_ptr = row_ptr; rv.col = col; rv.vsize = A->vsize; rv.cap = K;
    int64_t max_l = 0, max_S = 0;
    bro::slice_extents(rv, 32, o.min_bits, &max_l, &max_S);
    A->h = max_l > bro::kEllTinyCols && max_S < bro::kEllRowsMid ? 64 : 32;
  }
  A->opts.slice_h = A->h;
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
        bro::encode_bro_ell(rv, A->h, o.vec_words, 16 / A->vsize, o.min_bits, A->ell);
        A->s = A->ell.s;
        A->ell_words = (int64_t)A->ell.words.size();
        A->ell_slots = (int64_t)(A->ell.vals.size() / A->vsize);
        A->ell_max_l = A->ell.max_l;
        for (int64_t t = 0; t < A->s; ++t)
          A->ell_max_S = std::max<int64_t>(A->ell_max_S, int64_t(A->ell.symptr[t + 1] - A->ell.symptr[t]));
        if (o.value_codec == 1) {
          const int vr = bro::encode_value_index(rv, A->ell, A->vi);
          if (vr) {
            delete A;
            return fail(BRO_ERR_UNSUPPORTED, vr == 1 ? "value_codec 1: the BRO-ELL part holds more than 65,536 distinct values"
                                                     : "value_codec 1: the BRO-ELL part holds no finite value");
          }
        }
      } else {
        bro::build_plain_ell(rv, K, A->pell);
        A->pitch = A->pell.pitch;
      }
    }
    // COO part
    A->nnz_coo = A->nnz - A->nnz_ell;
    A->coo_T = o.coo_T ? o.coo_T : auto_coo_T(A->nnz_coo);
    A->opts.coo_T = A->coo_T;
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
        // COO lane streams always use the paper's V = 1 multiplexing (a lane's
        // word q at 32q + lane: one coalesced 128-byte row per q, staged by cp.async)
        bro::encode_bro_coo(A->nnz_coo, cr.data(), cc.data(), cv.data(), A->vsize, A->coo_T, 1, A->coo);
      else
        bro::build_plain_coo(A->nnz_coo, cr.data(), cc.data(), cv.data(), A->vsize, A->coo_T, A->coo);
      A->nI = A->coo.nI;
      A->coo_words = (int64_t)A->coo.words.size();
      // rows that span COO intervals (for the fix-up): interval i's first row
      // is cr[i*I], its last row cr[min((i+1)*I, N) - 1]
      const int64_t I = 32 * int64_t(A->coo_T), N = A->nnz_coo;
      A->coo_end_host.resize(A->nI);
      for (int64_t i = 0; i < A->nI; ++i) A->coo_end_host[i] = cr[std::min((i + 1) * I, N) - 1];
      auto base = [&](int64_t i) { return cr[i * I]; };
      for (int64_t i = 0; i + 1 < A->nI;) {
        const int32_t R = A->coo_end_host[i];
        if (base(i + 1) != R) { ++i; continue; }
        int64_t b = i + 1;
        while (b + 1 < A->nI && base(b + 1) == R) ++b;
        A->spans_host.push_back(int4{R, int(i), int(b), base(i) != R ? 1 : 0});
        i = b;
      }
      A->n_spans = int64_t(A->spans_host.size());
    }
    // x windows of the few-slice instance's blocks (row N1): BRO-ELL at h = 32
    // with fewer slices than the general instance keeps resident (148 SMs x 32)
    if (A->has_ell && o.codec && o.x_stage == 1 && A->h == 32 && A->ell_max_l > bro::kEllTinyCols &&
        A->s < kB200Warps && (o.ell_kernel == 0 || o.ell_kernel == bro::ELL_FEW) && !A->host_only) {
      const int64_t wpb = A->vsize == 8 ? 8 : 4;  // warps per block of the few-slice instance
      const int64_t E = 16 / A->vsize;            // x elements per 16 bytes
      const int64_t nb = (A->s + wpb - 1) / wpb;
      std::vector<int2> win(nb, int2{0, 0});
      int64_t maxb = 0;
      for (int64_t b = 0; b < nb; ++b) {
        int64_t lo = INT64_MAX, hi = -1;
        for (int64_t r = b * wpb * 32; r < std::min(m, (b + 1) * wpb * 32); ++r) {
          const int64_t len = std::min(K, row_ptr[r + 1] - row_ptr[r]);
          if (len <= 0) continue;
          lo = std::min<int64_t>(lo, col[row_ptr[r]]);
          hi = std::max<int64_t>(hi, col[row_ptr[r] + len - 1]);
        }
        if (hi < 0) continue;
        lo &= ~(E - 1);  // 16-byte aligned source
        int64_t cnt = (hi + 1 - lo + E - 1) / E * E;
        if (lo + cnt > n) cnt = (hi + 1 - lo) / E * E;  // never past x's end: the tail is gathered from global
        win[b] = int2{int(lo), int(cnt)};
        maxb = std::max(maxb, cnt * A->vsize);
      }
      if (maxb > 0 && maxb <= bro::kXStageMaxBytes) {
        A->xwin_host = std::move(win);
        A->xwin_bytes = int(maxb);
      }
    }
    // column range of every row block (h rows; ELL-only handles): which part
    // of x a block of rows needs, for the pipelined bro_spmv_host
    if (A->has_ell && !A->has_coo) {
      const int64_t H = A->h;
      const int64_t nb = (m + H - 1) / H;
      A->blk_cmin.assign(nb, INT32_MAX);
      A->blk_cmax.assign(nb, -1);
      for (int64_t i = 0; i < m; ++i) {
        if (row_ptr[i + 1] == row_ptr[i]) continue;
        const int64_t bi = i / H;
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
      if (A->vi.cb) {  // the codes and the table replace the values
        UP(A->d_vcodes, A->vi.codes);
        if (st == BRO_OK) st = dev_upload(A, &A->d_vdict, A->vi.dict.data(), A->vi.dict.size());
      } else if (st == BRO_OK) {
        st = dev_upload(A, &A->d_ell_vals, A->ell.vals.data(), A->ell.vals.size());
      }
    }
    if (A->xwin_bytes > 0) UP(A->d_xwin, A->xwin_host);
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
      // carries of the rows spanning intervals, the intervals' last rows and
      // the span list of the fix-up
      const size_t nU = size_t(A->nI);
      if (st == BRO_OK) st = dev_upload(A, &A->d_cf, nullptr, nU * A->vsize);
      if (st == BRO_OK) st = dev_upload(A, &A->d_cl, nullptr, nU * A->vsize);
      UP(A->d_coo_end, A->coo_end_host);
      UP(A->d_spans, A->spans_host);
    }
#undef UP
    if (st == BRO_OK) st = dtype == BRO_FP64 ? resolve_kernels<double>(A) : resolve_kernels<float>(A);
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
    A->coo_end_host = std::vector<int32_t>();
    A->spans_host = std::vector<int4>();
    A->vi.codes = std::vector<uint8_t>();
    A->vi.dict = bro::Bytes();
  } else {
    if (A->has_ell && o.codec) {
      bro_status_t st = choose_ell_instance(A, 148);
      if (st != BRO_OK) {
        delete A;
        return st;
      }
    }
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
  bro_status_t st = check_opts(*o);
  if (st) return st;
  // vec_words 0 = auto: V = 1, the paper's multiplexing, measured fastest for
  // both dtypes once the decode loop was cut down (C5 fp32 185 vs 196 us with
  // V = 4, C3 fp32 22.8 vs 23.4, C4/C2 level; profiles/r02/s2/vec/)
  if (o->vec_words == 0) o->vec_words = 1;
  (void)dtype;
  return BRO_OK;
}

// ------------------------------------------------------------------ launches
template <typename... Args>
cudaError_t launch(const Launch& L, int64_t grid, cudaStream_t st, Args&... args) {
  if (grid <= 0) return cudaSuccess;
  void* a[] = {static_cast<void*>(&args)...};
  return cudaLaunchKernel(L.k.fn, dim3(unsigned(grid)), dim3(unsigned(L.k.threads)), a, 0, st);
}

template <typename... Args>
cudaError_t launch_smem(const Launch& L, int64_t grid, size_t smem, cudaStream_t st, Args&... args) {
  if (grid <= 0) return cudaSuccess;
  void* a[] = {static_cast<void*>(&args)...};
  return cudaLaunchKernel(L.k.fn, dim3(unsigned(grid)), dim3(unsigned(L.k.threads)), a, smem, st);
}

// Launch as a programmatic dependent of the previous kernel on the stream
// (PDL): it may start while that kernel drains; it waits (griddepcontrol.wait)
// before touching what that kernel writes.
template <typename... Args>
cudaError_t launch_pdl(const Launch& L, int64_t grid, cudaStream_t st, Args&... args) {
  if (grid <= 0) return cudaSuccess;
  void* a[] = {static_cast<void*>(&args)...};
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(unsigned(grid));
  cfg.blockDim = dim3(unsigned(L.k.threads));
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelExC(&cfg, L.k.fn, a);
}

// Persistent grids: as many blocks as the device keeps resident, capped by the work.
int64_t persistent_grid(const Launch& L, int64_t units) {
  const int64_t w = L.k.warps_per_block();
  return std::min((units + w - 1) / w, L.resident_blocks);
}

template <typename T>
bro::dev::YOut<T> make_yout(T* y) {
  bro::dev::YOut<T> o{};
  o.p[0] = y;
  o.n = 1;
  return o;
}

// ELL part over the row blocks [b0, b1) (slices of BRO-ELL, h-row blocks of
// ELLPACK): the slice metadata / plain rows are addressed from the block, y
// from its first row.  mode: 0 spmv, 1 scatter, 2 decode (dec = output).
template <typename T>
cudaError_t launch_ell(const bro_matrix_s* A, int mode, const T* x, const bro::dev::YOut<T>& yo, int32_t* dec,
                       int64_t b0, int64_t b1, cudaStream_t st) {
  const int64_t H = A->h;
  const int64_t r0 = H * b0, r1 = std::min(A->m, H * b1);
  if (r1 <= r0) return cudaSuccess;
  bro::dev::YOut<T> y = yo;
  if (b0 > 0)
    for (int i = 0; i < y.n; ++i) y.p[i] += r0;
  if (b0 > 0 && y.mc) y.mc += r0;
  const Launch& L = A->ell_k[mode];
  if (A->opts.codec) {
    bro::dev::EllDev<T> p{r1 - r0, b1 - b0, A->d_words, A->d_bit_alloc, A->d_colptr + b0, A->d_symptr + b0,
                          static_cast<const T*>(A->d_ell_vals), x, A->d_xwin, A->d_vcodes,
                          static_cast<const T*>(A->d_vdict), uint32_t(A->vi.pz)};
    if (!L.k.fn) return cudaErrorNotSupported;  // scatter on a value-indexed handle
    // whole part, plain SpMV, 16-byte aligned x: the x-window-staged instance
    if (A->xstage && mode == 0 && b0 == 0 && b1 == A->s && (reinterpret_cast<uintptr_t>(x) & 15) == 0) {
      const int64_t w = A->ell_x.k.warps_per_block();
      return launch_smem(A->ell_x, (p.s + w - 1) / w, size_t(A->xwin_bytes), st, p, y, dec);
    }
    // split instances: several warps per slice
    const int64_t parts = A->h == 32 ? (A->ell_inst == bro::ELL_SPLIT ? 4 : A->ell_inst == bro::ELL_SPLIT2 ? 2 : 1) : 1;
    return launch(L, persistent_grid(L, p.s * parts), st, p, y, dec);
  }
  // decode mode covers the padding rows [m, pitch) too (they hold -1)
  const int64_t rows = mode == 2 && b0 == 0 ? A->pitch : r1 - r0;
  bro::dev::PellDev<T> p{rows, A->K, A->pitch, A->d_pell_col + r0, static_cast<const T*>(A->d_ell_vals) + r0, x};
  return launch(L, (p.m + L.k.threads - 1) / L.k.threads, st, p, y, dec);
}

template <typename T>
bro::dev::CooDev<T> coo_dev(const bro_matrix_s* A, const T* x) {
  return bro::dev::CooDev<T>{A->nnz_coo, A->nI, A->d_coo_words, A->d_coo_base, A->d_coo_width, A->d_coo_symptr,
                            A->d_coo_row, A->d_coo_col, static_cast<const T*>(A->d_coo_vals), x,
                            static_cast<T*>(A->d_cf), static_cast<T*>(A->d_cl), A->d_coo_end};
}

int64_t coo_grid(const bro_matrix_s* A, const Launch& L) {
  const int64_t w = L.k.warps_per_block();
  return (A->nI + w - 1) / w;  // one warp per interval
}

// y = A.x stored into every destination of yo (yo.p[0] = the local y on A's
// device).  ELL-only handles store all destinations from the ELL kernel's
// epilogue (fused exchange); handles with a COO part finish y locally and
// then replicate it (the COO part and the fix-up add into y).
template <typename T>
bro_status_t launch_spmv(bro_matrix_s* A, const T* x, const bro::dev::YOut<T>& yo, cudaStream_t st) {
  T* y = yo.p[0];
  const bool multi = yo.n > 1 || yo.mc != nullptr;
  const bool fused = !(A->has_coo && A->nI > 0);
  cudaError_t e = cudaSuccess;
  if (A->has_ell) {
    const int64_t nb = A->opts.codec ? A->s : (A->m + A->h - 1) / A->h;
    e = launch_ell<T>(A, fused && multi ? 1 : 0, x, fused ? yo : make_yout(y), nullptr, 0, nb, st);
  } else if (A->m > 0) {
    e = cudaMemsetAsync(y, 0, size_t(A->m) * sizeof(T), st);
  }
  if (e == cudaSuccess && A->has_coo && A->nI > 0) {
    bro::dev::CooDev<T> p = coo_dev<T>(A, x);
    int32_t* none = nullptr;
    // the COO kernel overlaps the ELL kernel's tail, the fix-up the COO
    // kernel's (programmatic dependent launches, bro_opts_t.pdl)
    const bool pdl = A->opts.pdl != 2;
    const bool after_ell = A->has_ell && pdl;
    e = after_ell ? launch_pdl(A->coo_k[0], coo_grid(A, A->coo_k[0]), st, p, y, none)
                  : launch(A->coo_k[0], coo_grid(A, A->coo_k[0]), st, p, y, none);
    if (e == cudaSuccess && A->n_spans > 0) {  // rows spanning intervals
      int64_t nS = A->n_spans;
      const int4* sp = A->d_spans;
      const T* cf = static_cast<const T*>(A->d_cf);
      const T* cl = static_cast<const T*>(A->d_cl);
      e = pdl ? launch_pdl(A->fix_k, (nS + 255) / 256, st, nS, sp, cf, cl, y)
              : launch(A->fix_k, (nS + 255) / 256, st, nS, sp, cf, cl, y);
    }
  }
  if (e == cudaSuccess && !fused && A->m > 0 && multi) {
    int64_t m = A->m;
    bro::dev::YOut<T> o = yo;
    e = launch(A->rep_k, std::min<int64_t>((A->m + 255) / 256, 148 * 8), st, m, o);
  }
  if (e == cudaSuccess) e = cudaGetLastError();
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
  const size_t H = size_t(A->h);
  const size_t slots = size_t(A->nI) * 32 * A->coo_T;
  auto set = [&](const void* h, const void* d, size_t b) { v.host = h; v.dev = d; v.bytes = b; };
  switch (part) {
    case BRO_PART_ELL_WORDS: if (bro_ell) set(A->ell.words.data(), A->d_words, 4 * size_t(A->ell_words)); break;
    case BRO_PART_ELL_BIT_ALLOC: if (bro_ell) set(A->ell.bit_alloc.data(), A->d_bit_alloc, size_t(A->ell_slots) / H); break;
    case BRO_PART_ELL_COLPTR: if (bro_ell) set(A->ell.colptr.data(), A->d_colptr, 8 * size_t(A->s + 1)); break;
    case BRO_PART_ELL_SYMPTR: if (bro_ell) set(A->ell.symptr.data(), A->d_symptr, 8 * size_t(A->s + 1)); break;
    case BRO_PART_ELL_VALS: if (bro_ell && !A->vi.cb) set(A->ell.vals.data(), A->d_ell_vals, vs * size_t(A->ell_slots)); break;
    case BRO_PART_ELL_VCODES: if (bro_ell && A->vi.cb) set(A->vi.codes.data(), A->d_vcodes, A->vi.codes.size()); break;
    case BRO_PART_ELL_VDICT: if (bro_ell && A->vi.cb) set(A->vi.dict.data(), A->d_vdict, A->vi.dict.size()); break;
    case BRO_PART_COO_WORDS: if (bro_coo) set(A->coo.words.data(), A->d_coo_words, 4 * size_t(A->coo_words)); break;
    case BRO_PART_COO_BASE_ROW: if (bro_coo) set(A->coo.base_row.data(), A->d_coo_base, 4 * size_t(A->nI)); break;
    case BRO_PART_COO_WIDTH: if (bro_coo) set(A->coo.width.data(), A->d_coo_width, size_t(A->nI)); break;
    case BRO_PART_COO_SYMPTR: if (bro_coo) set(A->coo.symptr.data(), A->d_coo_symptr, 8 * size_t(A->nI + 1)); break;
    case BRO_PART_COO_COL: if (coo) set(A->coo.col.data(), A->d_coo_col, 4 * slots); break;
    case BRO_PART_COO_VALS: if (coo) set(A->coo.vals.data(), A->d_coo_vals, vs * slots); break;
    case BRO_PART_COO_ROW: if (coo && !A->opts.codec) set(A->coo.row.data(), A->d_coo_row, 4 * slots); break;
    case BRO_PART_PELL_COL: if (plain_ell) set(A->pell.col.data(), A->d_pell_col, 4 * size_t(A->K * A->pitch)); break;
    case BRO_PART_PELL_VALS: if (plain_ell) set(A->pell.vals.data(), A->d_ell_vals, vs * size_t(A->K * A->pitch)); break;
    default: v.bytes = SIZE_MAX;
  }
  return v;
}

// Pipelined end-to-end SpMV of an ELL-only handle: x goes up in K pieces on
// one stream, each group of row blocks runs as soon as the pieces covering
// its columns (blk_cmin/blk_cmax) have arrived, and its y goes down on a third
// stream while later blocks compute — H2D, compute and D2H overlap (PCIe is
// full duplex).  Same kernels and per-row arithmetic as bro_spmv.
template <typename T>
bro_status_t spmv_host_pipelined(bro_matrix_s* A, const void* x_host, void* y_host, cudaStream_t st, int K) {
  const int64_t nb = int64_t(A->blk_cmax.size());
  const size_t vs = sizeof(T);
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
  const T* xs = static_cast<const T*>(A->d_xs);
  T* ys = static_cast<T*>(A->d_ys);
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
    e = launch_ell<T>(A, 0, xs, make_yout(ys), nullptr, b0, b1, st);
    if (e != cudaSuccess) return fail(BRO_ERR_CUDA, std::string("kernel launch: ") + cudaGetErrorString(e));
    cudaEventRecord(evy[c], st);
    cudaStreamWaitEvent(A->e2e_d2h, evy[c], 0);
    const int64_t r0 = A->h * b0, r1 = std::min(A->m, A->h * b1);
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
  o->slice_h = 0;
  o->sym_bits = 32;
  o->vec_words = 0;
  o->coo_T = 0;
  o->hyb_K = -1;
  o->codec = 1;
  o->min_bits = 0;
  o->ell_kernel = 0;
  o->pdl = 0;
  o->x_stage = 0;
  o->value_codec = 0;
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
  if (o.value_codec) return fail(BRO_ERR_ARG, "value_codec indexes BRO-ELL values: ELL and HYB handles only");
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
  if (A->vi.cb && !(A->has_coo && A->nI > 0) && (n_dst > 1 || y_mc))
    return fail(BRO_ERR_UNSUPPORTED, "value-indexed BRO-ELL handles have no scatter epilogue");
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
  // ELL-only handles with a large x: pipelined copies and compute
  if (A->has_ell && !A->has_coo && int64_t(A->blk_cmax.size()) >= kE2eChunks && xb >= kE2eMinBytes)
    return A->dtype == BRO_FP64 ? spmv_host_pipelined<double>(A, x_host, y_host, st, kE2eChunks)
                                : spmv_host_pipelined<float>(A, x_host, y_host, st, kE2eChunks);
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
  if (!A) return fail(BRO_ERR_ARG, "matrix is NULL");
  if (A->host_only) return fail(BRO_ERR_UNSUPPORTED, "host-only handle has no device copy");
  DeviceGuard g(A->device);
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  cudaError_t e = cudaSuccess;
  // the handle's own instances in decode mode: same staging, offsets and
  // extraction as bro_spmv, the decoded index stored instead of the FMA
  auto run = [&](auto* tag) {
    using T = std::remove_pointer_t<decltype(tag)>;
    if (d_ell_cols && A->has_ell) {
      const int64_t nb = A->opts.codec ? A->s : (A->m + A->h - 1) / A->h;
      if (A->opts.codec || A->K > 0) e = launch_ell<T>(A, 2, nullptr, make_yout<T>(nullptr), d_ell_cols, 0, nb, st);
    }
    if (e == cudaSuccess && d_coo_rows && A->has_coo && A->nI > 0) {
      bro::dev::CooDev<T> p = coo_dev<T>(A, nullptr);
      T* none = nullptr;
      e = launch(A->coo_k[2], coo_grid(A, A->coo_k[2]), st, p, none, d_coo_rows);
    }
  };
  if (A->dtype == BRO_FP64) run((double*)nullptr);
  else run((float*)nullptr);
  if (e == cudaSuccess) e = cudaGetLastError();
  if (e != cudaSuccess) return fail(BRO_ERR_CUDA, std::string("decode launch: ") + cudaGetErrorString(e));
  return BRO_OK;
}

bro_status_t bro_hyb_K(int64_t m, const int64_t* row_ptr, int64_t* K_out) {
  if (!row_ptr || !K_out || m < 0) return fail(BRO_ERR_ARG, "bad argument");
  *K_out = bro::hyb_K(m, row_ptr);
  return BRO_OK;
}

bro_status_t bro_reorder_bar(int64_t m, int64_t n, const int64_t* row_ptr, const int32_t* col_idx,
                             bro_dtype_t dtype, int32_t method, int32_t window, int64_t* perm_out) {
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
      if (window < 0) return fail(BRO_ERR_ARG, "window must be >= 0");
      bro::bar_window_order(m, row_ptr, col_idx, dtype == BRO_FP64 ? 8 : 4, window ? window : kBarWindow, perm_out);
      return BRO_OK;
    }
    if (method == 3) {  // Algorithm 2 windowed, line 2's sequence = the signature order (R27)
      if (window < 0) return fail(BRO_ERR_ARG, "window must be >= 0");
      std::vector<int64_t> seed(m);
      bro::bar_signature_order(m, row_ptr, col_idx, seed.data());
      bro::bar_window_order(m, row_ptr, col_idx, dtype == BRO_FP64 ? 8 : 4, window ? window : kBarWindow, perm_out,
                            seed.data());
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
  return fail(BRO_ERR_ARG, "method must be 0, 1, 2 or 3");
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
