/*
 * bro.h — C ABI of the B200-native BRO SpMV library (libbro.so).
 *
 * Implements the data-parallel hot path of Tang et al., "Accelerating Sparse
 * Matrix-Vector Multiplication on GPUs using Bit-Representation-Optimized
 * Schemes", SC'13:  y = A.x  over BRO-ELL (Alg. 1
 * P:L128-138), BRO-COO and BRO-HYB, plus the
 * uncompressed ELLPACK / COO / HYB baselines the paper compares against
 * (P:L51-81).
 *
 * Problem statement followed by the boundary:
 *   - A is fixed across the iterations of an iterative solver, so compression
 *     runs ONCE, offline, on the host, inside bro_create_*;
 *   - decompression runs online on the GPU, inside every bro_spmv;
 *   - host<->device transfers are not part of bro_spmv (bro_spmv_host is the
 *     end-to-end variant that includes them).
 *
 * Conventions
 *   - All functions are extern "C", never throw, and return bro_status_t.
 *     On error a thread-local message is available from bro_last_error().
 *   - Matrices are given as canonical CSR: row_ptr int64[m+1] with
 *     row_ptr[0] = 0 and non-decreasing; col_idx int32[nnz] 0-based, in
 *     [0, n) and STRICTLY increasing within each row (a repeated column would
 *     encode a zero delta, which BRO-ELL reserves for "invalid");
 *     vals float or double [nnz] (dtype).  m, n < 2^31.
 *   - Host input arrays are borrowed only for the duration of the call (they
 *     are validated, encoded and copied; the caller keeps ownership).
 *   - A handle owns all of its device memory until bro_destroy.
 *   - Device vectors passed to bro_spmv are caller-owned, of the handle's
 *     dtype, resident on the handle's device: x has n elements, y has m.
 *   - bro_stream_t is a cudaStream_t (struct CUstream_st*); NULL means the
 *     legacy default stream.  PyTorch passes
 *     torch.cuda.current_stream().cuda_stream.
 *
 * Encoded layout (bit-exact):
 *   BRO-ELL, slice height h = 32 or 64 rows (opts.slice_h; one warp per
 *   slice, h/32 rows per lane), sym_len = 32:
 *     colptr[t]  = sum_{t'<t} l_t'       (l_t = num_col of slice t)
 *     symptr[t]  = sum_{t'<t} S_t'       (S_t = 32-bit symbols per row stream)
 *     bit_alloc[colptr[t] + j] = b_{t,j} (b_p implied by S_t)
 *     symbol q of row r of slice t at words[h*symptr[t] + place(r,q,S_t,V)]
 *     value of slot (r,j) of slice t at vals[h*colptr[t] + place(r,j,l_t,Vv)]
 *     place(r,q,S,V) = h*V*(q/V) + r*V + q%V          if q/V < S/V
 *                    = h*V*F + r*(S-V*F) + (q-V*F)    otherwise (F = S/V)
 *     V = opts.vec_words (1 = the paper's comp_str_i[q*h+tid]), Vv = 16/sizeof(val).
 *     Row streams are concatenated b-bit deltas, most significant bit first,
 *     delta_0 = col_0 + 1, delta_j = col_j - col_{j-1}, 0 = padding.
 *   BRO-COO, intervals of 32*T entries (T = 8, 16 or 32): lane l of interval
 *     i owns the T consecutive entries e = i*32*T + T*l + t (DESIGN.md
 *     reading R13); deltas follow entry order, delta(e) = row(e) - row(e-1),
 *     delta of the first entry 0, base_row[i] = row of the first entry, one
 *     width width[i] per interval; lane l's T fields, MSB first,
 *     padded to S_i = ceil(T*width/32) symbols at
 *     coo_words[32*coo_symptr[i] + 32*q + l] (the paper's V = 1 multiplexing,
 *     whatever opts.vec_words says).
 *     col / vals (and plain COO rows) are stored per interval in the same
 *     lane-contiguous order in 16-byte chunks (reading R26): entry (l, t) at
 *     [i*32*T + place(l,t,T,C)], C = 4 for int32, 16/sizeof(val) for values;
 *     slots past nnz hold col 0 / value 0 (plain rows: the last row).
 *
 * Thread safety: distinct handles may be used concurrently.  A handle holds
 * per-call scratch (the COO carries, the bro_spmv_host buffers): at most ONE
 * call on a handle may be in flight at a time — serialize its calls on one
 * stream (or synchronize between streams), and never use it from two threads
 * at once.
 */
#ifndef BRO_H_
#define BRO_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define BRO_VERSION 1
/* device id that builds a host-only handle: encoded on the host, exportable,
 * never uploaded; bro_spmv on it returns BRO_ERR_UNSUPPORTED (no CPU path). */
#define BRO_DEVICE_HOST_ONLY (-1)

typedef struct bro_matrix_s* bro_matrix_t;
typedef struct CUstream_st* bro_stream_t;

typedef enum { BRO_FP32 = 0, BRO_FP64 = 1 } bro_dtype_t;

typedef enum {
  BRO_OK = 0,
  BRO_ERR_ARG = 1,         /* null pointer, bad option, aliasing x == y, buffer too small */
  BRO_ERR_INDEX = 2,       /* column out of range, unsorted or repeated column, bad row_ptr */
  BRO_ERR_SHAPE = 3,       /* m or n out of range (>= 2^31 or negative) */
  BRO_ERR_OOM = 4,         /* host or device allocation failed */
  BRO_ERR_CUDA = 5,        /* a CUDA runtime call or kernel launch failed */
  BRO_ERR_UNSUPPORTED = 6  /* option or operation not supported by this handle */
} bro_status_t;

typedef struct {
  int32_t slice_h;   /* BRO-ELL slice height h (a parameter of the method):
                        32 (one row per lane of the slice's warp), 64 (two rows per lane:
                        widths, offsets and setup shared by both rows), 0 (default) =
                        auto: 64 when m >= 303,104 (64 rows x 32 resident warps x 148
                        SMs: every resident warp of a B200 still gets slices), some
                        row of the ELL part has more than 4 entries and, at h = 32,
                        every row stream has fewer than 18 symbols; else 32.
                        bro_info_t.slice_h reports the value. */
  int32_t sym_bits;  /* sym_len. Must be 32. */
  int32_t vec_words; /* V: 1 or 4 symbols per lane chunk.  1 = the paper's multiplexing
                        (comp_str_i[q*h + tid]); 4 = 16-byte per-lane chunks (128-bit loads);
                        0 (default) = auto: 1 for both dtypes (measured fastest on B200). */
  int32_t coo_T;     /* BRO-COO entries per lane of an interval (interval = 32*T entries):
                        8, 16 or 32; 0 (default) = 8 (measured fastest on B200 for both
                        BRO-COO and plain COO: the kernels are latency-bound). */
  int64_t hyb_K;     /* HYB dividing column; -1 = the "less than a third" rule. */
  int32_t codec;     /* 1 = BRO compressed formats; 0 = uncompressed ELL/COO/HYB baseline. */
  int32_t min_bits;  /* 0 = natural widths; k in [1, 31] forces every BRO-ELL width
                        b_j = max(Gamma, k) — the simulated compression ratios of the
                        Fig. 3 experiment ("the number of bits allocated to each
                        index value ... was varied"). */
  int32_t ell_kernel;/* BRO-ELL kernel instance: 0 (default) = chosen at create from the
                        matrix shape; 1 tiny (every slice <= 4 columns), 2 few-slice
                        (h = 32), 3 small window (every row stream < 10 symbols), 4 mid
                        window (< 18), 5 general, 6 / 7 split slices (h = 32: 4 / 2 warps
                        share each slice, each owning a range of its columns and
                        decoding the columns before it without gathering; the block adds
                        the partial sums in part order — the "multiple threads per row"
                        of P:L416; at h = 64 they run the general instance).  An
                        instance the matrix does not fit gives BRO_ERR_ARG.  For A/B
                        measurements and tests. */
  int32_t pdl;       /* HYB / COO: 0 (default) = 1 = the COO kernel is launched as a
                        programmatic dependent of the ELL kernel (its loads, decode and x
                        gathers overlap the ELL kernel's tail; it waits before updating y),
                        and the fix-up as one of the COO kernel; 2 = plain stream order. */
  int32_t x_stage;   /* few-slice BRO-ELL instance (h = 32, fewer slices than 148 x 32):
                        1 = each block has the TMA engine copy its x column window
                        (<= 96 KB) into shared memory and gathers from there, when the
                        window fits and one pass of blocks covers the matrix
                        (bro_info_t.x_stage_bytes > 0); 0 (default) = gathers through
                        L1/L2 (measured faster on C2: 19.5 vs 22.6 us fp64). */
  int32_t value_codec;/* BRO-ELL values (codec 1, ELL and HYB handles): 0 (default) = stored
                        as they are (the paper's BRO formats); 1 = value indexing, the
                        "value data compression" named as future work by the
                        value-index method of the work the paper cites for it ([16],
                        P:L408; reading R28): the ELL part's distinct value
                        bit patterns (sorted as unsigned integers) in a table and one
                        1-byte (<= 256 distinct) or 2-byte (<= 65,536) code per slot,
                        slot (r, j) of slice t at h*colptr[t] + place(r, j, l_t, 4/cb, h);
                        padding slots hold the code of the first finite value of the
                        table.  Lossless bit for bit.  More than 65,536 distinct values, or
                        no finite value at all, gives
                        BRO_ERR_UNSUPPORTED; on a COO handle, BRO_ERR_ARG.  Value-indexed
                        ELL handles have no scatter
                        epilogue (bro_spmv_scatter with more than one destination gives
                        BRO_ERR_UNSUPPORTED); the COO part of a HYB handle keeps its values. */
} bro_opts_t;

typedef struct {
  int64_t m, n, nnz;
  int32_t dtype;              /* bro_dtype_t */
  int32_t codec;              /* 1 BRO, 0 uncompressed */
  int32_t format;             /* 0 ELL, 1 COO, 2 HYB */
  int32_t vec_words;
  int32_t slice_h;            /* BRO-ELL slice height (32 or 64) */
  int32_t coo_T;              /* BRO-COO entries per lane of an interval */
  int32_t ell_kernel;         /* BRO-ELL kernel instance resolved at create (see bro_opts_t) */
  int32_t x_stage_bytes;      /* shared memory per block of the x-staged instance (0: not staged) */
  int64_t K;                  /* ELL width bound: HYB K, or max row length for ELL */
  int64_t nnz_ell, nnz_coo;   /* entries in the ELL part and in the COO part */
  int64_t n_slices;           /* BRO-ELL slices s = ceil(m/h) (0 without an ELL part) */
  int64_t ell_slots;          /* value slots of the ELL part: h*colptr[s] (BRO) or K*pitch (plain) */
  int64_t ell_pitch;          /* plain ELL column pitch (m rounded up to 32) */
  int64_t n_intervals;        /* COO intervals ceil(nnz_coo / (32*T)) */
  int64_t ell_stream_bytes;   /* BRO-ELL compressed words (C of P:L246 for the ELL part) */
  int64_t coo_stream_bytes;   /* BRO-COO compressed row words */
  int64_t meta_bytes;         /* colptr, symptr, bit_alloc, COO headers */
  int64_t index_bytes;        /* all stored index data: streams + raw col/row arrays + metadata */
  int64_t value_bytes;        /* stored values including ELL padding */
  int64_t device_bytes;       /* device memory held by the handle */
  int64_t algorithmic_bytes;  /* bytes one bro_spmv must move: stored arrays + n*sizeof(x) + m*sizeof(y) */
  int64_t orig_index_bytes;   /* O of P:L246: 4*m*K (+ 8*nnz_coo for HYB/COO) */
  double eta_stream;          /* 1 - C/O, C = compressed streams (+ raw COO col for HYB) */
  double eta_total;           /* 1 - index_bytes/O (metadata included) */
  double encode_seconds;      /* host time spent validating + encoding */
  int32_t value_code_bytes;   /* value-indexed handles: bytes per code (1 or 2), else 0 */
  int32_t reserved0;
  int64_t value_dict_size;    /* value-indexed handles: distinct values |D| in the table, else 0 */
} bro_info_t;

/* Parts of the encoded representation, for bro_export_encoded. */
typedef enum {
  BRO_PART_ELL_WORDS = 0,     /* uint32[h*symptr[s]]   BRO-ELL multiplexed stream */
  BRO_PART_ELL_BIT_ALLOC = 1, /* uint8[colptr[s]]      per-slice per-column widths */
  BRO_PART_ELL_COLPTR = 2,    /* uint64[s+1] */
  BRO_PART_ELL_SYMPTR = 3,    /* uint64[s+1] */
  BRO_PART_ELL_VALS = 4,      /* value[h*colptr[s]]    sliced, interleaved, padding 0 */
  BRO_PART_COO_WORDS = 5,     /* uint32[32*coo_symptr[nI]] */
  BRO_PART_COO_BASE_ROW = 6,  /* uint32[nI] */
  BRO_PART_COO_WIDTH = 7,     /* uint8[nI] */
  BRO_PART_COO_SYMPTR = 8,    /* uint64[nI+1] */
  BRO_PART_COO_COL = 9,       /* int32[nI*32*T]  lane-contiguous chunks (reading R26), 0 past nnz */
  BRO_PART_COO_VALS = 10,     /* value[nI*32*T]  same arrangement, 0 past nnz */
  BRO_PART_COO_ROW = 11,      /* int32[nI*32*T]  plain COO rows (codec 0), last row past nnz */
  BRO_PART_PELL_COL = 12,     /* int32[K*pitch]  plain ELL, column-major, -1 = padding (codec 0) */
  BRO_PART_PELL_VALS = 13,    /* value[K*pitch]  plain ELL values (codec 0) */
  BRO_PART_ELL_VCODES = 14,   /* uint8/uint16[h*colptr[s]]  value codes (value_codec 1), 4-byte chunks */
  BRO_PART_ELL_VDICT = 15     /* value[|D|]  distinct values, bit patterns ascending (value_codec 1) */
} bro_part_t;

/* Fill *opts with the defaults: h 0 (auto), sym 32, V 0 (auto), T 0 (auto),
 * K auto, codec 1, min_bits 0, ell_kernel 0 (auto). */
void bro_opts_default(bro_opts_t* opts);

/* Build an ELL-only matrix (BRO-ELL if opts->codec == 1, else ELLPACK with
 * K = max row length).  device = CUDA ordinal or BRO_DEVICE_HOST_ONLY.
 * opts may be NULL (defaults).  On success *out owns the encoded matrix. */
bro_status_t bro_create_ell(int device, bro_dtype_t dtype, int64_t m, int64_t n,
                            const int64_t* row_ptr, const int32_t* col_idx,
                            const void* vals, const bro_opts_t* opts, bro_matrix_t* out);

/* Build a COO-only matrix (BRO-COO / plain COO).  Entries must be sorted by
 * (row, col) with strictly increasing columns within a row. */
bro_status_t bro_create_coo(int device, bro_dtype_t dtype, int64_t m, int64_t n, int64_t nnz,
                            const int32_t* row_idx, const int32_t* col_idx,
                            const void* vals, const bro_opts_t* opts, bro_matrix_t* out);

/* Build a HYB matrix: the first K entries of every row in (BRO-)ELL, the rest
 * in (BRO-)COO, K from opts->hyb_K or the rule of P:L81 (see bro_hyb_K). */
bro_status_t bro_create_hyb(int device, bro_dtype_t dtype, int64_t m, int64_t n,
                            const int64_t* row_ptr, const int32_t* col_idx,
                            const void* vals, const bro_opts_t* opts, bro_matrix_t* out);

/* y = A.x on `stream` (asynchronous).  y is overwritten (never accumulated);
 * rows without entries get 0 (Alg. 1 line 22).  x and y must not alias.
 * Launch errors are returned; device faults surface at the next sync. */
bro_status_t bro_spmv(bro_matrix_t A, const void* x_dev, void* y_dev, bro_stream_t stream);

/* Maximum number of y destinations of bro_spmv_scatter. */
#define BRO_MAX_DST 8

/* y = A.x stored into several destinations at once: the fused exchange of
 * the row-block iteration (BASELINE.json north_star: "x replicated via an
 * allgather per iteration, as in a CG loop").
 *   y_dsts  HOST array of n_dst (1..BRO_MAX_DST) DEVICE pointers, each to m
 *           values of the handle's dtype.  y_dsts[0] is the local y on the
 *           handle's device; the others may be any addresses that device can
 *           store to — typically this rank's block inside every peer GPU's
 *           x replica, peer-mapped through symmetric memory over NVLink.
 *           The array is read during the call only.
 *   y_mc    NULL, or an NVLS multicast address (m values) bound to every
 *           replica including y_dsts[0]'s memory: stores then go once
 *           through multimem.st and the switch fans them out.
 * For ELL-only handles (BRO-ELL, ELLPACK) the kernel's epilogue stores every
 * destination (no separate copy); handles with a COO part (COO, HYB) finish
 * y in y_dsts[0] and then replicate it (the COO part adds into y).
 * Asynchronous on `stream`; completion on a PEER is not signalled: the
 * caller orders readers after a cross-GPU barrier.  x must not alias any
 * destination.  Errors: BRO_ERR_ARG (n_dst out of range, NULL or aliasing
 * pointers), BRO_ERR_UNSUPPORTED (host-only handle), BRO_ERR_CUDA. */
bro_status_t bro_spmv_scatter(bro_matrix_t A, const void* x_dev, void* const* y_dsts, int32_t n_dst,
                              void* y_mc, bro_stream_t stream);

/* End-to-end y = A.x with HOST vectors: copies x (n values) host->device,
 * runs bro_spmv, copies y (m values) device->host and synchronizes `stream`.
 * Pinned host memory gives full PCIe bandwidth; pageable memory works.
 * ELL-only handles (BRO-ELL, ELLPACK) with x of at least 4 MB pipeline the
 * three steps in 8 pieces: x goes up on an internal stream, each block of
 * slices runs on `stream` as soon as the pieces covering its columns have
 * arrived, and its y goes down on a second internal stream while later
 * blocks compute.  The result is identical to bro_spmv's.  Returns after all
 * of it has completed. */
bro_status_t bro_spmv_host(bro_matrix_t A, const void* x_host, void* y_host, bro_stream_t stream);

/* Release the handle and all of its memory.  NULL is accepted. */
bro_status_t bro_destroy(bro_matrix_t A);

/* Sizes, byte counts and space savings of the encoded matrix. */
bro_status_t bro_get_info(bro_matrix_t A, bro_info_t* info);

/* Copy one encoded part to host memory.  If host_buf is NULL, *nbytes
 * receives the size; otherwise *nbytes must be >= the size and receives it.
 * Parts absent from this handle have size 0. */
bro_status_t bro_export_encoded(bro_matrix_t A, int32_t part, void* host_buf, size_t* nbytes);

/* GPU decode of the index streams, through the SAME kernel instances and
 * decode arithmetic as bro_spmv (their decode mode stores the decoded index
 * where bro_spmv would multiply): d_ell_cols (int32[info.ell_slots], may be
 * NULL) receives the decoded column of every ELL slot in V = 1 slot order —
 * slot h*colptr[t] + h*j + r for BRO-ELL, j*pitch + r for plain ELL — or -1
 * for padding; d_coo_rows (int32[nnz_coo], may be NULL) receives every COO
 * entry's row in COO order.  Asynchronous on `stream`. */
bro_status_t bro_decode_indices(bro_matrix_t A, int32_t* d_ell_cols, int32_t* d_coo_rows,
                                bro_stream_t stream);

/* The HYB dividing column K = min{k >= 0 : 3*|{i : len_i > k}| < m}
 * ("less than a third", pinned by the split of P:L79).  Host only. */
bro_status_t bro_hyb_K(int64_t m, const int64_t* row_ptr, int64_t* K_out);

/* BRO-aware row reordering (Sec. 3.4), host only.  Writes a
 * permutation perm[m] (row i of A' = row perm[i] of A, A' = P.A).
 * method 0 = signature clustering (stable sort by
 * row length then by the bit-width signature of the row's deltas, O(nnz log m));
 * method 1 = Algorithm 2 greedy on Eqn. (1) with h = w = 32, alpha = sym_len = 32 and
 * Omega(c) = 128-byte line of x[c] for the dtype (O(m^2 k / h); m <= 65536,
 * else BRO_ERR_UNSUPPORTED);
 * method 2 = Algorithm 2 with a candidate window (reading R24): line 11's
 * argmin runs over the W non-full partitions nearest to the row's own partition
 * floor(pos/32) in length-sorted order (O(m k W), any m; W >= v equals method 1);
 * W = window, 0 = 64 (ignored by methods 0 and 1);
 * method 3 = method 2 with line 2's length sort replaced by the method-0 signature order
 * (reading R27): the greedy refines the signature clusters by Eqn (1).
 * Partitions hold 32 rows except the last. */
bro_status_t bro_reorder_bar(int64_t m, int64_t n, const int64_t* row_ptr, const int32_t* col_idx,
                             bro_dtype_t dtype, int32_t method, int32_t window, int64_t* perm_out);

const char* bro_status_str(bro_status_t s);
/* Message of the last failed call on this thread ("" if none). */
const char* bro_last_error(void);
int bro_version(void);

#ifdef __cplusplus
}
#endif
#endif /* BRO_H_ */
