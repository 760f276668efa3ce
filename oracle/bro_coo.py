"""BRO-COO encoder/decoder (§3.2).

Test infrastructure only (see oracle/__init__.py).

What the text fixes:
  * only row_idx is compressed; col_idx and vals keep their values;
  * the row data is divided into intervals, each processed by one warp;
  * each interval is organised as a 2D array whose row index increases
    monotonically in the vertical direction, delta-encoded, bit-packed with
    ONE width per interval (stored in bit_alloc), then multiplexed as in
    BRO-ELL.

Fig. 2, which shows the arrangement, is an image absent from PAPER.md, so
the rest is reading R13 of DESIGN.md (the consecutive-delta arrangement of
SURVEY §8(f) NEXT-4):
  * intervals of I = 32*T entries (T = 8, 16 or 32 entries per lane);
  * lane l of interval i owns the T CONSECUTIVE entries
        e(l, t) = i*I + T*l + t,      t = 0 .. T-1,
    i.e. the 2D array R[t][l] = row(e(l, t)) is filled column by column,
    so the row index increases down every column (t) and from each column
    to the next (l);
  * delta encoding follows the entries' order e:
        delta(l, t) = row(e) - row(e - 1),   delta(0, 0) = 0,
    base_row[i] = row(i*I) (the row of the interval's first entry), so the
    row of entry e is base_row + the prefix sum of the deltas up to e (a
    lane-local sum plus a cross-lane scan of the lane totals);
  * positions past the last entry repeat the last row (delta 0);
  * b_i = Gamma(max delta) (0 allowed: one row per interval); lane l's
    stream is its T fields of b_i bits, MSB first, padded to
    S_i = ceil(T*b_i/32) symbols and multiplexed with BRO-ELL's place();
  * col and vals are stored in the same lane-contiguous arrangement,
    multiplexed for 16-byte chunk loads exactly like BRO-ELL's values
    (P:L116's multiplexing applied to the raw arrays, reading R26): entry
    (l, t) of interval i sits at i*I + place(l, t, T, Vc) with Vc = 4 for
    col (int32) and Vv = 16/sizeof(value) for vals; slots past the last
    entry hold col 0 and value 0.
The plain COO baseline uses the same arrangement with the rows stored
explicitly (int32, Vc = 4).
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

from .bro_ell import gamma, place


@dataclass
class BroCoo:
    nnz: int
    T: int
    V: int
    base_row: np.ndarray    # uint32[nI]
    width: np.ndarray       # uint8[nI]   (bit_alloc of P:L140, one per interval)
    symptr: np.ndarray      # uint64[nI+1] per-lane words before interval i
    words: np.ndarray       # uint32[32*symptr[nI]]
    col: np.ndarray         # int32[nI*I]  (lane-contiguous, chunk-multiplexed)
    vals: np.ndarray        # [nI*I]

    @property
    def n_intervals(self) -> int:
        return int(self.base_row.size)

    def stream_bytes(self) -> int:
        return int(32 * int(self.symptr[-1]) * 4)


def entry(i, lane, t, T):
    """COO entry held by lane `lane` at step t of interval i (lane-contiguous)."""
    return i * 32 * T + T * lane + t


def interval_rows(rows, i, T):
    """The 2D row array of interval i as R[lane][t] (positions past the end
    repeat the last row)."""
    N = len(rows)
    return [[int(rows[min(entry(i, lane, t, T), N - 1)]) for t in range(T)] for lane in range(32)]


def interval_deltas(R, base):
    """delta(l, t) = row(e) - row(e - 1) in entry order, delta(0, 0) = 0."""
    D = []
    prev = base
    for lane in range(32):
        d = []
        for t in range(len(R[lane])):
            d.append(R[lane][t] - prev)
            prev = R[lane][t]
        D.append(d)
    return D


def arrange(a, T, chunk, fill):
    """Lane-contiguous, chunk-multiplexed copy of a per-entry array:
    out[i*I + place(l, t, T, chunk)] = a[entry(i, l, t)], `fill` past the end."""
    a = np.asarray(a)
    N = a.size
    I = 32 * T
    nI = -(-N // I)
    out = np.full(nI * I, fill, dtype=a.dtype)
    for i in range(nI):
        for lane in range(32):
            for t in range(T):
                e = entry(i, lane, t, T)
                if e < N:
                    out[i * I + place(lane, t, T, chunk, 32)] = a[e]
    return out


def unarrange(b, N, T, chunk):
    """Inverse of arrange (first N entries, in COO order)."""
    I = 32 * T
    out = np.zeros(N, dtype=np.asarray(b).dtype)
    for e in range(N):
        i, r = divmod(e, I)
        lane, t = divmod(r, T)
        out[e] = b[i * I + place(lane, t, T, chunk, 32)]
    return out


def value_chunk(itemsize: int) -> int:
    return 16 // int(itemsize)


def encode(rows, cols, vals, T=32, V=4, sym_len=32) -> BroCoo:
    """Encode COO entries already sorted by (row, col)."""
    rows = np.asarray(rows, dtype=np.int64)
    vals = np.asarray(vals)
    N = rows.size
    I = 32 * T
    nI = -(-N // I)
    base_row = np.zeros(nI, dtype=np.uint32)
    width = np.zeros(nI, dtype=np.uint8)
    symptr = np.zeros(nI + 1, dtype=np.uint64)
    streams = []
    for i in range(nI):
        R = interval_rows(rows, i, T)
        base = R[0][0]
        D = interval_deltas(R, base)
        b = max(gamma(D[lane][t]) for lane in range(32) for t in range(T))
        S = -(-(T * b) // sym_len)
        lane_syms = []
        for lane in range(32):
            stream = 0
            for t in range(T):
                stream = (stream << b) | D[lane][t]        # MSB first
            stream <<= sym_len * S - T * b                  # padding bits
            mask = (1 << sym_len) - 1
            lane_syms.append([(stream >> (sym_len * (S - 1 - q))) & mask for q in range(S)])
        base_row[i] = base
        width[i] = b
        symptr[i + 1] = symptr[i] + S
        streams.append((S, lane_syms))
    words = np.zeros(32 * int(symptr[-1]), dtype=np.uint32)
    for i, (S, lane_syms) in enumerate(streams):
        wb = 32 * int(symptr[i])
        for lane in range(32):
            for q in range(S):
                words[wb + place(lane, q, S, V, 32)] = lane_syms[lane][q]
    col = arrange(np.asarray(cols, dtype=np.int32), T, 4, 0)
    v = arrange(vals, T, value_chunk(vals.dtype.itemsize), 0)
    return BroCoo(N, T, V, base_row, width, symptr, words, col, v)


def plain_rows(rows, T=32):
    """Row array of the plain COO baseline (same arrangement, last row repeated)."""
    rows = np.asarray(rows, dtype=np.int32)
    N = rows.size
    I = 32 * T
    nI = -(-N // I)
    out = arrange(rows, T, 4, 0)
    for i in range(nI):   # slots past the end repeat the last row
        for lane in range(32):
            for t in range(T):
                if entry(i, lane, t, T) >= N:
                    out[i * I + place(lane, t, T, 4, 32)] = rows[N - 1]
    return out


def decode_rows(C: BroCoo, sym_len=32):
    """Recover row_idx in COO order: each lane reads its T fields from its
    multiplexed stream ("decompression scheme is similar" to
    BRO-ELL's), then the rows are base_row plus the running sum of the
    deltas in entry order."""
    I = 32 * C.T
    out = np.zeros(C.nnz, dtype=np.int64)
    for i in range(C.n_intervals):
        b = int(C.width[i])
        S = int(C.symptr[i + 1] - C.symptr[i])
        wb = 32 * int(C.symptr[i])
        row = int(C.base_row[i])
        for lane in range(32):
            stream = 0
            for q in range(S):
                stream = (stream << sym_len) | int(C.words[wb + place(lane, q, S, C.V, 32)])
            total = S * sym_len
            for t in range(C.T):
                d = (stream >> (total - (t + 1) * b)) & ((1 << b) - 1) if b else 0
                row += d
                e = entry(i, lane, t, C.T)
                if e < C.nnz:
                    out[e] = row
    return out


def spmv_accumulate(C: BroCoo, x, y):
    """y[row] += val * x[col] for every COO entry (decoded rows)."""
    r = decode_rows(C)
    col = unarrange(C.col, C.nnz, C.T, 4)
    vals = unarrange(C.vals, C.nnz, C.T, value_chunk(C.vals.dtype.itemsize))
    for e in range(C.nnz):
        y[r[e]] += float(vals[e]) * float(x[int(col[e])])
    return y


def interval_shapes(rows, T=32, sym_len=32):
    """(base_row, width, S) of every interval, vectorised over the matrix —
    the same rules as encode() (a separate code path for full-size configs;
    pinned against encode() by tests/test_oracle_bro.py)."""
    rows = np.asarray(rows, dtype=np.int64)
    N = rows.size
    I = 32 * T
    nI = -(-N // I)
    if nI == 0:
        z = np.zeros(0, dtype=np.int64)
        return z, z, z
    pad = np.full(nI * I, rows[-1] if N else 0, dtype=np.int64)
    pad[:N] = rows
    R = pad.reshape(nI, I)                  # entry order inside each interval
    base = R[:, 0]
    d = np.diff(R, axis=1)                  # delta(e) = row(e) - row(e-1), e > 0
    dmax = d.max(axis=1) if I > 1 else np.zeros(nI, np.int64)
    from .bro_ell import gamma_np
    width = gamma_np(dmax)
    S = -(-(T * width) // sym_len)
    return base, width, S
