"""BRO-COO encoder/decoder (§3.2).

Test infrastructure only (see oracle/__init__.py).

PARITY UNPINNED (layout): Fig. 2, which shows the interval arrangement, is an
image absent from PAPER.md.  The text fixes only that
  * only row_idx is compressed; col_idx and vals stay as in COO;
  * row data is divided into intervals, each processed by one warp;
  * each interval is a 2D array whose row index increases monotonically in
    the vertical direction, delta-encoded, then bit-packed with ONE width per
    interval (stored in bit_alloc), then multiplexed as in BRO-ELL.
Reading R13/R14 fills the rest: intervals of I = 32*T entries
(T = 32 steps); element (t, lane) of interval i is COO entry i*I + 32*t + lane
(the warp-per-interval order of [5]), so each lane's column of the 2D
array is non-decreasing; lane deltas are taken down that column, the first
relative to the interval's base row (row of its first entry); positions past
the last entry repeat the last row (delta 0).  These choices are pinned only
by round trips and by SpMV through the decoder, not by the paper.
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
    col: np.ndarray         # int32[nnz] (unchanged COO order)
    vals: np.ndarray        # [nnz]

    @property
    def n_intervals(self) -> int:
        return int(self.base_row.size)

    def stream_bytes(self) -> int:
        return int(32 * int(self.symptr[-1]) * 4)


def interval_rows(rows, i, T):
    """The 2D row array of interval i: R[t][lane] (positions past the end
    repeat the last row)."""
    I = 32 * T
    N = len(rows)
    R = []
    for t in range(T):
        R.append([int(rows[min(i * I + 32 * t + lane, N - 1)]) for lane in range(32)])
    return R


def encode(rows, cols, vals, T=32, V=4, sym_len=32) -> BroCoo:
    """Encode COO entries already sorted by (row, col)."""
    rows = np.asarray(rows, dtype=np.int64)
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
        # delta encoding down each lane's column of the 2D array
        D = [[R[t][lane] - (R[t - 1][lane] if t > 0 else base) for lane in range(32)]
             for t in range(T)]
        b = max(gamma(D[t][lane]) for t in range(T) for lane in range(32))
        S = -(-(T * b) // sym_len)
        lane_syms = []
        for lane in range(32):
            stream = 0
            for t in range(T):
                stream = (stream << b) | D[t][lane]        # MSB first
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
    return BroCoo(N, T, V, base_row, width, symptr, words,
                  np.asarray(cols, dtype=np.int32), np.asarray(vals))


def decode_rows(C: BroCoo, sym_len=32):
    """Recover row_idx: each lane reads its stream with the BRO-ELL
    load-and-decode cycle ("decompression scheme is similar"),
    one uniform width per interval."""
    I = 32 * C.T
    out = np.zeros(C.nnz, dtype=np.int64)
    for i in range(C.n_intervals):
        b = int(C.width[i])
        S = int(C.symptr[i + 1] - C.symptr[i])
        wb = 32 * int(C.symptr[i])
        for lane in range(32):
            stream = 0
            for q in range(S):
                stream = (stream << sym_len) | int(C.words[wb + place(lane, q, S, C.V, 32)])
            total = S * sym_len
            row = int(C.base_row[i])
            for t in range(C.T):
                d = (stream >> (total - (t + 1) * b)) & ((1 << b) - 1) if b else 0
                row += d
                e = i * I + 32 * t + lane
                if e < C.nnz:
                    out[e] = row
    return out


def spmv_accumulate(C: BroCoo, x, y):
    """y[row] += val * x[col] for every COO entry (decoded rows)."""
    r = decode_rows(C)
    for e in range(C.nnz):
        y[r[e]] += float(C.vals[e]) * float(x[int(C.col[e])])
    return y
