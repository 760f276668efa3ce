"""Plain SpMV y = A.x — the result every BRO format must reproduce.

Test infrastructure only (see oracle/__init__.py).

The BRO schemes are lossless index compression ("compress the index
data"), so the exact result they reach is the plain definition
    y_i = sum_{(i,j) stored} a_ij * x_j
computed here in higher precision than the data: np.longdouble (x86 80-bit)
for fp64 data, fp64 for fp32 data (reading R18).  It also returns
S_i = sum_j |a_ij| |x_j|, the scale of the north-star tolerance
|y_gpu - y_ref| <= tol * S_i.
"""
from __future__ import annotations

import numpy as np


def acc_dtype(vals_dtype) -> np.dtype:
    """Accumulation precision of the oracle for a given value type."""
    return np.dtype(np.longdouble) if np.dtype(vals_dtype) == np.float64 else np.dtype(np.float64)


def csr_spmv(row_ptr, col, vals, x):
    """Return (y, S) in acc_dtype(vals.dtype); rows with no entries give 0."""
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    m = row_ptr.size - 1
    acc = acc_dtype(np.asarray(vals).dtype)
    a = np.asarray(vals).astype(acc)
    xv = np.asarray(x).astype(acc)[np.asarray(col, dtype=np.int64)]
    prod = a * xv
    absprod = np.abs(a) * np.abs(xv)
    y = np.zeros(m, dtype=acc)
    S = np.zeros(m, dtype=acc)
    nonempty = row_ptr[1:] > row_ptr[:-1]
    if prod.size:
        starts = row_ptr[:-1][nonempty]
        # consecutive non-empty rows own contiguous ranges, so reduceat over
        # their starts sums exactly each row's entries
        y[nonempty] = np.add.reduceat(prod, starts)
        S[nonempty] = np.add.reduceat(absprod, starts)
    return y, S


def csr_spmv_rows(row_ptr, col, vals, x, rows):
    """(y, S) for the selected rows only (sampled parity at full size)."""
    rows = np.asarray(rows, dtype=np.int64)
    acc = acc_dtype(np.asarray(vals).dtype)
    y = np.zeros(rows.size, dtype=acc)
    S = np.zeros(rows.size, dtype=acc)
    for k, r in enumerate(rows):
        a, b = int(row_ptr[r]), int(row_ptr[r + 1])
        av = np.asarray(vals[a:b]).astype(acc)
        xv = np.asarray(x).astype(acc)[np.asarray(col[a:b], dtype=np.int64)]
        y[k] = np.sum(av * xv)
        S[k] = np.sum(np.abs(av) * np.abs(xv))
    return y, S


def dense_from_csr(m, n, row_ptr, col, vals):
    """Dense m x n array (tiny matrices only)."""
    D = [[0.0] * n for _ in range(m)]
    for i in range(m):
        for p in range(int(row_ptr[i]), int(row_ptr[i + 1])):
            D[i][int(col[p])] += float(vals[p])
    return D


def dense_spmv(D, x):
    """Brute-force dense matvec with Python floats/loops (tiny inputs)."""
    return [sum(float(D[i][j]) * float(x[j]) for j in range(len(x))) for i in range(len(D))]


def coo_to_csr(m, row_idx, col_idx, vals):
    """COO (sorted or not) to CSR, stable in (row, col) order."""
    row_idx = np.asarray(row_idx, dtype=np.int64)
    col_idx = np.asarray(col_idx, dtype=np.int64)
    order = np.lexsort((col_idx, row_idx))
    counts = np.bincount(row_idx, minlength=m)
    row_ptr = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    return row_ptr, col_idx[order].astype(np.int32), np.asarray(vals)[order]


def csr_to_coo(row_ptr, col, vals):
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    rows = np.repeat(np.arange(row_ptr.size - 1, dtype=np.int64), np.diff(row_ptr))
    return rows, np.asarray(col), np.asarray(vals)


def within_tolerance(y_gpu, y_ref, S, tol):
    """Per-row check |y_gpu - y_ref| <= tol * S (north_star bound)."""
    y_gpu = np.asarray(y_gpu).astype(y_ref.dtype)
    err = np.abs(y_gpu - y_ref)
    return err <= tol * S, err
