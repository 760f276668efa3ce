"""ELLPACK, ELLPACK-R and the HYB split (§2.1.2-2.1.4).

Test infrastructure only (see oracle/__init__.py).
"""
from __future__ import annotations

import numpy as np

PAD = -1  # the paper's '*' (invalid slot)


def row_length(row_ptr):
    """ELLPACK-R row_length array: number of non-zeros per row."""
    return np.diff(np.asarray(row_ptr, dtype=np.int64))


def ell_arrays(row_ptr, col, vals, k=None):
    """ELLPACK: entries shifted left into m x k arrays, '*' = PAD
    (value 0) for slots past the row's length.  k defaults to the maximum row
    length ("k is the maximum number of non-zeros in a row")."""
    lens = row_length(row_ptr)
    m = lens.size
    if k is None:
        k = int(lens.max()) if m else 0
    C = np.full((m, k), PAD, dtype=np.int64)
    V = np.zeros((m, k), dtype=np.asarray(vals).dtype)
    for i in range(m):
        a = int(row_ptr[i])
        t = min(int(lens[i]), k)
        C[i, :t] = col[a:a + t]
        V[i, :t] = vals[a:a + t]
    return C, V


def hyb_K(row_ptr):
    """Dividing column K of the HYB split (same rule as [4,5] per P:L144).

    Reading R12: K is the smallest k >= 0 such that the number of
    rows with MORE than k non-zeros is less than a third of the rows,
        K = min{ k >= 0 : 3 * |{i : len_i > k}| < m }.
    The worked split of matrix A at P:L79 (ELL width 3) pins this reading:
    the literal "at least k" variant gives 4 and a Cusp-style row breakeven
    gives 0 (tests/test_oracle_pins.py).
    """
    lens = row_length(row_ptr)
    m = lens.size
    if m == 0:
        return 0
    k = 0
    while True:
        if 3 * int(np.count_nonzero(lens > k)) < m:
            return k
        k += 1


def hyb_split(row_ptr, col, vals, K):
    """Split CSR into the ELL part (first min(len_i, K) entries of each row)
    and the COO part (the rest, in (row, col) order) — P:L77-79.

    Returns (ell_row_ptr, ell_col, ell_vals, coo_row, coo_col, coo_vals)."""
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    lens = np.diff(row_ptr)
    m = lens.size
    ell_lens = np.minimum(lens, K)
    ell_ptr = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(ell_lens, out=ell_ptr[1:])
    rows = np.repeat(np.arange(m, dtype=np.int64), lens)
    pos = np.arange(int(row_ptr[-1]), dtype=np.int64) - np.repeat(row_ptr[:-1], lens)
    in_ell = pos < K
    col = np.asarray(col)
    vals = np.asarray(vals)
    return (ell_ptr, col[in_ell], vals[in_ell],
            rows[~in_ell], col[~in_ell], vals[~in_ell])
