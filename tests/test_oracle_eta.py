"""Pins of the oracle's space-savings arithmetic and layout shapes beyond the
ELL case (-m "not gpu"):

  * HYB eta (P:L246 with reading R19) on the paper's own HYB split of
    matrix A, worked by hand;
  * the C5 regression values of SURVEY.md section 8(c) (eta_stream and the
    symbols-per-row histogram, derived there by an independent script);
  * the method-0 row order (signature clustering) against a brute-force
    key sort built here from numpy features, not from oracle/bar.py.
"""
import json
import os

import numpy as np
import pytest

from gen import make_config, random_block, row_block
from oracle import bar, bro_coo, bro_ell, hyb, metrics

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_hyb_eta_paper_A_by_hand(matrix_A):
    """Matrix A split at K = 3.  O = ELL col_idx 4x3 + COO row_idx
    and col_idx of 2 entries = 12 + 4 int32 = 64 bytes ("2nnz").
    BRO-ELL of the ELL part with h = 2, sym_len = 4 (the setting of P:L116),
    by hand: rows (1-based) [1,3] [1,2,3] -> deltas [1,2] [1,1,1], widths
    [1,2,1] = 4 bits = 1 symbol per row; rows [2,3,5] [4,5] -> deltas [2,1,2]
    [4,1], widths [3,1,2] = 6 bits = 2 symbols per row: 2*4 + 2*8 = 24 bits
    = 3 bytes.  BRO-COO of the 2 COO entries (both in row 2): one interval,
    deltas 0, width 0, empty stream.  C = 3 + 0 + 4*2 (raw col) = 11 bytes:
    eta = 1 - 11/64 = 0.828125."""
    K = hyb.hyb_K(matrix_A.row_ptr)
    ep, ec, ev, cr, cc, cv = hyb.hyb_split(matrix_A.row_ptr, matrix_A.col, matrix_A.vals, K)
    O = metrics.hyb_index_bytes(4, K, cr.size)
    assert O == 64
    E = bro_ell.encode(ep, ec, ev, 4, 5, h=2, sym_len=4, V=1)
    assert E.stream_bytes() == 3
    C = bro_coo.encode(cr, cc, cv, T=1, V=1)
    assert C.width.tolist() == [0] and C.stream_bytes() == 0
    Cb = metrics.bro_hyb_stream_bytes(E.stream_bytes(), C.stream_bytes(), cr.size)
    assert Cb == 11
    assert metrics.eta(Cb, O) == pytest.approx(0.828125, abs=0)


def _c5_shapes():
    """slice_shapes over h-aligned row blocks of C5 (deltas depend only on a
    row's own columns, so blocking does not change the result)."""
    A = make_config(5)
    S_all = []
    step = 32 * 31250  # 1M rows
    for r0 in range(0, A.m, step):
        B = row_block(A, r0, min(A.m, r0 + step))
        _, S, _ = bro_ell.slice_shapes(B.row_ptr, B.col, B.m, 32, 32)
        S_all.append(S)
    return A, np.concatenate(S_all)


@pytest.mark.slow
def test_c5_layout_regression_values():
    with open(os.path.join(ROOT, "tests", "golden", "survey_c5_layout.json")) as f:
        g = json.load(f)
    A, S = _c5_shapes()
    assert A.nnz == g["nnz"] and S.size == g["n_slices"]
    hist = {str(k): int(v) for k, v in zip(*np.unique(S, return_counts=True))}
    assert hist == g["symbols_per_row_histogram"]
    stream = 32 * 4 * int(S.sum())
    K = int(A.row_lengths().max())
    eta = metrics.eta(stream, metrics.ell_index_bytes(A.m, K))
    assert round(eta, g["eta_stream_digits"]) == g["eta_stream"]
    assert round(stream / 1e6, 1) == g["stream_mb"]


def _numpy_signature_keys(A):
    """Method-0 key from numpy features: (length, jump flags as a tuple,
    first column, row id); jump flag j >= 1 = the j-th delta needs more than
    2 bits (delta = column difference >= 4)."""
    lens = np.diff(A.row_ptr)
    keys = []
    for i in range(A.m):
        c = np.asarray(A.col[A.row_ptr[i]:A.row_ptr[i + 1]], dtype=np.int64)
        jumps = tuple((np.diff(c) >= 4).astype(int).tolist())
        keys.append((int(lens[i]), jumps, int(c[0]) if c.size else -1, i))
    return keys


@pytest.mark.parametrize("seed", [0, 5])
def test_signature_order_bruteforce_keys(seed):
    A = row_block(random_block(seed=seed, families=6, fam_rows=32), 0, 181)
    keys = _numpy_signature_keys(A)
    want = [k[3] for k in sorted(keys)]
    got = bar.signature_order(A.row_ptr, A.col, A.m).tolist()
    assert got == want
    # properties of the order: lengths non-decreasing; equal (length, jumps)
    # rows are contiguous and ordered by first column
    kk = [keys[i] for i in got]
    assert all(a[0] <= b[0] for a, b in zip(kk, kk[1:]))
    seen = {}
    for p, k in enumerate(kk):
        g = (k[0], k[1])
        if g in seen:
            assert seen[g] == p - 1, "signature group not contiguous"
        seen[g] = p
