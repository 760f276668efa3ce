"""Pins of the value-indexing oracle (oracle/value_index.py, reading R28: the
"value data compression" of P:L416 by the value-index method of [16])
against things other than itself: the paper's matrix A worked by hand, the
27-point stencil's closed form, the code-width thresholds and a bitwise round
trip through the plain BRO-ELL value layout."""
import numpy as np
import pytest

from gen import random_csr, stencil_27pt
from oracle import bro_ell, value_index as vi


def test_paper_A_codes_by_hand(matrix_A):
    """A at h = 2: values 1..9 are D = [1..9] (positive doubles sort
    by bit pattern as by value), code = value - 1, one byte each; slice 0
    (l = 5): one 4-code chunk per row then the tail column, slice 1 (l = 3):
    tail only (P:L116 multiplexing with 4-byte chunks)."""
    A = matrix_A
    E = bro_ell.encode(A.row_ptr, A.col, A.vals, A.m, A.n, h=2, sym_len=32, V=1)
    V = vi.encode(A.row_ptr, A.vals, A.m, 2, E.num_col, E.colptr)
    assert V.cb == 1
    assert [float(v) for v in V.dict_vals] == [1, 2, 3, 4, 5, 6, 7, 8, 9]
    assert V.codes.tolist() == [2, 1, 0, 0, 1, 5, 4, 3, 0, 0,
                                0, 8, 6, 7, 2, 0]


def test_stencil_closed_form():
    """27-point stencil (26 on the diagonal, -1 off): D = [26.0, -1.0]
    (0x403A... < 0xBFF0... as unsigned), so the code of a slot is 0 exactly
    on the diagonal and 1 elsewhere."""
    A = stencil_27pt(5)
    E = bro_ell.encode(A.row_ptr, A.col, A.vals, A.m, A.n, h=32, sym_len=32, V=1)
    V = vi.encode(A.row_ptr, A.vals, A.m, 32, E.num_col, E.colptr)
    assert V.cb == 1 and [float(v) for v in V.dict_vals] == [26.0, -1.0]
    for t in range(E.s):
        l = int(E.num_col[t])
        base = 32 * int(E.colptr[t])
        for r in range(32):
            row = 32 * t + r
            if row >= A.m:
                continue
            cols = A.col[A.row_ptr[row]:A.row_ptr[row + 1]]
            for j, c in enumerate(cols):
                assert V.codes[base + bro_ell.place(r, j, l, 4, 32)] == (0 if c == row else 1)


@pytest.mark.parametrize("nd,cb", [(1, 1), (256, 1), (257, 2), (65536, 2), (65537, None)])
def test_code_width_thresholds(nd, cb):
    vals = np.arange(nd, dtype=np.float64) * 0.5 - 3.0
    got = vi.distinct(np.concatenate([vals, vals[::-1]]))
    if cb is None:
        assert got is None
    else:
        D, Dv, c = got
        assert c == cb and D.size == nd and np.all(np.diff(D.astype(object)) > 0)


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
@pytest.mark.parametrize("h", [2, 32, 64])
def test_round_trip_bitwise(dtype, h):
    """D[code] at every stored slot equals the stored value bit for bit, with
    -0.0 / 0.0 and two NaN payloads kept apart (lossless on bit patterns)."""
    A = random_csr(150, 90, 7, max_len=13, empty_frac=0.1)
    rng = np.random.default_rng(3)
    pool = np.array([0.0, -0.0, 1.5, -2.25, 3e-300 if dtype == np.float64 else 3e-30, 7.0], dtype=dtype)
    nan1 = np.array([0x7FF8000000000001 if dtype == np.float64 else 0x7FC00001],
                    dtype=np.uint64 if dtype == np.float64 else np.uint32).view(dtype)
    nan2 = np.array([0x7FF8000000000002 if dtype == np.float64 else 0x7FC00002],
                    dtype=np.uint64 if dtype == np.float64 else np.uint32).view(dtype)
    pool = np.concatenate([pool, nan1, nan2])
    vals = pool[rng.integers(0, pool.size, A.nnz)]
    E = bro_ell.encode(A.row_ptr, A.col, vals, A.m, A.n, h=h, sym_len=32, V=1)
    V = vi.encode(A.row_ptr, vals, A.m, h, E.num_col, E.colptr)
    assert V.cb == 1 and V.dict_bits.size == np.unique(vi._bits(vals)).size
    back = vi.slot_values(V, h, E.num_col, E.colptr, E.Vv)
    cols = bro_ell.decoded_slots(E)  # V=1 slot order; map to the Vv value layout
    for t in range(E.s):
        l = int(E.num_col[t])
        base = h * int(E.colptr[t])
        for r in range(h):
            for j in range(l):
                if cols[base + h * j + r] < 0:
                    continue  # padding
                p = base + bro_ell.place(r, j, l, E.Vv, h)
                assert vi._bits(back[p:p + 1])[0] == vi._bits(E.vals[p:p + 1])[0]


def test_cap_takes_the_ell_part_only():
    """With cap = K only the first K values of each row enter D (HYB's ELL part)."""
    rp = np.array([0, 3, 4])
    col = np.array([0, 1, 2, 0], dtype=np.int32)
    vals = np.array([5.0, 6.0, 99.0, 7.0])
    E = bro_ell.encode(rp, col, vals, 2, 3, h=2, sym_len=32, V=1)
    V = vi.encode(rp, vals, 2, 2, np.array([2]), np.array([0, 2], dtype=np.uint64), cap=2)
    assert [float(v) for v in V.dict_vals] == [5.0, 6.0, 7.0]
    assert V.codes.tolist() == [0, 1, 2, 0]
    del E


def test_padding_code_is_first_finite_value():
    """Padding slots hold pz, the code of the first finite value of D (a
    padding product is then a finite value times 0): D = [+inf, -1.0]
    (0x7FF0... < 0xBFF0... as unsigned) gives pz = 1; a part whose values are
    all non-finite is not indexed."""
    rp = np.array([0, 1, 3])
    col = np.array([0, 0, 1], dtype=np.int32)
    vals = np.array([np.inf, -1.0, np.inf])
    E = bro_ell.encode(rp, col, vals, 2, 2, h=2, sym_len=32, V=1)
    V = vi.encode(rp, vals, 2, 2, E.num_col, E.colptr)
    assert [float(v) for v in V.dict_vals] == [np.inf, -1.0] and V.pz == 1
    # slice l = 2, tail layout: row 0 [inf, pad], row 1 [-1, inf]
    assert V.codes.tolist() == [0, 1, 1, 0]
    assert vi.encode(rp, np.array([np.inf, np.nan, -np.inf]), 2, 2, E.num_col, E.colptr) is None
