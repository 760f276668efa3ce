"""Pins of the oracle's BRO-ELL / BRO-COO encoders and decoders (-m "not gpu").

What fixes each expectation:
  * matrix A with h = 2, sym_len = 4 compresses to 32 bits; the
    alternatives (no padding, global or per-row widths, 0-based delta with
    c_{-1}=0, sym_len 32) give other totals or break the invalid marker;
  * round trips through a line-by-line transcription of Algorithm 1
    (P:L128-138), which fixes the bit order (MSB first: `sym << b`), the
    zero-means-invalid rule and the multiplexing index;
  * SpMV through the decoder equals the plain CSR SpMV;
  * closed form: C1 (5-point Laplacian, 64x64) needs 27 bits per interior row
    (deltas ~ {2^12, 63, 1, 1, 63}) -> one 32-bit symbol per row, eta = 0.8.
"""
import numpy as np
import pytest
from hypothesis import given, settings, strategies as st, HealthCheck

from gen import Csr, laplacian_2d, random_csr
from oracle import bro_coo, bro_ell, metrics, spmv


def _cols(A):
    return [A.col[A.row_ptr[i]:A.row_ptr[i + 1]].tolist() for i in range(A.m)]


# ---------------------------------------------------------------- BRO-ELL

def test_paper_A_compressed_size(matrix_A, golden_A):
    g = golden_A["bro_ell"]
    E = bro_ell.encode(matrix_A.row_ptr, matrix_A.col, matrix_A.vals, 4, 5,
                       h=g["h"], sym_len=g["sym_len"], V=1)
    assert E.stream_bytes() * 8 == g["stream_bits"]          # 32 bits
    assert E.num_col.tolist() == [5, 3]
    # decode with the literal Algorithm 1
    assert bro_ell.decode(E) == _cols(matrix_A)
    assert metrics.eta(E.stream_bytes(), g["col_idx_bytes"]) == pytest.approx(0.95)


def test_paper_A_derived_layout(matrix_A):
    """Bit pattern implied by the rules (derived, Fig. 1 is an image):
    slice 0 widths [1,2,1,1,1] b_p=2, slice 1 widths [3,1,2] b_p=2;
    V=1 words [1100,1011,0000,1100 | 0101,1001,1000,0000]."""
    E = bro_ell.encode(matrix_A.row_ptr, matrix_A.col, matrix_A.vals, 4, 5, h=2, sym_len=4, V=1)
    assert E.bit_alloc.tolist() == [1, 2, 1, 1, 1, 3, 1, 2]
    assert [E.slices[0].b_p, E.slices[1].b_p] == [2, 2]
    assert E.words.tolist() == [0b1100, 0b1011, 0b0000, 0b1100, 0b0101, 0b1001, 0b1000, 0b0000]


def test_paper_A_alternative_readings_rejected(matrix_A):
    """The 32-bit total of P:L116 rules out the readings DESIGN.md rejects."""
    rows = _cols(matrix_A)
    d = [bro_ell.row_deltas(c) for c in rows]
    g = bro_ell.gamma
    # no padding: sum of per-slice widths = 6 + 6 = 12 bits per row pair
    no_pad = sum(2 * sum(max(g(d[r][j]) if j < len(d[r]) else 0 for r in s)
                         for j in range(max(len(d[r]) for r in s))) for s in ([0, 1], [2, 3]))
    assert no_pad == 24
    # one global width per column (no slices)
    glob = 4 * sum(max(g(dd[j]) if j < len(dd) else 0 for dd in d) for j in range(5))
    assert glob > 32
    # 0-based column with c_{-1} = 0 makes a row starting at column 0 look invalid
    zero_based_first = [c[0] - 0 for c in rows]
    assert 0 in zero_based_first


def test_alg1_strict_and_nonstrict_agree(matrix_A):
    E = bro_ell.encode(matrix_A.row_ptr, matrix_A.col, matrix_A.vals, 4, 5, h=2, sym_len=4, V=1)
    assert bro_ell.decode(E, strict=True) == bro_ell.decode(E, strict=False)
    x = np.arange(1, 6, dtype=np.float64)
    assert bro_ell.spmv(E, x).tolist() == [9.0, 50.0, 64.0, 47.0]


def test_c1_closed_form():
    A = laplacian_2d(64)
    E = bro_ell.encode(A.row_ptr, A.col, A.vals, A.m, A.n, h=32, sym_len=32, V=4)
    assert E.s == 128 and set(E.S.tolist()) == {1}
    assert E.stream_bytes() == 128 * 32 * 4
    assert metrics.eta(E.stream_bytes(), metrics.ell_index_bytes(A.m, 5)) == pytest.approx(0.8)
    assert bro_ell.decode(E) == _cols(A)


@st.composite
def csr_strategy(draw):
    m = draw(st.integers(0, 70))
    wide = draw(st.booleans())
    n = draw(st.sampled_from([1, 7, 100, 5000, 2**31 - 1])) if wide else draw(st.integers(1, 300))
    rows, cols = [], []
    for i in range(m):
        k = draw(st.integers(0, min(n, 12)))
        if k == 0:
            continue
        if n > 10**6:
            c = sorted(set(draw(st.lists(st.sampled_from(
                [0, 1, 2, 3, n - 3, n - 2, n - 1, n // 2, n // 3, 2**20, 2**20 + 1]),
                min_size=1, max_size=k))))
        else:
            c = sorted(set(draw(st.lists(st.integers(0, n - 1), min_size=1, max_size=k))))
        rows += [i] * len(c)
        cols += c
    rp = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(np.bincount(np.array(rows, dtype=np.int64), minlength=m), out=rp[1:])
    vals = np.array([draw(st.sampled_from([1.0, -2.5, 0.0, 3.25])) for _ in cols], dtype=np.float64)
    return Csr(m, n, rp, np.array(cols, dtype=np.int64), vals, "hyp")


@settings(max_examples=60, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(A=csr_strategy(), h=st.sampled_from([2, 4, 32]), sym=st.sampled_from([4, 8, 32, 64]),
       V=st.sampled_from([1, 2, 4]))
def test_bro_ell_roundtrip_fuzz(A, h, sym, V):
    if sym < 32 and A.n > 2**(sym - 1):
        sym = 32  # a field wider than sym_len cannot be multiplexed (b_j <= sym_len)
    E = bro_ell.encode(A.row_ptr, A.col, A.vals, A.m, A.n, h=h, sym_len=sym, V=V)
    assert bro_ell.decode(E, strict=True) == _cols(A)
    assert bro_ell.decode(E, strict=False) == _cols(A)
    # vectorised shape computation agrees with the step-by-step encoder
    l, S, w = bro_ell.slice_shapes(A.row_ptr, A.col, A.m, h, sym)
    assert l.tolist() == E.num_col.tolist() and S.tolist() == E.S.tolist()
    assert w.tolist() == E.bit_alloc.tolist()


@pytest.mark.parametrize("seed", range(3))
def test_bro_ell_spmv_equals_csr(seed):
    A = random_csr(200, 3000, seed, max_len=40, empty_frac=0.2, wide_cols=bool(seed % 2))
    x = np.random.default_rng(seed).uniform(-1, 1, A.n)
    E = bro_ell.encode(A.row_ptr, A.col, A.vals, A.m, A.n, h=32, sym_len=32, V=4)
    y = bro_ell.spmv(E, x)
    yr, S = spmv.csr_spmv(A.row_ptr, A.col, A.vals, x)
    assert np.all(np.abs(y - np.array(yr, np.float64)) <= 1e-13 * np.array(S, np.float64) + 1e-300)


def test_place_v1_is_paper_multiplexing():
    """V = 1: symbol q of row r sits at q*h + r (Alg. 1 line 12)."""
    for h in (2, 32):
        for S in (1, 3, 5):
            for r in range(h):
                for q in range(S):
                    assert bro_ell.place(r, q, S, 1, h) == q * h + r


def test_place_is_a_bijection():
    for h in (2, 32):
        for V in (2, 4):
            for S in range(0, 11):
                pos = sorted(bro_ell.place(r, q, S, V, h) for r in range(h) for q in range(S))
                assert pos == list(range(h * S))


def test_sampled_slices_match_full_encode():
    A = random_csr(300, 1000, 5, max_len=50, empty_frac=0.1)
    full = bro_ell.encode(A.row_ptr, A.col, A.vals, A.m, A.n)
    part = bro_ell.encode(A.row_ptr, A.col, A.vals, A.m, A.n, slices=[0, 3, 9])
    for t in (0, 3, 9):
        a, b = 32 * int(full.symptr[t]), 32 * int(full.symptr[t + 1])
        assert np.array_equal(full.words[a:b], part.words[a:b])
        a, b = 32 * int(full.colptr[t]), 32 * int(full.colptr[t + 1])
        assert np.array_equal(full.vals[a:b], part.vals[a:b])


# ---------------------------------------------------------------- BRO-COO

def _coo(A):
    rows, cols, vals = spmv.csr_to_coo(A.row_ptr, A.col, A.vals)
    return rows, cols, vals


@st.composite
def coo_rows_strategy(draw):
    n = draw(st.integers(0, 3000))
    steps = draw(st.lists(st.sampled_from([0, 0, 0, 1, 1, 2, 5, 100, 2**20, 2**30]),
                          min_size=n, max_size=n))
    return np.cumsum(np.array(steps, dtype=np.int64)) if n else np.zeros(0, np.int64)


@settings(max_examples=40, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(rows=coo_rows_strategy(), T=st.sampled_from([1, 8, 16, 32]), V=st.sampled_from([1, 4]))
def test_bro_coo_roundtrip_fuzz(rows, T, V):
    rows = rows[rows < 2**31 - 1]
    cols = np.arange(rows.size, dtype=np.int32)
    vals = np.arange(rows.size, dtype=np.float64) + 0.5
    C = bro_coo.encode(rows, cols, vals, T=T, V=V)
    assert np.array_equal(bro_coo.decode_rows(C), rows)
    assert np.array_equal(bro_coo.unarrange(C.col, rows.size, T, 4), cols)
    assert np.array_equal(bro_coo.unarrange(C.vals, rows.size, T, 2), vals)
    I = 32 * T
    for i in range(C.n_intervals):
        # one width per interval = Gamma of the largest consecutive
        # difference of the sorted rows inside the interval (brute force)
        seg = rows[i * I:(i + 1) * I]
        dmax = int(np.max(np.diff(seg))) if seg.size > 1 else 0
        assert int(C.width[i]) == dmax.bit_length() <= 32
        assert int(C.base_row[i]) == int(seg[0])


def test_bro_coo_hand_example_T1():
    """One interval of 32 entries, T = 1 (lane l holds entry l): rows
    0 x10, 1 x10, 5 x12.  Deltas in entry order: 1 at entry 10, 4 at entry
    20, else 0 -> one width b = Gamma(4) = 3; each lane stream is
    3 bits MSB first padded to a 32-bit symbol: lane 10 = 001 -> 0x20000000,
    lane 20 = 100 -> 0x80000000, every other lane 0 (worked by hand)."""
    rows = np.array([0] * 10 + [1] * 10 + [5] * 12)
    C = bro_coo.encode(rows, np.zeros(32, np.int32), np.zeros(32), T=1, V=1)
    assert C.width.tolist() == [3] and C.base_row.tolist() == [0]
    assert C.symptr.tolist() == [0, 1]
    want = [0] * 32
    want[10], want[20] = 0x20000000, 0x80000000
    assert C.words.tolist() == want
    assert np.array_equal(bro_coo.decode_rows(C), rows)


def test_bro_coo_hand_example_T2_lane_contiguous():
    """T = 2, 64 entries, row(e) = e // 3 (worked by hand): lane l holds
    entries 2l and 2l+1 (consecutive), deltas are 1 where e % 3 == 0
    (e > 0), width 1; lane stream = [delta(2l), delta(2l+1)] MSB first:
    lane 0 (e 0,1) 00 -> 0; lane 1 (e 2,3) 01 -> 0x40000000; lane 3
    (e 6,7) 10 -> 0x80000000; lane 4 (e 8,9) 01 -> 0x40000000; lane 2
    (e 4,5) 00 -> 0.  col/vals are stored lane-contiguously: with 4-entry
    chunks, lane l's 2 entries sit at 2l, 2l+1 (place() tail of a 2-slot
    lane stream), so col equals COO order here."""
    rows = np.arange(64) // 3
    cols = np.arange(64, dtype=np.int32) * 7
    C = bro_coo.encode(rows, cols, np.ones(64), T=2, V=1)
    assert C.width.tolist() == [1]
    assert C.words[:5].tolist() == [0, 0x40000000, 0, 0x80000000, 0x40000000]
    assert np.array_equal(C.col, cols)
    assert np.array_equal(bro_coo.decode_rows(C), rows)


def test_bro_coo_values_chunked_like_bro_ell():
    """T = 8, fp64: lane l's 8 values are 4 chunks of 2 (16 bytes); chunk c
    of all 32 lanes is one contiguous 512-byte row: entry (l, t) at
    64*(t//2) + 2*l + t%2 (BRO-ELL's value multiplexing)."""
    N = 256
    vals = np.arange(N, dtype=np.float64)
    C = bro_coo.encode(np.zeros(N, np.int64), np.zeros(N, np.int32), vals, T=8, V=4)
    for lane in (0, 1, 31):
        for t in range(8):
            assert C.vals[64 * (t // 2) + 2 * lane + t % 2] == 8 * lane + t


def test_bro_coo_single_row_interval_has_zero_width():
    rows = np.full(2048, 7, dtype=np.int64)
    C = bro_coo.encode(rows, np.arange(2048), np.ones(2048))
    assert C.width.tolist() == [0, 0] and C.base_row.tolist() == [7, 7]
    assert C.words.size == 0
    assert np.array_equal(bro_coo.decode_rows(C), rows)


def test_bro_coo_tail_interval_padding():
    """A ragged last interval: slots past the end hold col 0 / value 0, the
    plain baseline repeats the last row there."""
    rows = np.sort(np.random.default_rng(5).integers(0, 90, 300))
    C = bro_coo.encode(rows, np.arange(300, dtype=np.int32), np.ones(300), T=8)
    assert C.col.size == 2 * 256 and C.vals.size == 512
    assert np.count_nonzero(C.vals) == 300
    pr = bro_coo.plain_rows(rows, T=8)
    assert np.array_equal(bro_coo.unarrange(pr, 300, 8, 4), rows)
    assert np.count_nonzero(pr == rows[-1]) >= 512 - 300


@pytest.mark.parametrize("T", [8, 32])
def test_bro_coo_spmv_equals_csr(T):
    A = random_csr(400, 900, 3, max_len=30, empty_frac=0.3, long_frac=0.02, long_len=700)
    rows, cols, vals = _coo(A)
    x = np.random.default_rng(0).uniform(-1, 1, A.n)
    C = bro_coo.encode(rows, cols, vals, T=T)
    y = bro_coo.spmv_accumulate(C, x, np.zeros(A.m))
    yr, S = spmv.csr_spmv(A.row_ptr, A.col, A.vals, x)
    assert np.all(np.abs(y - np.array(yr, np.float64)) <= 1e-13 * np.array(S, np.float64) + 1e-300)


@pytest.mark.parametrize("T", [1, 8, 32])
@pytest.mark.parametrize("seed", range(3))
def test_bro_coo_interval_shapes_match_encoder(T, seed):
    rows = np.sort(np.random.default_rng(seed).integers(0, 5000 * (seed + 1), 3000 + 77 * seed))
    C = bro_coo.encode(rows, np.zeros(rows.size, np.int32), np.zeros(rows.size), T=T)
    base, width, S = bro_coo.interval_shapes(rows, T)
    assert base.tolist() == C.base_row.tolist()
    assert width.tolist() == C.width.tolist()
    assert S.tolist() == np.diff(C.symptr.astype(np.int64)).tolist()
