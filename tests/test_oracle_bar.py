"""Pins of the oracle's BAR reordering (oracle/bar.py, Sec. 3.4,
P:L151-212) — -m "not gpu".

What fixes each expectation:
  * Eqn (2)'s term: on matrix A with h = 2 and alpha = sym_len = 4,
    sum over the natural partitions of ceil(sum_j d(S, j) / alpha) symbols per
    row x h rows x alpha bits = the 32-bit stream of P:L116; at h = 32 the
    same sum equals the BRO-ELL encoder's symbol count (symptr[s]);
  * Eqn (3)'s term (reading R20): distinct 128-byte x lines per (partition,
    column) counted independently with numpy.unique;
  * Algorithm 2 on a hand example whose answer is forced (rows touching the
    same x lines with the same delta widths end up together);
  * the windowed variant (reading R24): W = 1 is the stable length sort of
    line 2 (closed form when h | m), W >= v is the paper's algorithm.
"""
import math

import numpy as np
import pytest

from gen import Csr, random_block, random_csr
from oracle import bar, bro_ell


def _rows(A, ids):
    return [A.col[A.row_ptr[i]:A.row_ptr[i + 1]].tolist() for i in ids]


def test_d_term_reproduces_paper_32_bits(matrix_A):
    """A at h = 2, sym_len = 4 compresses to 32 bits."""
    h, alpha = 2, 4
    total_sym = 0
    for S in ([0, 1], [2, 3]):
        rc = _rows(matrix_A, S)
        k = max(len(c) for c in rc)
        total_sym += math.ceil(sum(bar.d_term(rc, j) for j in range(k)) / alpha)
    assert total_sym * h * alpha == 32


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_d_term_equals_encoder_symbols(seed):
    """At h = alpha = 32 the Eqn (2) term of the natural slices is the
    BRO-ELL symbol count per row stream, summed over slices."""
    A = random_csr(200, 5000, seed, max_len=40, empty_frac=0.1, wide_cols=seed == 2)
    E = bro_ell.encode(A.row_ptr, A.col, A.vals, A.m, A.n)
    total = 0
    for t in range(-(-A.m // 32)):
        rc = _rows(A, range(32 * t, min(A.m, 32 * t + 32)))
        k = max((len(c) for c in rc), default=0)
        total += math.ceil(sum(bar.d_term(rc, j) for j in range(k)) / 32)
    assert total == int(E.symptr[-1])


@pytest.mark.parametrize("vsize", [8, 4])
def test_c_term_counts_distinct_lines(vsize):
    A = random_csr(150, 3000, 5, max_len=30, empty_frac=0.1)
    parts = [list(range(32 * t, min(A.m, 32 * t + 32))) for t in range(-(-A.m // 32))]
    ours = 0
    for S in parts:
        rc = _rows(A, S)
        k = max((len(c) for c in rc), default=0)
        ours += sum(bar.c_term(rc, j, vsize) for j in range(k))
    rows = np.repeat(np.arange(A.m), np.diff(A.row_ptr))
    j = np.arange(A.nnz) - A.row_ptr[rows]
    keys = np.stack([rows // 32, j, A.col.astype(np.int64) * vsize // 128], axis=1)
    assert ours == np.unique(keys, axis=0).shape[0]
    # and Phi is the sum of both terms (h = w: factor 1)
    dsym = 0
    for S in parts:
        rc = _rows(A, S)
        k = max((len(c) for c in rc), default=0)
        dsym += math.ceil(sum(bar.d_term(rc, j) for j in range(k)) / 32)
    assert bar.phi(parts, A.row_ptr, A.col, vsize=vsize) == dsym + ours


def test_algorithm2_hand_example():
    """4 rows of length 2, h = 2: seeds are rows 0 and 2 (sorted positions 0
    and h).  Row 1 = [500, 501] shares row 2's x lines (31, 31) and delta
    widths, so it joins S_2 at zero cost (S_1 would add 2 lines); row 3 =
    [2, 3] joins S_1 (its lines 0, 0 are row 0's).  P:L175-212."""
    cols = [[0, 1], [500, 501], [498, 499], [2, 3]]
    rp = np.array([0, 2, 4, 6, 8], dtype=np.int64)
    A = Csr(4, 1000, rp, np.array(sum(cols, []), dtype=np.int32), np.ones(8), "hand")
    perm = bar.algorithm2(A.row_ptr, A.col, A.m, h=2)
    assert perm.tolist() == [0, 3, 2, 1]


def test_window_one_is_length_sort():
    """W = 1: every row goes to its own partition floor(pos / h) (it always
    has room when h | m), so the result is line 2's stable length sort."""
    A = random_block(seed=5, families=4, fam_rows=32)
    perm = bar.algorithm2(A.row_ptr, A.col, A.m, h=32, window=1)
    lens = np.diff(A.row_ptr)
    assert perm.tolist() == sorted(range(A.m), key=lambda i: (lens[i], i))


def test_window_covering_all_partitions_is_algorithm2():
    A = random_block(seed=6, families=3, fam_rows=32)
    Ab = Csr(90, A.n, A.row_ptr[:91].copy(), A.col[:A.row_ptr[90]], A.vals[:A.row_ptr[90]], "b")
    for M in (A, Ab):
        full = bar.algorithm2(M.row_ptr, M.col, M.m, h=32)
        assert np.array_equal(bar.algorithm2(M.row_ptr, M.col, M.m, h=32, window=3), full)


def test_algorithm2_output_is_equipartition():
    A = random_block(seed=7, families=5, fam_rows=32)
    for W in (None, 2):
        perm = bar.algorithm2(A.row_ptr, A.col, A.m, h=32, window=W)
        assert np.array_equal(np.sort(perm), np.arange(A.m))


def test_algorithm2_order_window1_is_the_order():
    """Reading R27: with a window of one partition every row lands in its own
    partition pos // h, so the result is the seed order itself (closed form),
    whatever order is passed for line 2."""
    from gen import random_block, row_block
    A = row_block(random_block(seed=3, families=5, fam_rows=32), 0, 150)
    order = bar.signature_order(A.row_ptr, A.col, A.m)
    got = bar.algorithm2(A.row_ptr, A.col, A.m, h=32, window=1, order=order)
    assert np.array_equal(got, order)
    rev = order[::-1].copy()
    assert np.array_equal(bar.algorithm2(A.row_ptr, A.col, A.m, h=32, window=1, order=rev), rev)


def test_algorithm2_default_order_is_length_sort():
    """order=None and an explicit stable length sort give the same greedy."""
    from gen import random_block
    A = random_block(seed=4, families=3, fam_rows=32)
    lens = np.diff(A.row_ptr)
    D = np.array(sorted(range(A.m), key=lambda i: (int(lens[i]), i)))
    assert np.array_equal(bar.algorithm2(A.row_ptr, A.col, A.m, h=32, window=2),
                          bar.algorithm2(A.row_ptr, A.col, A.m, h=32, window=2, order=D))
