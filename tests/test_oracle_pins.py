"""Pins of the CPU oracle against things other than itself (-m "not gpu").

Each test names what fixes the expected value: the paper's worked example
(tests/golden/paper_matrix_A.json, with PAPER.md line citations), a closed
form, brute force on tiny inputs, or an independent library (scipy.sparse).
"""
import numpy as np
import pytest
import scipy.sparse as sp

from gen import laplacian_2d, random_csr, stencil_27pt
from oracle import hyb, metrics, spmv


# ---------------------------------------------------------------- plain SpMV

def test_paper_A_matvec_by_hand(matrix_A):
    """A of P:L63 times x = [1..5]: rows 3*1+2*3, 2+12+15+16+5, 2+27+35, 32+15."""
    x = np.arange(1, 6, dtype=np.float64)
    y, S = spmv.csr_spmv(matrix_A.row_ptr, matrix_A.col, matrix_A.vals, x)
    assert [float(v) for v in y] == [9.0, 50.0, 64.0, 47.0]
    D = spmv.dense_from_csr(4, 5, matrix_A.row_ptr, matrix_A.col, matrix_A.vals)
    assert spmv.dense_spmv(D, x) == [9.0, 50.0, 64.0, 47.0]
    assert [float(v) for v in S] == [9.0, 50.0, 64.0, 47.0]  # all terms positive


@pytest.mark.parametrize("seed", range(6))
def test_csr_spmv_vs_dense_bruteforce(seed):
    A = random_csr(17, 13, seed, max_len=9, empty_frac=0.3)
    x = np.random.default_rng(seed).uniform(-1, 1, 13)
    y, S = spmv.csr_spmv(A.row_ptr, A.col, A.vals, x)
    D = spmv.dense_from_csr(A.m, A.n, A.row_ptr, A.col, A.vals)
    yd = spmv.dense_spmv(D, x)
    assert np.allclose(np.array(y, dtype=np.float64), yd, rtol=0, atol=1e-14)
    Dabs = [[abs(v) for v in row] for row in D]
    assert np.allclose(np.array(S, dtype=np.float64), spmv.dense_spmv(Dabs, np.abs(x)), atol=1e-14)


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_csr_spmv_vs_scipy(dtype):
    A = random_csr(3000, 2500, 7, max_len=60, empty_frac=0.2, long_frac=0.01,
                   long_len=400).astype(dtype)
    x = np.random.default_rng(1).uniform(-1, 1, A.n).astype(dtype)
    y, S = spmv.csr_spmv(A.row_ptr, A.col, A.vals, x)
    M = sp.csr_matrix((A.vals.astype(np.float64), A.col, A.row_ptr), shape=(A.m, A.n))
    ys = M @ x.astype(np.float64)
    assert np.all(np.abs(np.array(y, dtype=np.float64) - ys) <= 1e-13 * np.array(S, np.float64) + 1e-300)
    # sampled-row variant agrees with the whole-matrix variant
    rows = np.array([0, 5, 17, 2999])
    yr, Sr = spmv.csr_spmv_rows(A.row_ptr, A.col, A.vals, x, rows)
    assert np.all(np.abs(yr - y[rows]) <= 1e-15 * Sr + 1e-300)


def test_laplacian_closed_form():
    """4 on the diagonal, -1 off: with x = 1 interior rows give 0, edge rows 1,
    corner rows 2 — exact small integers."""
    A = laplacian_2d(64)
    assert A.m == 4096 and A.nnz == 5 * 64 * 64 - 4 * 64
    y, _ = spmv.csr_spmv(A.row_ptr, A.col, A.vals, np.ones(A.n))
    g = 64
    i, j = np.divmod(np.arange(A.m), g)
    nb = (i > 0).astype(int) + (i < g - 1) + (j > 0) + (j < g - 1)
    assert np.array_equal(np.array(y, dtype=np.float64), (4 - nb).astype(np.float64))


def test_27pt_closed_form():
    """26 on the diagonal, -1 off: with x = 1, y_i = 27 - len_i exactly; and
    nnz of the g^3 grid is (3g-2)^3 (598^3 at g = 200)."""
    A = stencil_27pt(12)
    assert A.nnz == (3 * 12 - 2) ** 3
    y, _ = spmv.csr_spmv(A.row_ptr, A.col, A.vals, np.ones(A.n))
    assert np.array_equal(np.array(y, dtype=np.float64), 27.0 - A.row_lengths())


def test_tolerance_helper():
    yref = np.array([1.0, 2.0], dtype=np.longdouble)
    S = np.array([1.0, 1.0], dtype=np.longdouble)
    ok, _ = spmv.within_tolerance(np.array([1.0 + 1e-13, 2.1]), yref, S, 1e-12)
    assert ok.tolist() == [True, False]


# ---------------------------------------------------------------- ELL / HYB

def _nulls(a):
    return [[None if v == hyb.PAD else int(v) + 1 for v in row] for row in a]


def test_ell_arrays_paper(matrix_A, golden_A):
    C, V = hyb.ell_arrays(matrix_A.row_ptr, matrix_A.col, matrix_A.vals)
    assert _nulls(C) == golden_A["ell"]["col_idx"]
    gv = golden_A["ell"]["vals"]
    for i in range(4):
        for j in range(5):
            if gv[i][j] is not None:
                assert V[i, j] == gv[i][j]
            else:
                assert V[i, j] == 0


def test_row_length_paper(matrix_A, golden_A):
    assert hyb.row_length(matrix_A.row_ptr).tolist() == golden_A["ellpack_r"]["row_length"]


def test_hyb_split_paper(matrix_A, golden_A):
    """P:L79 splits A at ELL width 3 with COO (2,4,4) and (2,5,1) (1-based).
    Reading R12: K = min{k : 3*|{len > k}| < m} gives 3; the literal
    'at least k' variant would give 4 and is rejected by this pin."""
    K = hyb.hyb_K(matrix_A.row_ptr)
    assert K == 3
    lens = hyb.row_length(matrix_A.row_ptr)
    at_least = next(k for k in range(10) if 3 * np.count_nonzero(lens >= k) < 4)
    assert at_least == 4  # the alternative reading disagrees with P:L79
    ep, ec, ev, cr, cc, cv = hyb.hyb_split(matrix_A.row_ptr, matrix_A.col, matrix_A.vals, K)
    g = golden_A["hyb"]
    assert (cr + 1).tolist() == g["coo_row_idx"]
    assert (cc + 1).tolist() == g["coo_col_idx"]
    assert cv.tolist() == g["coo_vals"]
    C, V = hyb.ell_arrays(ep, ec, ev, K)
    assert _nulls(C) == g["ell_col_idx"]


@pytest.mark.parametrize("seed", range(4))
def test_hyb_split_partition_random(seed):
    A = random_csr(300, 500, seed, max_len=30, empty_frac=0.2, long_frac=0.05, long_len=120)
    K = hyb.hyb_K(A.row_ptr)
    lens = A.row_lengths()
    assert 3 * np.count_nonzero(lens > K) < A.m
    assert K == 0 or 3 * np.count_nonzero(lens > K - 1) >= A.m
    ep, ec, ev, cr, cc, cv = hyb.hyb_split(A.row_ptr, A.col, A.vals, K)
    x = np.random.default_rng(seed).uniform(-1, 1, A.n)
    ye, _ = spmv.csr_spmv(ep, ec, ev, x)
    rp, c2, v2 = spmv.coo_to_csr(A.m, cr, cc, cv)
    yc, _ = spmv.csr_spmv(rp, c2, v2, x)
    y, S = spmv.csr_spmv(A.row_ptr, A.col, A.vals, x)
    assert np.all(np.abs(ye + yc - y) <= 1e-15 * S + 1e-300)


# ---------------------------------------------------------------- eta / kappa

def test_eta_kappa_paper(golden_A):
    """kappa = 1/(1-eta) maps the break-even savings 17/9/23 % to the
    compression ratios 1.2/1.1/1.3x printed at P:L250."""
    g = golden_A["eta_kappa"]
    for e, k in g["pairs"]:
        assert abs(metrics.kappa(e) - k) <= g["kappa_rounding"]
    # matrix A: 32-bit stream vs 80-byte col_idx
    e = metrics.eta(32 / 8, 80)
    assert abs(e - 0.95) < 1e-12 and abs(metrics.kappa(e) - 20.0) < 1e-9
    assert metrics.ell_index_bytes(4, 5) == golden_A["bro_ell"]["col_idx_bytes"]
