"""GPU parity: libbro.so (through the C ABI) vs the CPU oracle (-m gpu).

Bar (north_star): decoded index streams bit-exact; fp64 y within
1e-12 * sum_j |a_ij||x_j| per row, fp32 within 1e-5 * the same sum.
"""
import numpy as np
import pytest

from gen import Csr, make_config, make_x, random_csr, row_block
from oracle import bro_coo, bro_ell, hyb, spmv

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

TOL = {np.float64: 1e-12, np.float32: 1e-5}


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch.device("cuda:0")


def _run(lib, A, fmt, codec, dtype, dev, V=4, x=None, stream=None):
    M = lib.BroMatrix(A, fmt=fmt, codec=codec, device=0, dtype=dtype, vec_words=V)
    if x is None:
        x = make_x(A.n, 3, dtype)
    xd = torch.from_numpy(np.ascontiguousarray(x, dtype=dtype)).to(dev)
    y = M.spmv(xd, stream=stream)
    torch.cuda.synchronize()
    return M, x, y.cpu().numpy()


def _check_y(A, x, y, dtype):
    y_ref, S = spmv.csr_spmv(A.row_ptr, A.col, A.vals.astype(dtype), x.astype(dtype))
    ok, err = spmv.within_tolerance(y, y_ref, S, TOL[dtype])
    bad = np.nonzero(~ok)[0]
    assert ok.all(), f"{bad.size} rows out of tolerance, first {bad[:5]}, err {err[bad[:5]]}"


CASES = [
    ("tiny", lambda: random_csr(7, 9, 0, max_len=5, empty_frac=0.3)),
    ("ragged", lambda: random_csr(1000, 1500, 1, max_len=50, empty_frac=0.1)),
    ("wide", lambda: random_csr(777, 2**31 - 1, 2, max_len=20, wide_cols=True)),
    ("long", lambda: random_csr(600, 5000, 3, max_len=10, long_frac=0.03, long_len=3000)),
    ("all_empty", lambda: random_csr(100, 50, 4, max_len=0)),
]


@pytest.mark.parametrize("name,mk", CASES, ids=[c[0] for c in CASES])
@pytest.mark.parametrize("fmt", ["ell", "hyb", "coo"])
@pytest.mark.parametrize("codec", [1, 0])
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_spmv_random(lib, dev, name, mk, fmt, codec, dtype):
    A = mk()
    M, x, y = _run(lib, A, fmt, codec, dtype, dev)
    _check_y(A, x, y, dtype)
    M.close()


@pytest.mark.parametrize("V", [1, 2, 4])
def test_vec_words_variants(lib, dev, V):
    A = random_csr(2000, 3000, 5, max_len=90, empty_frac=0.05, long_frac=0.01, long_len=600)
    for fmt in ("ell", "hyb"):
        M, x, y = _run(lib, A, fmt, 1, np.float64, dev, V=V)
        _check_y(A, x, y, np.float64)
        M.close()


# "wide" (n = 2^31 - 1) is left out: its 16 GB x dominates the run time and it
# is already covered by test_spmv_random
SMALL_CASES = [c for c in CASES if c[0] != "wide"]
BULK_CASES = SMALL_CASES + [
    ("multiblock", lambda: random_csr(3000, 4000, 12, max_len=90, empty_frac=0.05)),
    ("short", lambda: random_csr(5000, 7000, 13, max_len=3, empty_frac=0.1)),
]


@pytest.mark.parametrize("kernel", ["bulk", "od"])
@pytest.mark.parametrize("ring_kb", ["", "1", "64"])
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_bro_ell_v1_kernels(lib, dev, kernel, ring_kb, dtype, monkeypatch):
    """V = 1 (the paper's multiplexing): the bulk-staged kernel (TMA ring of
    whole slices, 2..8 slots per warp depending on BRO_RING_KB) and the
    register-staged kernel give the oracle's y on every case, including slices
    with several 32-column blocks and slices too large to stage."""
    monkeypatch.setenv("BRO_ELL_KERNEL", "1" if kernel == "od" else "2")
    monkeypatch.setenv("BRO_RING_KB", ring_kb)
    for _, mk in BULK_CASES:
        A = mk()
        for fmt in ("ell", "hyb"):
            M, x, y = _run(lib, A, fmt, 1, dtype, dev, V=1)
            _check_y(A, x, y, dtype)
            M.close()


@pytest.mark.parametrize("short", ["0", "1"])
@pytest.mark.parametrize("V", [1, 2, 4])
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_short_slice_kernel(lib, dev, short, V, dtype, monkeypatch):
    """Slices of <= 4 columns (the ELL part of webbase-like HYB) run in the
    short-slice instance (G = 4, 6-row window, more resident warps); it and
    the general instance give the oracle's y, with empty rows, h not dividing
    m and 31-bit deltas."""
    monkeypatch.setenv("BRO_ELL_SHORT", short)
    for A in (random_csr(5001, 7000, 16, max_len=4, empty_frac=0.2),
              random_csr(333, 2**20, 17, max_len=4, wide_cols=True),
              random_csr(4000, 9000, 18, max_len=12, long_frac=0.05, long_len=300)):
        for fmt in ("ell", "hyb"):
            M, x, y = _run(lib, A, fmt, 1, dtype, dev, V=V)
            _check_y(A, x, y, dtype)
            M.close()


@pytest.mark.parametrize("upi", ["1", "2", "4"])
@pytest.mark.parametrize("codec", [1, 0])
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_coo_work_units(lib, dev, upi, codec, dtype, monkeypatch):
    """COO traversal split into 1, 2 or 4 work units per 1024-entry interval
    (carries per unit, deterministic fix-up over units) gives the oracle's y,
    including units entirely past nnz and rows spanning many units."""
    monkeypatch.setenv("BRO_COO_UPI", upi)
    cases = SMALL_CASES + [("longrow", lambda: random_csr(40, 20000, 14, max_len=5, long_frac=0.2,
                                                    long_len=5000)),
                     ("tail", lambda: random_csr(300, 400, 15, max_len=4))]
    for _, mk in cases:
        A = mk()
        for fmt in ("coo", "hyb"):
            for V in (1, 4):
                M, x, y = _run(lib, A, fmt, codec, dtype, dev, V=V)
                _check_y(A, x, y, dtype)
                M.close()


def test_empty_matrix(lib, dev):
    A = Csr(0, 5, np.zeros(1, np.int64), np.zeros(0, np.int32), np.zeros(0), "empty")
    M = lib.BroMatrix(A, fmt="hyb", device=0)
    y = M.spmv(torch.zeros(5, dtype=torch.float64, device=dev))
    torch.cuda.synchronize()
    assert y.numel() == 0
    M.close()


def test_single_long_row_spans_intervals(lib, dev):
    """One row of 10,000 entries: COO intervals whose first = last row."""
    n = 20000
    cols = np.sort(np.random.default_rng(0).choice(n, 10000, replace=False))
    rp = np.array([0, 0, 10000, 10000], dtype=np.int64)
    A = Csr(3, n, rp, cols.astype(np.int32), np.random.default_rng(1).uniform(-1, 1, 10000), "longrow")
    for fmt in ("coo", "hyb"):
        for codec in (1, 0):
            M, x, y = _run(lib, A, fmt, codec, np.float64, dev)
            _check_y(A, x, y, np.float64)
            M.close()


def test_x_with_inf_outside_pattern(lib, dev):
    """Padding slots never read x (Alg. 1 line 17 skips invalid slots)."""
    A = random_csr(300, 400, 6, max_len=30, empty_frac=0.2)
    x = make_x(A.n, 1)
    used = np.zeros(A.n, bool)
    used[A.col] = True
    x[~used] = np.inf
    for fmt in ("ell", "hyb", "coo"):
        M, _, y = _run(lib, A, fmt, 1, np.float64, dev, x=x)
        assert np.all(np.isfinite(y))
        _check_y(A, x, y, np.float64)
        M.close()


def test_decode_parity_bit_exact(lib, dev):
    A = random_csr(3000, 100000, 8, max_len=60, empty_frac=0.1, long_frac=0.02, long_len=500,
                   wide_cols=True)
    for V in (1, 4):
        M = lib.BroMatrix(A, fmt="hyb", codec=1, device=0, vec_words=V)
        info = M.info
        cols_d = torch.empty(info["ell_slots"], dtype=torch.int32, device=dev)
        rows_d = torch.empty(max(info["nnz_coo"], 1), dtype=torch.int32, device=dev)
        lib.bro_decode_indices(M.h, cols_d.data_ptr(), rows_d.data_ptr(), 0)
        torch.cuda.synchronize()
        K = info["K"]
        ep, ec, ev, cr, cc, cv = hyb.hyb_split(A.row_ptr, A.col, A.vals, K)
        E = bro_ell.encode(ep, ec, ev, A.m, A.n, V=V)
        assert np.array_equal(cols_d.cpu().numpy(), bro_ell.decoded_slots(E))
        C = bro_coo.encode(cr, cc, cv, V=V)
        assert np.array_equal(rows_d.cpu().numpy()[:info["nnz_coo"]], bro_coo.decode_rows(C))
        M.close()


def test_deterministic(lib, dev):
    A = random_csr(5000, 5000, 9, max_len=20, long_frac=0.01, long_len=2500)
    M = lib.BroMatrix(A, fmt="hyb", device=0)
    xd = torch.from_numpy(make_x(A.n, 0)).to(dev)
    y1 = M.spmv(xd).clone()
    y2 = M.spmv(xd)
    torch.cuda.synchronize()
    assert torch.equal(y1, y2)
    M.close()


def test_side_stream_and_host_e2e(lib, dev):
    A = random_csr(4000, 4000, 10, max_len=40, long_frac=0.01, long_len=800)
    M = lib.BroMatrix(A, fmt="hyb", device=0)
    x = make_x(A.n, 4)
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        xd = torch.from_numpy(x).to(dev)
        y = M.spmv(xd, stream=s)
    s.synchronize()
    y_host = M.spmv_host(x)
    assert np.array_equal(y.cpu().numpy(), y_host)
    _check_y(A, x, y_host, np.float64)
    M.close()


def test_alias_rejected(lib, dev):
    A = random_csr(64, 64, 11)
    M = lib.BroMatrix(A, fmt="ell", device=0)
    xd = torch.from_numpy(make_x(64, 0)).to(dev)
    with pytest.raises(lib.BroError, match="ARG"):
        lib.bro_spmv(M.h, xd.data_ptr(), xd.data_ptr(), 0)
    M.close()


# ---------------------------------------------------------------- the five configs

@pytest.mark.parametrize("cfg,fmt", [(1, "ell"), (2, "ell"), (3, "hyb")])
@pytest.mark.parametrize("codec", [1, 0])
def test_configs_full_oracle(lib, dev, cfg, fmt, codec):
    for dtype in (np.float64, np.float32):
        A = make_config(cfg, dtype)
        M, x, y = _run(lib, A, fmt, codec, dtype, dev, x=make_x(A.n, cfg, dtype))
        _check_y(A, x, y, dtype)
        M.close()


def test_config4_bar_reordered_hyb(lib, dev):
    """C4: random-block, reordered with BAR (signature clustering), BRO-HYB
    fp32 and fp64 vs the oracle on every row."""
    from gen import permute_rows
    A0 = make_config(4)
    perm = lib.bro_reorder_bar(A0.m, A0.n, A0.row_ptr, A0.col, method=0)
    A = permute_rows(A0, perm)
    for dtype in (np.float64, np.float32):
        M, x, y = _run(lib, A, "hyb", 1, dtype, dev, x=make_x(A.n, 4, dtype))
        _check_y(A, x, y, dtype)
        M.close()


def test_config5_full_size(lib, dev):
    """C5 at full size in bench.py's launch configuration: every row against
    the closed form (x = 1 -> y_i = 27 - len_i exactly), sampled rows against
    the oracle for random x, and sampled slices decoded bit-exactly."""
    A = make_config(5)
    M = lib.BroMatrix(A, fmt="ell", codec=1, device=0)
    ones = torch.ones(A.n, dtype=torch.float64, device=dev)
    y = M.spmv(ones).cpu().numpy()
    assert np.array_equal(y, 27.0 - A.row_lengths())
    x = make_x(A.n, 5)
    y = M.spmv(torch.from_numpy(x).to(dev)).cpu().numpy()
    rows = np.unique(np.concatenate([np.arange(40), A.m - 1 - np.arange(40),
                                     np.random.default_rng(0).integers(0, A.m, 3000)]))
    yr, S = spmv.csr_spmv_rows(A.row_ptr, A.col, A.vals, x, rows)
    ok, err = spmv.within_tolerance(y[rows], yr, S, 1e-12)
    assert ok.all(), float(err.max())
    cols_d = torch.empty(M.info["ell_slots"], dtype=torch.int32, device=dev)
    lib.bro_decode_indices(M.h, cols_d.data_ptr(), 0, 0)
    cols = cols_d.cpu().numpy()
    sample = [0, 3, 6250, 125000, 249999]
    E = bro_ell.encode(A.row_ptr, A.col, A.vals, A.m, A.n, slices=sample)
    ref = bro_ell.decoded_slots(E, slices=sample)
    for t in sample:
        a, b = 32 * int(E.colptr[t]), 32 * int(E.colptr[t + 1])
        assert np.array_equal(cols[a:b], ref[a:b])
    M.close()


def test_config5_full_size_f32(lib, dev):
    """C5 fp32 at full size (bench.py --dtype f32's launch configuration):
    x = 1 gives small integers, exact in fp32 (y_i = 27 - len_i); sampled
    rows against the oracle within 1e-5 * sum|a||x| for random x."""
    A = make_config(5, np.float32)
    M = lib.BroMatrix(A, fmt="ell", codec=1, device=0, dtype=np.float32)
    ones = torch.ones(A.n, dtype=torch.float32, device=dev)
    y = M.spmv(ones).cpu().numpy()
    assert np.array_equal(y, (27.0 - A.row_lengths()).astype(np.float32))
    x = make_x(A.n, 5, np.float32)
    y = M.spmv(torch.from_numpy(x).to(dev)).cpu().numpy()
    rows = np.unique(np.concatenate([np.arange(40), A.m - 1 - np.arange(40),
                                     np.random.default_rng(2).integers(0, A.m, 3000)]))
    yr, S = spmv.csr_spmv_rows(A.row_ptr, A.col, A.vals.astype(np.float32), x, rows)
    ok, err = spmv.within_tolerance(y[rows], yr, S, TOL[np.float32])
    assert ok.all(), float(err.max())
    M.close()


def test_config5_row_blocks(lib, dev):
    """Row-block partition used by the multi-GPU driver: local blocks with
    global columns reproduce the global product (one GPU, 4 blocks)."""
    from paper_conf_sc_tangtrwckgtw13_b200.dist import partition_rows
    A = make_config(5)
    x = make_x(A.n, 5)
    xd = torch.from_numpy(x).to(dev)
    bounds = partition_rows(A.row_ptr, 4)
    ys = []
    for p in range(4):
        B = row_block(A, bounds[p], bounds[p + 1])
        M = lib.BroMatrix(B, fmt="ell", device=0)
        ys.append(M.spmv(xd).cpu().numpy())
        M.close()
    y = np.concatenate(ys)
    rows = np.random.default_rng(1).integers(0, A.m, 2000)
    yr, S = spmv.csr_spmv_rows(A.row_ptr, A.col, A.vals, x, rows)
    ok, _ = spmv.within_tolerance(y[rows], yr, S, 1e-12)
    assert ok.all()
