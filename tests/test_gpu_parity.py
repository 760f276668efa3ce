"""GPU parity: libbro.so (through the C ABI) vs the CPU oracle (-m gpu).

Bar (north_star): decoded index streams bit-exact; fp64 y within
1e-12 * sum_j |a_ij||x_j| per row, fp32 within 1e-5 * the same sum.

Decoded indices come from the SAME kernel instances bro_spmv runs (their
decode mode, include/bro.h bro_decode_indices) and are compared with the
matrix's own column / row indices placed in the decode layout: the oracle's
decode(encode(idx)) == idx round trips (tests/test_oracle_bro.py) make that
the oracle's decode too.
"""
import numpy as np
import pytest

from gen import Csr, dense_band, make_config, make_x, permute_rows, random_csr, row_block
from oracle import hyb, spmv

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

TOL = {np.float64: 1e-12, np.float32: 1e-5}


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch.device("cuda:0")


def _run(lib, A, fmt, codec, dtype, dev, x=None, stream=None, **kw):
    M = lib.BroMatrix(A, fmt=fmt, codec=codec, device=0, dtype=dtype, **kw)
    if x is None:
        x = make_x(A.n, 3, dtype)
    xd = torch.from_numpy(np.ascontiguousarray(x, dtype=dtype)).to(dev)
    y = M.spmv(xd, stream=stream)
    torch.cuda.synchronize()
    return M, x, y.cpu().numpy()


def _check_y(A, x, y, dtype, chunk_rows=None):
    """Every row within tol * S_i of the oracle (chunked over rows for the
    full-size configs: each chunk is an exact row block of the oracle)."""
    rows = [(0, A.m)] if chunk_rows is None else [(r, min(A.m, r + chunk_rows))
                                                  for r in range(0, A.m, chunk_rows)]
    for r0, r1 in rows:
        B = row_block(A, r0, r1) if chunk_rows is not None else A
        y_ref, S = spmv.csr_spmv(B.row_ptr, B.col, B.vals.astype(dtype), x.astype(dtype))
        ok, err = spmv.within_tolerance(y[r0:r1], y_ref, S, TOL[dtype])
        bad = np.nonzero(~ok)[0]
        assert ok.all(), f"rows {r0}+: {bad.size} out of tolerance, first {bad[:5] + r0}, err {err[bad[:5]]}"


def ell_slot_reference(row_ptr, col, m, h):
    """Decoded column of every ELL slot, slot h*colptr[t] + h*j + r (V = 1
    slot order, include/bro.h), -1 for padding, built from the CSR itself."""
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    lens = np.diff(row_ptr)
    s = -(-m // h)
    lp = np.zeros(s * h, dtype=np.int64)
    lp[:m] = lens
    colptr = np.zeros(s + 1, dtype=np.int64)
    np.cumsum(lp.reshape(s, h).max(axis=1) if s else lp[:0], out=colptr[1:])
    out = np.full(h * int(colptr[-1]), -1, dtype=np.int32)
    nnz = int(row_ptr[-1])
    rows = np.repeat(np.arange(m, dtype=np.int64), lens)
    pos = np.arange(nnz, dtype=np.int64) - np.repeat(row_ptr[:-1], lens)
    out[h * colptr[rows // h] + h * pos + rows % h] = col
    return out


def check_decode(M, A, K=None):
    """Every slot of the ELL part and every COO row, bit-exact."""
    info = M.info
    cols_d, rows_d = M.decode_indices()
    torch.cuda.synchronize()
    if info["format"] == 0:        # ELL
        ep, ec = A.row_ptr, A.col
        cr = np.zeros(0, np.int64)
    elif info["format"] == 2:      # HYB
        ep, ec, _, cr, _, _ = hyb.hyb_split(A.row_ptr, A.col, A.vals, info["K"])
    else:                          # COO
        ep = None
        cr = np.repeat(np.arange(A.m, dtype=np.int64), np.diff(A.row_ptr))
    if ep is not None:
        if info["codec"]:
            ref = ell_slot_reference(ep, ec, A.m, info["slice_h"])
            got = cols_d.cpu().numpy()
        else:
            Cm, _ = hyb.ell_arrays(ep, ec, np.zeros(ec.size), info["K"])
            ref = np.full((info["K"], info["ell_pitch"]), -1, dtype=np.int32)
            ref[:, :A.m] = Cm.T
            ref = ref.ravel()
            got = cols_d.cpu().numpy()
        assert got.size == ref.size
        bad = np.nonzero(got != ref)[0]
        assert bad.size == 0, f"{bad.size} ELL slots differ, first {bad[:5]}: {got[bad[:5]]} vs {ref[bad[:5]]}"
    if info["nnz_coo"]:
        got = rows_d.cpu().numpy()
        assert np.array_equal(got, cr.astype(np.int32)), "COO rows differ"


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
    if name != "wide":
        check_decode(M, A)
    M.close()


# "wide" (n = 2^31 - 1) is left out below: its 16 GB x dominates the run time
# and it is covered by test_spmv_random
SMALL_CASES = [c for c in CASES if c[0] != "wide"]
INSTANCE_CASES = SMALL_CASES + [
    ("multiblock", lambda: random_csr(3000, 4000, 12, max_len=90, empty_frac=0.05)),
    ("short", lambda: random_csr(5000, 7000, 13, max_len=4, empty_frac=0.1)),
    ("wide31", lambda: random_csr(333, 2**20, 17, max_len=4, wide_cols=True)),
    ("mixed", lambda: random_csr(4000, 9000, 18, max_len=12, long_frac=0.05, long_len=300)),
]


def _fits(A, h, inst):
    from oracle import bro_ell
    if A.m == 0:
        return inst == 5
    l, S, _ = bro_ell.slice_shapes(A.row_ptr, A.col, A.m, h, 32)
    small, mid = S.max(initial=0) < 10, S.max(initial=0) < 18
    return {1: l.max(initial=0) <= 4, 2: True, 3: small, 4: mid, 5: True, 6: True, 7: True}[inst]


@pytest.mark.parametrize("inst", [1, 2, 3, 4, 5, 6, 7])
@pytest.mark.parametrize("h", [32, 64])
@pytest.mark.parametrize("V", [1, 4])
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_ell_instances(lib, dev, inst, h, V, dtype):
    """Every BRO-ELL kernel instance (bro_opts_t.ell_kernel: tiny, few-slice,
    small / mid / general window, split slices with 4 / 2 warps per slice —
    h = 64 runs the general instance for those) at h = 32 and 64, V = 1 and 4, gives the
    oracle's y on every row and decodes every slot bit-exactly, for the
    matrices it fits (empty rows, h not dividing m, 31-bit deltas, several
    32-column blocks per slice)."""
    ran = 0
    for name, mk in INSTANCE_CASES:
        A = mk()
        for fmt in ("ell", "hyb"):
            if fmt == "hyb":
                K = hyb.hyb_K(A.row_ptr)
                ep, ec, ev, _, _, _ = hyb.hyb_split(A.row_ptr, A.col, A.vals, K)
                E = Csr(A.m, A.n, ep, ec, ev)
            else:
                E = A
            if not _fits(E, h, inst):
                continue
            M, x, y = _run(lib, A, fmt, 1, dtype, dev, vec_words=V, slice_h=h, ell_kernel=inst)
            assert M.info["ell_kernel"] == inst and M.info["slice_h"] == h
            _check_y(A, x, y, dtype)
            check_decode(M, A)
            M.close()
            ran += 1
    assert ran > 0


COO_CASES = SMALL_CASES + [
    ("longrow", lambda: random_csr(40, 20000, 14, max_len=5, long_frac=0.2, long_len=5000)),
    ("tail", lambda: random_csr(300, 400, 15, max_len=4)),
    ("one_row", lambda: random_csr(1, 60000, 23, max_len=0, long_frac=1.0, long_len=40000)),
    ("many", lambda: random_csr(40000, 50000, 21, max_len=6, empty_frac=0.2, long_frac=0.002, long_len=900)),
]


@pytest.mark.parametrize("T", [8, 16, 32])
@pytest.mark.parametrize("codec", [1, 0])
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_coo_intervals(lib, dev, T, codec, dtype):
    """(BRO-)COO with 8, 16 and 32 entries per lane: rows spanning many lanes
    and intervals (deterministic fix-up), ragged last intervals, one-row
    intervals (width 0), lanes entirely past nnz; y on every row, rows
    decoded bit-exactly, and the same bits on a second call."""
    for _, mk in COO_CASES:
        A = mk()
        for fmt in ("coo", "hyb"):
            for V in ((1, 4) if codec else (4,)):
                M, x, y = _run(lib, A, fmt, codec, dtype, dev, vec_words=V, coo_T=T)
                assert M.info["coo_T"] == T
                _check_y(A, x, y, dtype)
                check_decode(M, A)
                y2 = M.spmv(torch.from_numpy(x).to(dev)).cpu().numpy()
                assert np.array_equal(y, y2)
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
    """Padding slots never read x (Alg. 1 line 17 skips invalid slots), nor
    do COO slots past nnz."""
    A = random_csr(300, 400, 6, max_len=30, empty_frac=0.2)
    x = make_x(A.n, 1)
    used = np.zeros(A.n, bool)
    used[A.col] = True
    x[~used] = np.inf
    x[0] = np.inf if not used[0] else x[0]
    for fmt in ("ell", "hyb", "coo"):
        for h in (32, 64):
            M, _, y = _run(lib, A, fmt, 1, np.float64, dev, x=x, slice_h=h)
            assert np.all(np.isfinite(y))
            _check_y(A, x, y, np.float64)
            M.close()


def test_vector_checks(lib, dev):
    """The binding rejects a y of the wrong dtype, length or device before
    any pointer reaches the library."""
    A = random_csr(64, 50, 11)
    M = lib.BroMatrix(A, fmt="ell", device=0)
    x = torch.zeros(50, dtype=torch.float64, device=dev)
    for y in (torch.zeros(64, dtype=torch.float32, device=dev), torch.zeros(63, dtype=torch.float64, device=dev),
              torch.zeros(128, dtype=torch.float64, device=dev)[::2], torch.zeros(64, dtype=torch.float64)):
        with pytest.raises(ValueError):
            M.spmv(x, y)
    with pytest.raises(ValueError):
        M.spmv(torch.zeros(49, dtype=torch.float64, device=dev))
    with pytest.raises(ValueError):
        M.spmv_host(np.zeros(49))
    with pytest.raises(ValueError):
        M.spmv_host(np.zeros(50), np.zeros(64, np.float32))
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


@pytest.mark.parametrize("h", [32, 64])
@pytest.mark.parametrize("codec", [1, 0])
def test_host_e2e_pipelined(lib, dev, h, codec):
    """ELL-only handles with x >= 4 MB run bro_spmv_host as the 8-piece
    pipeline (x pieces, row blocks gated by their column ranges, y pieces):
    bitwise equal to bro_spmv."""
    A = random_csr(600_000, 600_000, 31, max_len=12, empty_frac=0.05)
    M = lib.BroMatrix(A, fmt="ell", codec=codec, device=0, slice_h=h)
    x = make_x(A.n, 6)
    y = M.spmv(torch.from_numpy(x).to(dev)).cpu().numpy()
    y_host = M.spmv_host(x)
    assert np.array_equal(y, y_host)
    _check_y(A, x, y, np.float64)
    M.close()


def test_alias_rejected(lib, dev):
    A = random_csr(64, 64, 11)
    M = lib.BroMatrix(A, fmt="ell", device=0)
    xd = torch.from_numpy(make_x(64, 0)).to(dev)
    with pytest.raises(lib.BroError, match="ARG"):
        lib.bro_spmv(M.h, xd.data_ptr(), xd.data_ptr(), 0)
    M.close()


@pytest.mark.parametrize("min_bits", [1, 16, 31])
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_forced_widths_dense(lib, dev, min_bits, dtype):
    """Fig. 3 analog (NEXT-3): the dense matrix with every width
    forced up to min_bits runs the same kernels; y on every row and every
    slot decoded bit-exactly."""
    A = dense_band(50_000, 32)
    for h in (32, 64):
        M, x, y = _run(lib, A, "ell", 1, dtype, dev, min_bits=min_bits, slice_h=h)
        _check_y(A, x, y, dtype)
        check_decode(M, A)
        M.close()


# ---------------------------------------------------------------- the five configs

@pytest.mark.parametrize("cfg,fmt", [(1, "ell"), (2, "ell"), (3, "hyb")])
@pytest.mark.parametrize("codec", [1, 0])
def test_configs_full_oracle(lib, dev, cfg, fmt, codec):
    """C1-C3, both dtypes, bench.py's handle options: every row vs the
    oracle, every slot / COO row decoded bit-exactly."""
    for dtype in (np.float64, np.float32):
        A = make_config(cfg, dtype)
        M, x, y = _run(lib, A, fmt, codec, dtype, dev, x=make_x(A.n, cfg, dtype))
        _check_y(A, x, y, dtype)
        check_decode(M, A)
        M.close()


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_config4_bench_input(lib, dev, dtype):
    """C4 exactly as bench.py builds it (BAR method 3, reading R27, for this
    dtype) in bench.py's handle configuration: BRO-HYB on every row vs the
    oracle, every ELL slot and COO row decoded bit-exactly."""
    import bench
    A, fmt = bench.load_workload("C4", dtype, lib)
    M, x, y = _run(lib, A, fmt, 1, dtype, dev, x=make_x(A.n, 4, dtype))
    _check_y(A, x, y, dtype)
    check_decode(M, A)
    M.close()


def test_config4_bar_reordered_hyb(lib, dev):
    """C4: random-block, reordered with BAR (signature clustering), BRO-HYB
    fp32 and fp64 vs the oracle on every row, every index decoded."""
    A0 = make_config(4)
    perm = lib.bro_reorder_bar(A0.m, A0.n, A0.row_ptr, A0.col, method=0)
    A = permute_rows(A0, perm)
    for dtype in (np.float64, np.float32):
        M, x, y = _run(lib, A, "hyb", 1, dtype, dev, x=make_x(A.n, 4, dtype))
        _check_y(A, x, y, dtype)
        check_decode(M, A)
        M.close()
        Mb, x, y = _run(lib, A, "hyb", 0, dtype, dev, x=make_x(A.n, 4, dtype))
        _check_y(A, x, y, dtype)
        Mb.close()


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
@pytest.mark.parametrize("h", [0, 32])
def test_config5_full_size(lib, dev, dtype, h):
    """C5 at full size in bench.py's launch configuration (h = 0: auto) and
    at h = 32: x = 1 gives y_i = 27 - len_i exactly (small integers); random
    x: EVERY row against the oracle (chunked row blocks); every slot of the
    8M-row BRO-ELL decoded bit-exactly."""
    A = make_config(5, dtype)
    M = lib.BroMatrix(A, fmt="ell", codec=1, device=0, dtype=dtype, slice_h=h)
    tdt = torch.float64 if dtype == np.float64 else torch.float32
    y = M.spmv(torch.ones(A.n, dtype=tdt, device=dev)).cpu().numpy()
    assert np.array_equal(y, (27.0 - A.row_lengths()).astype(dtype))
    x = make_x(A.n, 5, dtype)
    y = M.spmv(torch.from_numpy(x).to(dev)).cpu().numpy()
    _check_y(A, x, y, dtype, chunk_rows=1_000_000)
    check_decode(M, A)
    M.close()


def test_config5_row_blocks(lib, dev):
    """Row-block partition used by the multi-GPU driver: local blocks with
    global columns reproduce the global product (one GPU, 4 blocks), every
    row within the oracle's bound."""
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
    _check_y(A, x, y, np.float64, chunk_rows=2_000_000)


@pytest.mark.parametrize("fmt", ["hyb", "coo"])
@pytest.mark.parametrize("codec", [1, 0])
def test_pdl_chain_same_bits(lib, dev, fmt, codec):
    """The COO kernel launched as a programmatic dependent of the ELL kernel
    (and the fix-up of the COO kernel) gives the same bits as plain stream
    order (bro_opts_t.pdl = 2), and the oracle's y."""
    A = random_csr(30000, 30000, 41, max_len=9, empty_frac=0.1, long_frac=0.01, long_len=2000)
    x = make_x(A.n, 7)
    ys = []
    for pdl in (0, 2):
        M, _, y = _run(lib, A, fmt, codec, np.float64, dev, x=x, pdl=pdl)
        _check_y(A, x, y, np.float64)
        ys.append(y)
        M.close()
    assert np.array_equal(ys[0], ys[1])


def _banded(m, bw, seed, per_row=24):
    """Random banded matrix: per_row distinct columns within [i - bw, i + bw]."""
    rng = np.random.default_rng(seed)
    rows, cols = [], []
    for i in range(m):
        lo, hi = max(0, i - bw), min(m, i + bw + 1)
        c = np.sort(rng.choice(np.arange(lo, hi), size=min(per_row, hi - lo), replace=False))
        rows.append(np.full(c.size, i))
        cols.append(c)
    r, c = np.concatenate(rows), np.concatenate(cols)
    rp = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(np.bincount(r, minlength=m), out=rp[1:])
    return Csr(m, m, rp, c.astype(np.int32), rng.uniform(-1, 1, c.size), f"band{m}_{bw}")


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_x_window_staging(lib, dev, dtype):
    """Row N1: the few-slice instance with each block's x window staged in
    shared memory by the TMA engine gives the same bits as the global-gather
    instance (same arithmetic, same order) and the oracle's y; windows that
    end at x's last element (n not a multiple of 16 bytes: the tail is
    gathered from global), a window too large to stage (no staging), and a
    misaligned x (the C ABI falls back to global gathers)."""
    cases = [make_config(1), make_config(2), _banded(20001, 300, 3), _banded(3000, 2999, 4, per_row=40)]
    for A in cases:
        A = A.astype(dtype)
        x = make_x(A.n, 11, dtype)
        Ms, ys = [], []
        for xs in (1, 0):
            M, _, y = _run(lib, A, "ell", 1, dtype, dev, x=x, x_stage=xs)
            _check_y(A, x, y, dtype)
            Ms.append(M)
            ys.append(y)
        staged = Ms[0].info["x_stage_bytes"]
        assert Ms[1].info["x_stage_bytes"] == 0
        if dtype == np.float64 and (A.name.startswith("C") or A.name == "band20001_300"):
            assert staged > 0, A.name
        assert np.array_equal(ys[0], ys[1]), A.name
        # misaligned x through the raw C ABI: one element into a padded buffer
        tdt = torch.float64 if dtype == np.float64 else torch.float32
        buf = torch.zeros(A.n + 1, dtype=tdt, device=dev)
        buf[1:] = torch.from_numpy(x).to(dev)
        yd = torch.empty(A.m, dtype=tdt, device=dev)
        lib.bro_spmv(Ms[0].h, buf.data_ptr() + buf.element_size(), yd.data_ptr(), 0)
        torch.cuda.synchronize()
        assert np.array_equal(yd.cpu().numpy(), ys[1])
        for M in Ms:
            M.close()


@pytest.mark.parametrize("inst", [1, 2, 3, 4, 5, 6, 7])
@pytest.mark.parametrize("h", [32, 64])
@pytest.mark.parametrize("V", [1, 4])
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_value_index_instances(lib, dev, inst, h, V, dtype):
    """value_codec 1 (reading R28) through every BRO-ELL instance, ELL and HYB
    handles, 1-byte and 2-byte codes: y on every row within the oracle's bound
    AND bit-identical to the same instance reading the stored values (the
    table returns the same bits, the FMAs run in the same order); decode mode
    bit-exact."""
    ran = 0
    for k, (name, mk) in enumerate(INSTANCE_CASES):
        A = mk()
        if A.nnz == 0 or A.n > 2**24:
            continue
        rng = np.random.default_rng(k)
        pool = rng.uniform(-1, 1, 3 if k % 2 else 300)
        A = Csr(A.m, A.n, A.row_ptr, A.col, pool[rng.integers(0, pool.size, A.nnz)], A.name)
        for fmt in ("ell", "hyb"):
            if fmt == "hyb":
                K = hyb.hyb_K(A.row_ptr)
                ep, ec, ev, _, _, _ = hyb.hyb_split(A.row_ptr, A.col, A.vals, K)
                E = Csr(A.m, A.n, ep, ec, ev)
            else:
                E = A
            if not _fits(E, h, inst):
                continue
            x = make_x(A.n, 9, dtype)
            M, _, y = _run(lib, A, fmt, 1, dtype, dev, x=x, vec_words=V, slice_h=h, ell_kernel=inst, value_codec=1)
            assert M.info["value_code_bytes"] == (1 if M.info["value_dict_size"] <= 256 else 2)
            _check_y(A, x, y, dtype)
            check_decode(M, A)
            M.close()
            Mp, _, yp = _run(lib, A, fmt, 1, dtype, dev, x=x, vec_words=V, slice_h=h, ell_kernel=inst)
            Mp.close()
            assert np.array_equal(y.view(np.uint8), yp.view(np.uint8)), f"{name} {fmt}: not bit-identical"
            ran += 1
    assert ran > 0


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_value_index_nonfinite_table(lib, dev, dtype):
    """A table whose first entry is +inf (D = [+inf, -1.0, -2.0] as unsigned
    bit patterns 0x7FF0.. < 0xBFF0.. < 0xC000..): padding slots take the first
    finite code (reading R28), so ragged rows give the same bits as the
    stored-values handle, non-finite rows included; finite rows within the
    oracle's bound."""
    A = random_csr(3000, 2500, 31, max_len=20, empty_frac=0.1)
    rng = np.random.default_rng(5)
    vals = np.array([np.inf, -1.0, -2.0], dtype=dtype)[rng.choice(3, A.nnz, p=[0.01, 0.49, 0.5])]
    A = Csr(A.m, A.n, A.row_ptr, A.col, vals, "inf-table")
    x = make_x(A.n, 2, dtype)
    for inst in (0, 1, 5):
        for h in (32, 64):
            if inst == 1:
                continue
            M, _, y = _run(lib, A, "ell", 1, dtype, dev, x=x, slice_h=h, ell_kernel=inst, value_codec=1)
            assert M.info["value_dict_size"] == 3
            M.close()
            P, _, yp = _run(lib, A, "ell", 1, dtype, dev, x=x, slice_h=h, ell_kernel=inst)
            P.close()
            assert np.array_equal(y.view(np.uint8), yp.view(np.uint8))
    fin = np.array([np.isfinite(vals[A.row_ptr[i]:A.row_ptr[i + 1]]).all() for i in range(A.m)])
    with np.errstate(invalid="ignore"):  # the inf rows make NaNs in the oracle too
        y_ref, S = spmv.csr_spmv(A.row_ptr, A.col, A.vals, x)
    ok, _ = spmv.within_tolerance(y[fin], np.asarray(y_ref)[fin], np.asarray(S)[fin], TOL[dtype])
    assert ok.all() and not np.isfinite(y[~fin]).any()


def test_value_index_scatter_rejected(lib, dev):
    """A value-indexed ELL handle has no scatter epilogue: more than one
    destination is BRO_ERR_UNSUPPORTED (one destination is a plain SpMV)."""
    A = make_config(1)
    M = lib.BroMatrix(A, fmt="ell", codec=1, device=0, value_codec=1)
    x = torch.from_numpy(make_x(A.n, 1)).to(dev)
    ys = [torch.empty(A.m, dtype=torch.float64, device=dev) for _ in range(2)]
    with pytest.raises(lib.BroError, match="UNSUPPORTED"):
        M.spmv_scatter(x, [t.data_ptr() for t in ys])
    M.spmv_scatter(x, [ys[0].data_ptr()])
    torch.cuda.synchronize()
    assert torch.equal(ys[0], M.spmv(x))
    M.close()


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_config5_value_index(lib, dev, dtype):
    """C5 with value indexing (D = {26, -1}, 1-byte codes) in bench.py's
    launch configuration: x = 1 gives y_i = 27 - len_i exactly; random x:
    bit-identical to the stored-values BRO-ELL handle (whose every row
    test_config5_full_size checks against the oracle) and every row against
    the oracle on 3 chunks."""
    A = make_config(5, dtype)
    M = lib.BroMatrix(A, fmt="ell", codec=1, device=0, dtype=dtype, value_codec=1)
    assert M.info["value_code_bytes"] == 1 and M.info["value_dict_size"] == 2
    tdt = torch.float64 if dtype == np.float64 else torch.float32
    y = M.spmv(torch.ones(A.n, dtype=tdt, device=dev)).cpu().numpy()
    assert np.array_equal(y, (27.0 - A.row_lengths()).astype(dtype))
    x = make_x(A.n, 5, dtype)
    xd = torch.from_numpy(x).to(dev)
    y = M.spmv(xd).cpu().numpy()
    M.close()
    P = lib.BroMatrix(A, fmt="ell", codec=1, device=0, dtype=dtype)
    yp = P.spmv(xd).cpu().numpy()
    P.close()
    assert np.array_equal(y.view(np.uint8), yp.view(np.uint8))
    for r0 in (0, 3_500_000, A.m - 500_000):
        B = row_block(A, r0, r0 + 500_000)
        y_ref, S = spmv.csr_spmv(B.row_ptr, B.col, B.vals, x)
        ok, _ = spmv.within_tolerance(y[r0:r0 + 500_000], y_ref, S, TOL[dtype])
        assert ok.all()
