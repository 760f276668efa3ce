"""GPU: kernel instances chosen by size or by tuning variables, against the
oracle (-m gpu): the persistent pipelined (BRO-)COO kernel (coo_spmv_pipe;
BRO_COO_KERNEL=2 forces it wherever there are >= 8 intervals,
BRO_COO_PIPE_MINB picks 16 or 24 warps/SM) on cases spanning many intervals,
a ragged last interval, rows crossing intervals and warps, and long rows; and
the general BRO-ELL instances a large matrix can take (window rows, cp.async
value ring)."""
import os

import numpy as np
import pytest

from gen import make_config, make_x, random_csr
from oracle import spmv

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

TOL = {np.float64: 1e-12, np.float32: 1e-5}


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch.device("cuda:0")


@pytest.fixture
def pipe_env():
    old = {k: os.environ.get(k) for k in ("BRO_COO_KERNEL", "BRO_COO_PIPE_MINB")}
    yield
    for k, v in old.items():
        if v is None:
            os.environ.pop(k, None)
        else:
            os.environ[k] = v


CASES = [
    # ~ 9.5 intervals of COO entries, ragged tail, short rows
    ("short", lambda: random_csr(4000, 5000, 21, max_len=5, empty_frac=0.2)),
    # long rows crossing many intervals and warps
    ("long", lambda: random_csr(3000, 9000, 22, max_len=12, long_frac=0.05, long_len=4000)),
    # one row of 40,000 entries (every interval one row, width 0)
    ("one_row", lambda: random_csr(1, 60000, 23, max_len=0, long_frac=1.0, long_len=40000)),
    ("c1", lambda: make_config(1)),
]


@pytest.mark.parametrize("name,mk", CASES, ids=[c[0] for c in CASES])
@pytest.mark.parametrize("fmt", ["coo", "hyb"])
@pytest.mark.parametrize("codec", [1, 0])
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
@pytest.mark.parametrize("minb", ["2", "3"])
def test_coo_pipe_vs_oracle(lib, dev, pipe_env, name, mk, fmt, codec, dtype, minb):
    A = mk()
    os.environ["BRO_COO_KERNEL"] = "2"
    os.environ["BRO_COO_PIPE_MINB"] = minb
    for V in ((1, 4) if codec else (4,)):
        M = lib.BroMatrix(A, fmt=fmt, codec=codec, device=0, dtype=dtype, vec_words=V)
        if M.info["n_intervals"] < 8:
            M.close()
            pytest.skip("fewer than 8 intervals: the per-unit kernel runs")
        x = make_x(A.n, 9, dtype)
        y = M.spmv(torch.from_numpy(x).to(dev))
        torch.cuda.synchronize()
        y_ref, S = spmv.csr_spmv(A.row_ptr, A.col, A.vals.astype(dtype), x)
        ok, err = spmv.within_tolerance(y.cpu().numpy(), y_ref, S, TOL[dtype])
        bad = np.nonzero(~ok)[0]
        assert ok.all(), f"V={V}: {bad.size} rows out of tolerance, first {bad[:5]} err {err[bad[:5]]}"
        # deterministic: a second call gives the same bits
        y2 = M.spmv(torch.from_numpy(x).to(dev))
        torch.cuda.synchronize()
        assert torch.equal(y, y2)
        M.close()


def test_coo_pipe_config4_sampled(lib, dev, pipe_env):
    """C4 (the config BRO_COO_KERNEL=0's auto choice sends to the pipelined
    kernel) on 3,000 sampled rows, both dtypes."""
    import bench
    os.environ["BRO_COO_KERNEL"] = "0"
    for dtype in (np.float64, np.float32):
        A, _ = bench.load_workload("C4", dtype, lib)
        M = lib.BroMatrix(A, fmt="hyb", codec=1, device=0, dtype=dtype)
        x = make_x(A.n, 4, dtype)
        y = M.spmv(torch.from_numpy(x).to(dev)).cpu().numpy()
        rows = np.random.default_rng(5).integers(0, A.m, 3000)
        yr, S = spmv.csr_spmv_rows(A.row_ptr, A.col, A.vals.astype(dtype), x, rows)
        ok, _ = spmv.within_tolerance(y[rows], yr, S, TOL[dtype])
        assert ok.all()
        M.close()


@pytest.fixture
def ell_env():
    keys = ("BRO_ELL_CPV", "BRO_ELL_SMALLWIN", "BRO_ELL_FEW_G", "BRO_ELL_TINY")
    old = {k: os.environ.get(k) for k in keys}
    yield
    for k, v in old.items():
        if v is None:
            os.environ.pop(k, None)
        else:
            os.environ[k] = v


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
@pytest.mark.parametrize("env", ["BRO_ELL_SMALLWIN=0", "BRO_ELL_SMALLWIN=1", "BRO_ELL_CPV=1", "BRO_ELL_CPV=2"])
def test_bro_ell_instances_stencil(lib, dev, ell_env, dtype, env):
    """The general BRO-ELL instances a large matrix can take (34-row window,
    10-row small window, cp.async value ring with 1 or 2 groups ahead) on a
    27-point stencil big enough to fill the GPU (6,750 slices, S <= 7),
    every row against the oracle."""
    from gen.matrices import stencil_27pt
    A = stencil_27pt(60)
    k, v = env.split("=")
    os.environ[k] = v
    M = lib.BroMatrix(A, fmt="ell", codec=1, device=0, dtype=dtype)
    assert M.info["n_slices"] >= 148 * 32
    x = make_x(A.n, 6, dtype)
    y = M.spmv(torch.from_numpy(x).to(dev))
    torch.cuda.synchronize()
    y_ref, S = spmv.csr_spmv(A.row_ptr, A.col, A.vals.astype(dtype), x)
    ok, err = spmv.within_tolerance(y.cpu().numpy(), y_ref, S, TOL[dtype])
    assert ok.all(), f"{np.count_nonzero(~ok)} rows out of tolerance"
    M.close()


TINY_CASES = [
    ("short", lambda: random_csr(20000, 30000, 31, max_len=4, empty_frac=0.2)),
    ("wide", lambda: random_csr(9000, 2**31 - 1, 32, max_len=4, wide_cols=True)),
    ("ragged_m", lambda: random_csr(7777, 5000, 33, max_len=3, empty_frac=0.5)),
]


@pytest.mark.parametrize("name,mk", TINY_CASES, ids=[c[0] for c in TINY_CASES])
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
@pytest.mark.parametrize("tiny", ["1", "2"])
def test_bro_ell_tiny_slices(lib, dev, ell_env, name, mk, dtype, tiny):
    """The register-resident tiny-slice BRO-ELL kernel (every slice <= 4
    columns; BRO_ELL_TINY = 1: one slice per warp iteration, 2: two
    interleaved) for V = 1, 2, 4, including 31-bit first deltas, empty rows and
    m not a multiple of 32; every row against the oracle."""
    A = mk()
    os.environ["BRO_ELL_TINY"] = tiny
    x = make_x(A.n, 7, dtype)
    y_ref, S = spmv.csr_spmv(A.row_ptr, A.col, A.vals.astype(dtype), x)
    xd = torch.from_numpy(x).to(dev)
    for V in (1, 2, 4):
        M = lib.BroMatrix(A, fmt="ell", codec=1, device=0, dtype=dtype, vec_words=V)
        assert M.info["K"] <= 4
        y = M.spmv(xd)
        torch.cuda.synchronize()
        ok, err = spmv.within_tolerance(y.cpu().numpy(), y_ref, S, TOL[dtype])
        assert ok.all(), f"V={V}: {np.count_nonzero(~ok)} rows out of tolerance"
        M.close()
    os.environ.pop("BRO_ELL_TINY", None)


@pytest.fixture
def e2e_env():
    keys = ("BRO_E2E_CHUNKS", "BRO_E2E_MIN_KB")
    old = {k: os.environ.get(k) for k in keys}
    os.environ["BRO_E2E_MIN_KB"] = "0"  # pipeline these small cases too
    yield
    for k, v in old.items():
        if v is None:
            os.environ.pop(k, None)
        else:
            os.environ[k] = v


E2E_CASES = [
    ("c1", lambda: make_config(1)),
    ("banded_ragged", lambda: random_csr(10007, 10007, 41, max_len=30, empty_frac=0.1)),
    ("wide", lambda: random_csr(3000, 50000, 42, max_len=8, wide_cols=True)),
    ("empty_rows", lambda: random_csr(2000, 2000, 43, max_len=0)),
]


@pytest.mark.parametrize("name,mk", E2E_CASES, ids=[c[0] for c in E2E_CASES])
@pytest.mark.parametrize("codec", [1, 0])
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_spmv_host_pipelined(lib, dev, e2e_env, name, mk, codec, dtype):
    """bro_spmv_host of an ELL-only handle pipelines x pieces, row blocks and
    y pieces over three streams; every chunking gives exactly bro_spmv's y
    (same kernels, same per-row arithmetic)."""
    A = mk()
    x = make_x(A.n, 8, dtype)
    M = lib.BroMatrix(A, fmt="ell", codec=codec, device=0, dtype=dtype)
    y_dev = M.spmv(torch.from_numpy(x).to(dev)).cpu().numpy()
    xh = torch.from_numpy(x).pin_memory().numpy()
    for K in ("1", "2", "8", "64"):
        os.environ["BRO_E2E_CHUNKS"] = K
        yh = torch.empty(A.m, dtype=torch.float64 if dtype == np.float64 else torch.float32).pin_memory().numpy()
        yh[:] = np.nan
        M.spmv_host(xh, yh)
        assert np.array_equal(yh, y_dev), f"K={K}"
    M.close()
