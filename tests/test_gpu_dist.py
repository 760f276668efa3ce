"""GPU: the fused exchange surface (bro_spmv_scatter) and the row-block
iteration x_{k+1} = A.x_k with every exchange mode, against the CPU oracle
(-m gpu).  The multi-rank cases run 2 processes on the one GPU of the test
box over gloo (the NCCL path needs one GPU per rank); they exercise the same
dist.py schedule, handles and kernels as bench.py --gpus N.
"""
import os
import socket

import numpy as np
import pytest

from gen import make_config, make_x, random_csr
from oracle import spmv

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch.device("cuda:0")


SCATTER_CASES = [
    ("ragged", lambda: random_csr(1000, 1500, 1, max_len=50, empty_frac=0.1)),
    ("long", lambda: random_csr(600, 5000, 3, max_len=10, long_frac=0.03, long_len=3000)),
    ("c1", lambda: make_config(1)),
]


@pytest.mark.parametrize("name,mk", SCATTER_CASES, ids=[c[0] for c in SCATTER_CASES])
@pytest.mark.parametrize("fmt", ["ell", "hyb", "coo"])
@pytest.mark.parametrize("codec", [1, 0])
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_spmv_scatter_matches_spmv(lib, dev, name, mk, fmt, codec, dtype):
    """Every destination of bro_spmv_scatter holds exactly bro_spmv's y (same
    kernels, same summation order), for 1, 3 and BRO_MAX_DST destinations."""
    A = mk()
    M = lib.BroMatrix(A, fmt=fmt, codec=codec, device=0, dtype=dtype)
    x = torch.from_numpy(make_x(A.n, 5, dtype)).to(dev)
    y = M.spmv(x)
    tdt = y.dtype
    for nd in (1, 3, lib.BRO_MAX_DST):
        bufs = [torch.full((A.m + 7,), float("nan"), dtype=tdt, device=dev) for _ in range(nd)]
        # destinations at different offsets inside their buffers (peer blocks)
        ptrs = [b.data_ptr() + (i % 4) * b.element_size() for i, b in enumerate(bufs)]
        M.spmv_scatter(x, ptrs)
        torch.cuda.synchronize()
        for i, b in enumerate(bufs):
            o = i % 4
            assert torch.equal(b[o:o + A.m], y), f"destination {i}"
            assert torch.isnan(b[:o]).all() and torch.isnan(b[o + A.m:]).all()  # nothing outside
    M.close()


def test_spmv_scatter_errors(lib, dev):
    A = random_csr(100, 100, 0, max_len=5)
    M = lib.BroMatrix(A, fmt="ell", device=0)
    x = torch.from_numpy(make_x(A.n, 1)).to(dev)
    y = torch.empty(A.m, dtype=torch.float64, device=dev)
    with pytest.raises(lib.BroError, match="BRO_ERR_ARG"):
        M.spmv_scatter(x, [])
    with pytest.raises(lib.BroError, match="BRO_ERR_ARG"):
        M.spmv_scatter(x, [y.data_ptr()] * (lib.BRO_MAX_DST + 1))
    with pytest.raises(lib.BroError, match="BRO_ERR_ARG"):
        M.spmv_scatter(x, [y.data_ptr(), x.data_ptr()])  # aliasing x
    with pytest.raises(lib.BroError, match="BRO_ERR_ARG"):
        M.spmv_scatter(x, [y.data_ptr(), 0])
    M.close()


def test_row_block_single_rank_iteration(lib, dev):
    """world = 1: step() is x_{k+1} = A.x_k in the double-buffered replicas."""
    from paper_conf_sc_tangtrwckgtw13_b200.dist import RowBlockSpmv
    A = make_config(1)
    x0 = make_x(A.n, 1) * 0.1
    blk = RowBlockSpmv(A, 0, 1, dev, fmt="ell")
    blk.set_x(x0)
    prev = x0.copy()
    for _ in range(3):
        blk.step()
        torch.cuda.synchronize()
        got = blk.x_current().cpu().numpy()
        y_ref, S = spmv.csr_spmv(A.row_ptr, A.col, A.vals, prev)
        assert spmv.within_tolerance(got, y_ref, S, 1e-12)[0].all()
        prev = got
    blk.close()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _dist_worker(rank, world, port, q, exchange, fmt, cfg, iters):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    try:
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        from paper_conf_sc_tangtrwckgtw13_b200.dist import RowBlockSpmv, partition_rows
        if cfg == "c1":
            A = make_config(1)
            bounds = None
        else:  # unequal blocks: padded x layout + column remap
            A = random_csr(3000, 3000, 11, max_len=30, empty_frac=0.05, long_frac=0.0, long_len=0)
            bounds = partition_rows(A.row_ptr, world)
        x0 = make_x(A.n, 2) * 0.1
        dev = torch.device("cuda", 0)
        blk = RowBlockSpmv(A, rank, world, dev, fmt=fmt, bounds=bounds, exchange=exchange)
        blk.set_x(x0)
        stream = torch.cuda.current_stream(dev)
        # every iteration, every row: x_{k+1} within 1e-12 * S_i of the
        # oracle's A.x_k applied to the GPU's own x_k (north_star bound)
        ok = True
        prev = x0.copy()
        for _ in range(iters):
            blk.step(stream)
            torch.cuda.synchronize()
            got = blk.x_current().cpu().numpy()
            y_ref, S = spmv.csr_spmv(A.row_ptr, A.col, A.vals, prev)
            ok = ok and bool(spmv.within_tolerance(got, y_ref, S, 1e-12)[0].all())
            prev = got
        q.put((rank, ok, getattr(blk, "split", None), ""))
        dist.barrier()
        blk.close()
        dist.destroy_process_group()
    except Exception as e:  # noqa: BLE001
        q.put((rank, False, None, f"{type(e).__name__}: {e}"))


def _run_world2(exchange, fmt, cfg, iters=4):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_dist_worker, args=(r, 2, port, q, exchange, fmt, cfg, iters)) for r in range(2)]
    for p in ps:
        p.start()
    for p in ps:
        p.join(timeout=300)
    return sorted(q.get(timeout=10) for _ in range(2))


@pytest.mark.parametrize("cfg", ["c1", "ragged"])
@pytest.mark.parametrize("fmt", ["ell", "hyb"])
@pytest.mark.parametrize("exchange", ["allgather", "overlap"])
def test_row_block_iteration_world2(dev, exchange, fmt, cfg):
    res = _run_world2(exchange, fmt, cfg)
    assert [r[:2] for r in res] == [(0, True), (1, True)], res
    if exchange == "overlap" and cfg == "c1":
        assert all(r[2] is not None and r[2][1] > r[2][0] for r in res), res  # a real interior


def test_row_block_iteration_world2_p2p(dev):
    """Fused scatter into symmetric-memory replicas (2 ranks on one GPU).
    Skipped if this box cannot map symmetric memory for a gloo group."""
    res = _run_world2("p2p", "ell", "c1")
    errs = [r[3] for r in res if r[3]]
    if errs and any("symm" in e.lower() or "rendezvous" in e.lower() or "not supported" in e.lower()
                    for e in errs):
        pytest.skip(f"symmetric memory unavailable here: {errs[0][:200]}")
    assert [r[:2] for r in res] == [(0, True), (1, True)], res
