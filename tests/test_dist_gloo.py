"""Host-side logic of the row-block multi-GPU iteration, on CPU (-m "not gpu"):
partitioning, and the allgather of y blocks with world_size 2 over gloo
(local products from the oracle stand in for the GPU kernel here)."""
import os
import socket

import numpy as np
import pytest

from gen import make_config, random_csr, row_block
from oracle import spmv

import paper_conf_sc_tangtrwckgtw13_b200.dist as dist_mod


def test_partition_rows_properties():
    A = random_csr(5000, 5000, 0, max_len=60, empty_frac=0.1, long_frac=0.01, long_len=900)
    for P in (1, 2, 3, 4, 8):
        b = dist_mod.partition_rows(A.row_ptr, P)
        assert b[0] == 0 and b[-1] == A.m and np.all(np.diff(b) >= 0)
        assert np.all(b[1:-1] % 32 == 0)
        nnz = np.diff(A.row_ptr[b])
        assert nnz.max() <= A.nnz / P + 32 * 900 + 1  # within one slice of long rows of the target


def test_choose_partition_c5_is_equal_blocks():
    A = make_config(1)  # 4096 rows: equal blocks for P | 128
    for P in (1, 2, 4, 8):
        b = dist_mod.choose_partition(A.row_ptr, P)
        assert np.all(np.diff(b) == A.m // P)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A = random_csr(1000, 1000, 5, max_len=30, empty_frac=0.1, long_frac=0.02, long_len=400)
        x = np.random.default_rng(1).uniform(-1, 1, A.n)
        b = dist_mod.partition_rows(A.row_ptr, world)
        M = int(np.max(np.diff(b)))
        B = row_block(A, int(b[rank]), int(b[rank + 1]))
        y_loc, _ = spmv.csr_spmv(B.row_ptr, B.col, B.vals, x)
        y_pad = torch.zeros(M, dtype=torch.float64)
        y_pad[: B.m] = torch.from_numpy(np.array(y_loc, dtype=np.float64))
        out = torch.zeros(M * world, dtype=torch.float64)
        dist_mod.allgather_blocks(y_pad, out)
        g = dist_mod.gathered_to_global(out, b, M).numpy()
        y_ref, S = spmv.csr_spmv(A.row_ptr, A.col, A.vals, x)
        ok, _ = spmv.within_tolerance(g, y_ref, S, 1e-15)
        q.put((rank, bool(ok.all()), g.size == A.m))
    finally:
        dist.destroy_process_group()


def test_allgather_world2_gloo():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    for p in ps:
        p.join(timeout=180)
    res = sorted(q.get(timeout=10) for _ in range(2))
    assert res == [(0, True, True), (1, True, True)]
