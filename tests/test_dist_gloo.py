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
        g = dist_mod.padded_to_global(out, b).numpy()
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


# ------------------------------------------------------------ exchange host logic
def test_padded_layout_round_trip_and_remap():
    """Padded x layout (block p at [p*M, p*M + rows_p)): global <-> padded is
    a bijection on the rows and remapped columns address the same x values."""
    A = random_csr(1000, 1000, 3, max_len=20, empty_frac=0.05, long_frac=0.0, long_len=0)
    b = dist_mod.partition_rows(A.row_ptr, 3)
    M = dist_mod.block_pitch(b)
    x = np.random.default_rng(2).uniform(-1, 1, A.n)
    xp = dist_mod.global_to_padded(x, b)
    assert xp.size == 3 * M
    assert np.array_equal(dist_mod.padded_to_global(xp, b), x)
    cp = dist_mod.remap_columns(A.col, b)
    assert np.array_equal(xp[cp], x[A.col])  # same operand for every entry
    assert cp.max() < 3 * M
    # equal blocks: identity
    be = dist_mod.equal_row_partition(4096, 4)
    assert np.array_equal(dist_mod.remap_columns(np.arange(4096), be), np.arange(4096))


def test_interior_split_stencil_planes():
    """27-point stencil on g^3 split in P equal row blocks (whole planes):
    only the first and last plane of a block touch remote x blocks, so the
    interior is the block minus one plane at each end (rounded to 32)."""
    from gen.matrices import stencil_27pt
    g, P = 16, 4
    A = stencil_27pt(g)
    b = dist_mod.equal_row_partition(A.m, P, align=32)
    plane = g * g
    for p in range(P):
        r0, r1 = int(b[p]), int(b[p + 1])
        B = row_block(A, r0, r1)
        mk = dist_mod.local_rows_mask(B.row_ptr, B.col, r0, r1)
        a, e = dist_mod.interior_split(mk)
        lo = 0 if p == 0 else plane
        hi = (r1 - r0) if p == P - 1 else (r1 - r0) - plane
        assert a == -(-lo // 32) * 32
        assert e == (hi if hi == r1 - r0 else hi // 32 * 32)
        # the defining property: interior rows need only the own block of x
        x = np.random.default_rng(p).uniform(-1, 1, A.n)
        xo = np.zeros_like(x)
        xo[r0:r1] = x[r0:r1]
        y_full, _ = spmv.csr_spmv(B.row_ptr, B.col, B.vals, x)
        y_own, _ = spmv.csr_spmv(B.row_ptr, B.col, B.vals, xo)
        assert np.array_equal(np.asarray(y_full)[a:e], np.asarray(y_own)[a:e])
        assert not np.array_equal(np.asarray(y_full), np.asarray(y_own)) or P == 1


def test_interior_split_degenerate():
    assert dist_mod.interior_split(np.zeros(0, bool)) == (0, 0)
    assert dist_mod.interior_split(np.zeros(100, bool)) == (0, 0)
    assert dist_mod.interior_split(np.ones(100, bool)) == (0, 100)
    mk = np.ones(1000, bool)
    mk[::10] = False  # no long run: not worth a split
    assert dist_mod.interior_split(mk) == (0, 0)


def _iter_worker(rank, world, port, q, iters):
    """x_{k+1} = A.x_k over row blocks with the padded layout and an in-place
    allgather (gloo); the oracle's local products stand in for the kernel."""
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        A = random_csr(900, 900, 8, max_len=12, empty_frac=0.1, long_frac=0.0, long_len=0)
        b = dist_mod.partition_rows(A.row_ptr, world)
        M = dist_mod.block_pitch(b)
        r0, r1 = int(b[rank]), int(b[rank + 1])
        a0, a1 = int(A.row_ptr[r0]), int(A.row_ptr[r1])
        cp = dist_mod.remap_columns(A.col[a0:a1], b)
        rp = A.row_ptr[r0:r1 + 1] - a0
        x0 = np.random.default_rng(4).uniform(-1, 1, A.n) * 0.1
        X = [torch.from_numpy(dist_mod.global_to_padded(x0, b)), torch.zeros(world * M, dtype=torch.float64)]
        for k in range(iters):
            xin, xout = X[k % 2], X[(k + 1) % 2]
            y, _ = spmv.csr_spmv(rp, cp, A.vals[a0:a1], xin.numpy())
            xout[rank * M: rank * M + (r1 - r0)] = torch.from_numpy(np.asarray(y, dtype=np.float64))
            dist_mod.allgather_blocks(xout[rank * M: (rank + 1) * M], xout)
        got = dist_mod.padded_to_global(X[iters % 2], b).numpy()
        ref = x0.copy()
        for _ in range(iters):
            ref = np.asarray(spmv.csr_spmv(A.row_ptr, A.col, A.vals, ref)[0], dtype=np.float64)
        q.put((rank, bool(np.allclose(got, ref, rtol=1e-12, atol=1e-300))))
    finally:
        dist.destroy_process_group()


def test_padded_iteration_world2_gloo():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_iter_worker, args=(r, 2, port, q, 3)) for r in range(2)]
    for p in ps:
        p.start()
    for p in ps:
        p.join(timeout=180)
    res = sorted(q.get(timeout=10) for _ in range(2))
    assert res == [(0, True), (1, True)]
