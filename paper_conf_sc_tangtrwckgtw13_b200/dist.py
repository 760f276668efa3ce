"""Row-block multi-GPU SpMV iteration (one process per GPU).

A is split into contiguous row blocks whose boundaries are multiples of the
slice height (32), balanced by nnz; every rank encodes its block with GLOBAL
column indices and keeps a full replica of x.  One iteration, as in a CG
loop (BASELINE.json north_star): local bro_spmv, then one allgather of the
y blocks over NCCL (NVLink 5 / NVSwitch) into the replicated vector.
torch.distributed is plumbing only; the SpMV runs in libbro.so.
"""
from __future__ import annotations

import numpy as np


def partition_rows(row_ptr, P: int, align: int = 32) -> np.ndarray:
    """Boundaries b_0 = 0 < ... < b_P = m, each b_p a multiple of `align`
    (except b_P = m), chosen so that nnz of each block is ~ nnz/P."""
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    m = row_ptr.size - 1
    nnz = int(row_ptr[-1])
    cand = np.arange(0, m + 1, align, dtype=np.int64)
    b = np.zeros(P + 1, dtype=np.int64)
    for p in range(1, P):
        target = nnz * p // P
        k = int(np.searchsorted(row_ptr[cand], target, side="left"))
        k = min(max(k, 0), cand.size - 1)
        b[p] = max(int(cand[k]), int(b[p - 1]))
    b[P] = m
    for p in range(P - 1, 0, -1):
        b[p] = min(b[p], b[p + 1])
    return b


def equal_row_partition(m: int, P: int, align: int = 32):
    """Equal row blocks when m is a multiple of align*P (C5 at P = 1..8), else None."""
    if m % (align * P):
        return None
    return np.arange(P + 1, dtype=np.int64) * (m // P)


def choose_partition(row_ptr, P: int, align: int = 32, max_imbalance: float = 0.02) -> np.ndarray:
    """Equal blocks (gather output == x layout, no padding) if their nnz
    imbalance is below max_imbalance, else nnz-balanced blocks."""
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    m = row_ptr.size - 1
    eq = equal_row_partition(m, P, align)
    if eq is not None:
        nnzs = np.diff(row_ptr[eq])
        if nnzs.max() <= (1 + max_imbalance) * max(row_ptr[-1] / P, 1):
            return eq
    return partition_rows(row_ptr, P, align)


def allgather_blocks(y_pad, out, group=None):
    """out[p*M:(p+1)*M] = y_pad of rank p (NCCL all_gather_into_tensor; gloo
    falls back to a list allgather)."""
    import torch
    import torch.distributed as dist
    try:
        dist.all_gather_into_tensor(out, y_pad, group=group)
    except (RuntimeError, NotImplementedError, AttributeError):
        parts = list(torch.chunk(out, dist.get_world_size(group)))
        dist.all_gather(parts, y_pad, group=group)
        if parts[0].data_ptr() != out.data_ptr():
            torch.cat(parts, out=out)
    return out


def gathered_to_global(xg, bounds, M):
    """Strip per-block padding from an allgathered buffer (length P*M) to the
    global vector (length m)."""
    import torch
    P = len(bounds) - 1
    if all(bounds[p + 1] - bounds[p] == M for p in range(P)):
        return xg[: bounds[-1]]
    return torch.cat([xg[p * M: p * M + (bounds[p + 1] - bounds[p])] for p in range(P)])


class _RowBlock:
    """Rows [r0, r1) of a CSR matrix, columns kept global."""

    def __init__(self, A, r0, r1):
        a, b = int(A.row_ptr[r0]), int(A.row_ptr[r1])
        self.m, self.n = r1 - r0, A.n
        self.row_ptr = np.asarray(A.row_ptr[r0:r1 + 1], dtype=np.int64) - a
        self.col = A.col[a:b]
        self.vals = A.vals[a:b]
        self.nnz = b - a


class RowBlockSpmv:
    """This rank's block of A as a libbro handle plus the iteration buffers."""

    def __init__(self, A, rank: int, world: int, device, fmt="ell", codec=1, dtype=None,
                 bounds=None, vec_words=0):
        import torch
        from .bro import BroMatrix
        self.bounds = np.asarray(bounds if bounds is not None else choose_partition(A.row_ptr, world))
        r0, r1 = int(self.bounds[rank]), int(self.bounds[rank + 1])
        self.rows = (r0, r1)
        self.M = int(np.max(np.diff(self.bounds)))
        B = _RowBlock(A, r0, r1)
        self.nnz_local = B.nnz
        self.mat = BroMatrix(B, fmt=fmt, codec=codec, device=device.index or 0, dtype=dtype,
                             vec_words=vec_words)
        tdt = torch.float64 if self.mat.dtype == np.float64 else torch.float32
        self.y_pad = torch.zeros(self.M, dtype=tdt, device=device)
        self.xg = torch.zeros(self.M * world, dtype=tdt, device=device)
        self.y_local = self.y_pad[: r1 - r0]

    def spmv(self, x, stream=None):
        return self.mat.spmv(x, self.y_local, stream=stream)

    def step(self, x, stream=None, group=None):
        """Local SpMV then the allgather of y blocks (one CG-style iteration)."""
        self.spmv(x, stream)
        allgather_blocks(self.y_pad, self.xg, group)
        return self.xg
