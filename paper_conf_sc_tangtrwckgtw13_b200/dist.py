"""Row-block multi-GPU SpMV iteration (one process per GPU).

A (square) is split into contiguous row blocks whose boundaries are multiples
of the slice height (32), balanced by nnz; every rank encodes its block and
keeps a full replica of x.  One iteration, as in a CG loop (BASELINE.json
north_star): x_{k+1} = A.x_k, each rank computing its block of rows and the
blocks being exchanged so that every rank holds all of x_{k+1}.

x lives in a PADDED layout: block p occupies [p*M, p*M + rows_p) with M the
largest block, so that an allgather of equal M-element pieces lands every
block in place; columns are remapped into that layout at encode time
(identity when all blocks are equal, e.g. C5 at P = 1..8).  Two replicas
X[0], X[1] alternate: iteration k reads X[k%2] and writes X[(k+1)%2].

Exchange modes:
  allgather  local SpMV into this rank's block of X[(k+1)%2], then an
             in-place NCCL all_gather_into_tensor (the baseline schedule).
  overlap    the block is split into head / interior / tail row ranges; the
             interior rows touch only this rank's own x block, which it wrote
             itself, so their SpMV runs while the allgather that completes
             x_k is in flight on a second stream; head and tail follow it.
  p2p        fused exchange: X[0], X[1] are symmetric-memory buffers mapped
             into every peer; the ELL kernel's epilogue stores each y value
             into all replicas (bro_spmv_scatter: NVLink P2P stores, or one
             NVLS multimem.st when the group has multicast), so the transfer
             overlaps the SpMV row by row; one cross-GPU barrier per
             iteration orders the next read.
torch.distributed is plumbing only; every SpMV runs in libbro.so.
"""
from __future__ import annotations

import numpy as np

EXCHANGES = ("allgather", "overlap", "p2p")


# ---------------------------------------------------------------- host logic
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


def block_pitch(bounds) -> int:
    """M = the largest block: every block's slot in the padded x layout."""
    return int(np.max(np.diff(np.asarray(bounds, dtype=np.int64))))


def remap_columns(col, bounds) -> np.ndarray:
    """Global column c (row c of block p) -> p*M + (c - b_p), its index in the
    padded x layout.  Identity when all blocks have M rows."""
    bounds = np.asarray(bounds, dtype=np.int64)
    M = block_pitch(bounds)
    col = np.asarray(col)
    if np.all(np.diff(bounds) == M):
        return col.astype(np.int32, copy=False)
    p = np.searchsorted(bounds, col, side="right") - 1
    return (p * M + (col - bounds[p])).astype(np.int32)


def padded_to_global(xg, bounds):
    """Strip per-block padding from a padded x (length P*M) to the global
    vector (length m); works on numpy arrays and torch tensors."""
    bounds = np.asarray(bounds, dtype=np.int64)
    P, M = len(bounds) - 1, block_pitch(bounds)
    if all(bounds[p + 1] - bounds[p] == M for p in range(P)):
        return xg[: int(bounds[-1])]
    parts = [xg[p * M: p * M + int(bounds[p + 1] - bounds[p])] for p in range(P)]
    if isinstance(xg, np.ndarray):
        return np.concatenate(parts)
    import torch
    return torch.cat(parts)


def global_to_padded(x, bounds):
    """Inverse of padded_to_global (padding slots 0); numpy."""
    bounds = np.asarray(bounds, dtype=np.int64)
    P, M = len(bounds) - 1, block_pitch(bounds)
    out = np.zeros(P * M, dtype=np.asarray(x).dtype)
    for p in range(P):
        r0, r1 = int(bounds[p]), int(bounds[p + 1])
        out[p * M: p * M + (r1 - r0)] = x[r0:r1]
    return out


def local_rows_mask(row_ptr, col, lo: int, hi: int) -> np.ndarray:
    """Row i is local if every column of it lies in [lo, hi) (this rank's own
    x block, in the padded layout); empty rows are local."""
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    m = row_ptr.size - 1
    col = np.asarray(col)
    remote = ((col < lo) | (col >= hi)).astype(np.int64)
    c = np.concatenate([[0], np.cumsum(remote)])
    return (c[row_ptr[1:]] - c[row_ptr[:-1]]) == 0 if m else np.zeros(0, bool)


def interior_split(local_mask, align: int = 32, min_frac: float = 0.25):
    """(a, b): the longest run of local rows, shrunk to `align`-multiples
    (b may also be the block end).  Rows [a, b) depend only on this rank's own
    x block; [0, a) and [b, m) need remote blocks.  (0, 0) when the run is
    shorter than min_frac of the block (no overlap worth a split)."""
    mk = np.asarray(local_mask, dtype=bool)
    m = mk.size
    if m == 0:
        return 0, 0
    d = np.diff(np.concatenate([[0], mk.astype(np.int8), [0]]))
    starts, ends = np.flatnonzero(d == 1), np.flatnonzero(d == -1)
    if starts.size == 0:
        return 0, 0
    k = int(np.argmax(ends - starts))
    a, b = int(starts[k]), int(ends[k])
    a = -(-a // align) * align
    if b != m:
        b = b // align * align
    if b - a < max(1, int(min_frac * m)):
        return 0, 0
    return a, b


class _Rows:
    """Rows [r0, r1) of a CSR matrix, columns remapped to the padded layout."""

    def __init__(self, row_ptr, col, vals, r0, r1, n):
        a, b = int(row_ptr[r0]), int(row_ptr[r1])
        self.m, self.n = r1 - r0, n
        self.row_ptr = np.asarray(row_ptr[r0:r1 + 1], dtype=np.int64) - a
        self.col = col[a:b]
        self.vals = vals[a:b]
        self.nnz = b - a


# ---------------------------------------------------------------- GPU iteration
def allgather_blocks(y_pad, out, group=None):
    """out[p*M:(p+1)*M] = y_pad of rank p (NCCL all_gather_into_tensor, in
    place when y_pad is out's own slice; gloo falls back to a list allgather)."""
    import torch
    import torch.distributed as dist
    try:
        dist.all_gather_into_tensor(out, y_pad, group=group)
    except (RuntimeError, NotImplementedError, AttributeError, ValueError):
        parts = list(torch.chunk(out, dist.get_world_size(group)))
        src = y_pad.clone()
        dist.all_gather(parts, src, group=group)
    return out


class RowBlockSpmv:
    """This rank's block of A as libbro handle(s) plus the iteration buffers."""

    def __init__(self, A, rank: int, world: int, device, fmt="ell", codec=1, dtype=None,
                 bounds=None, vec_words=0, exchange="allgather", group=None, **layout):
        import torch
        from .bro import BroMatrix
        if exchange not in EXCHANGES:
            raise ValueError(f"exchange must be one of {EXCHANGES}")
        if A.m != A.n:
            raise ValueError("the row-block iteration needs a square matrix (x_{k+1} = A.x_k)")
        self.rank, self.world, self.group, self.exchange = rank, world, group, exchange
        self.device = device
        self.bounds = np.asarray(bounds if bounds is not None else choose_partition(A.row_ptr, world))
        r0, r1 = int(self.bounds[rank]), int(self.bounds[rank + 1])
        self.rows = (r0, r1)
        self.M = M = block_pitch(self.bounds)
        self.off = rank * M
        a, b = int(A.row_ptr[r0]), int(A.row_ptr[r1])
        col = remap_columns(A.col[a:b], self.bounds)
        rp = np.asarray(A.row_ptr[r0:r1 + 1], dtype=np.int64) - a
        vals = A.vals[a:b]
        n_pad = world * M
        self.nnz_local = b - a
        dev_index = device.index or 0
        # layout: BroMatrix options (slice_h, coo_T, ell_kernel, ...)
        mk = dict(fmt=fmt, codec=codec, device=dev_index, dtype=dtype, vec_words=vec_words, **layout)
        # the whole block (kernel-only timing, allgather / p2p modes)
        self.mat = BroMatrix(_Rows(rp, col, vals, 0, r1 - r0, n_pad), **mk)
        self.tdt = torch.float64 if self.mat.dtype == np.float64 else torch.float32
        self.isz = np.dtype(self.mat.dtype).itemsize
        self.mloc = r1 - r0
        # overlap mode: head / interior / tail handles
        self.parts = []
        if exchange == "overlap":
            ia, ib = interior_split(local_rows_mask(rp, col, self.off, self.off + self.mloc))
            self.split = (ia, ib)
            for lo, hi, kind in ((ia, ib, "interior"), (0, ia, "head"), (ib, self.mloc, "tail")):
                if hi > lo:
                    self.parts.append((kind, lo, BroMatrix(_Rows(rp, col, vals, lo, hi, n_pad), **mk)))
            if ia == ib:  # nothing local enough: one handle after the exchange
                self.parts = [("tail", 0, self.mat)]
        # the two x replicas
        self.X = None
        self.hdl = None
        self.mc = [0, 0]
        if exchange == "p2p" and world > 1:
            import torch.distributed._symmetric_memory as symm
            self.X = [symm.empty(n_pad, dtype=self.tdt, device=device) for _ in range(2)]
            for Xi in self.X:
                Xi.zero_()
            gname = group.group_name if group is not None else torch.distributed.group.WORLD.group_name
            self.hdl = [symm.rendezvous(Xi, gname) for Xi in self.X]
            self.dst = []
            for i, (Xi, h) in enumerate(zip(self.X, self.hdl)):
                base = Xi.data_ptr() - int(h.buffer_ptrs[rank])  # tensor offset in the symmetric allocation
                ptrs = [int(h.buffer_ptrs[rank]) + base + self.off * self.isz]
                ptrs += [int(h.buffer_ptrs[p]) + base + self.off * self.isz for p in range(world) if p != rank]
                self.dst.append(ptrs)
                mcp = 0
                try:
                    mcp = int(h.multicast_ptr or 0)
                except (AttributeError, RuntimeError, TypeError):
                    pass
                if mcp:
                    self.mc[i] = mcp + base + self.off * self.isz
        else:
            self.X = [torch.zeros(n_pad, dtype=self.tdt, device=device) for _ in range(2)]
        self.k = 0
        self.gathered = 0  # X[0] starts complete (set_x)
        self.comm = torch.cuda.Stream(device) if exchange == "overlap" else None
        self.ev_y = torch.cuda.Event() if exchange == "overlap" else None
        self.ev_ag = torch.cuda.Event() if exchange == "overlap" else None
        # NVLS multicast stores only on request (BRO_MULTICAST=1): not yet
        # exercised on a multi-GPU box
        import os
        self.use_mc = os.environ.get("BRO_MULTICAST", "0") == "1"

    # -- state
    def set_x(self, x_global):
        """x_0 (global, length m, numpy) into X[0] (padded layout); k = 0."""
        import torch
        xp = global_to_padded(np.asarray(x_global, dtype=self.mat.dtype), self.bounds)
        self.X[0].copy_(torch.from_numpy(xp))
        self.X[1].zero_()
        self.k = 0
        self.gathered = 0
        if self.hdl is not None:
            torch.cuda.synchronize(self.device)
            self.hdl[0].barrier(channel=0)
            torch.cuda.synchronize(self.device)

    def complete(self, stream=None):
        """Make X[k%2] hold all of x_k.  The overlap schedule defers the
        allgather of x_k to the start of iteration k (where it overlaps the
        interior rows), so after step() only this rank's block of x_k is
        final until complete() (or the next step) gathers the rest."""
        import torch
        if self.exchange != "overlap" or self.world == 1 or self.gathered == self.k:
            return
        stream = stream or torch.cuda.current_stream(self.device)
        xin = self.X[self.k % 2]
        with torch.cuda.stream(stream):
            allgather_blocks(xin[self.off: self.off + self.M], xin, self.group)
        self.gathered = self.k

    def x_current(self, stream=None):
        """x_k as the global vector (a torch view/copy on the device)."""
        self.complete(stream)
        return padded_to_global(self.X[self.k % 2], self.bounds)

    def y_block(self, which=None):
        k = self.k if which is None else which
        return self.X[k % 2][self.off: self.off + self.mloc]

    # -- kernels
    def spmv(self, x=None, stream=None, y=None):
        """Local SpMV only (no exchange): y = A_p.x (kernel-only timing)."""
        x = self.X[self.k % 2] if x is None else x
        y = self.X[(self.k + 1) % 2][self.off: self.off + self.mloc] if y is None else y
        return self.mat.spmv(x, y, stream=stream)

    def step(self, stream=None, exchange=None):
        """One iteration x_{k+1} = A.x_k with this rank's exchange mode (or
        `exchange="allgather"`, which any instance can run); returns the
        padded X holding x_{k+1} (complete once `stream` and, for p2p, the
        barrier have run)."""
        import torch
        stream = stream or torch.cuda.current_stream(self.device)
        exchange = exchange or self.exchange
        if exchange != "allgather" and exchange != self.exchange:
            raise ValueError(f"this instance was built for {self.exchange!r}")
        xin, xout = self.X[self.k % 2], self.X[(self.k + 1) % 2]
        yout = xout[self.off: self.off + self.mloc]
        if self.world == 1:
            self.mat.spmv(xin, yout, stream=stream)
        elif exchange == "allgather":
            self.mat.spmv(xin, yout, stream=stream)
            with torch.cuda.stream(stream):
                allgather_blocks(xout[self.off: self.off + self.M], xout, self.group)
        elif exchange == "overlap":
            self._step_overlap(xin, xout, stream)
        else:
            mc = self.mc[(self.k + 1) % 2] if self.use_mc else 0
            self.mat.spmv_scatter(xin, self.dst[(self.k + 1) % 2], mc, stream=stream)
            with torch.cuda.stream(stream):
                self.hdl[(self.k + 1) % 2].barrier(channel=0)
        self.k += 1
        if exchange != "overlap":
            self.gathered = self.k
        return xout

    def _step_overlap(self, xin, xout, stream):
        import torch
        # the allgather completing x_k (this rank's block of xin was written by
        # the previous iteration on `stream`) runs on the comm stream ...
        if self.gathered != self.k:
            self.ev_y.record(stream)
            self.comm.wait_event(self.ev_y)
            with torch.cuda.stream(self.comm):
                allgather_blocks(xin[self.off: self.off + self.M], xin, self.group)
        self.ev_ag.record(self.comm)
        # ... while the interior rows (own x block only) run on `stream`
        waited = False
        for kind, lo, mat in self.parts:
            if kind != "interior" and not waited:
                stream.wait_event(self.ev_ag)
                waited = True
            y = xout[self.off + lo: self.off + lo + mat.m]
            mat.spmv(xin, y, stream=stream)
        if not waited:
            stream.wait_event(self.ev_ag)

    def close(self):
        for _, _, mat in self.parts:
            if mat is not self.mat:
                mat.close()
        self.mat.close()
