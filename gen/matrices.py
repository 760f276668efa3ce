"""Seeded CSR generators for the five BASELINE.json configs (+ small fuzz cases).

Recipes (restated in DESIGN.md "Input recipe"):

C1  2D 5-point Laplacian, 64x64 grid, natural ordering, 4 on the diagonal,
    -1 off it.  m = 4096, nnz = 20224.
C2  FEM-like banded: 17x17x72 node grid, 27-point node neighbourhood, each
    undirected off-diagonal node edge kept with q = 0.86, 3x3 dense DOF
    blocks, vals U[-1,1).  m = 62424, nnz ~ 4.0M (cant-shaped).
C3  webbase-like power law: lengths 5% 1 / 65% 2 / 30% 3, 1.5% of rows
    overridden by floor(10*u^(-1/1.1)) clipped to [10, 4700]; columns w.p. 0.7
    local (i + Laplace(256)), else 50/50 Zipf(1.8)-popular (through a fixed
    permutation) or uniform; no repeats within a row.  m = 1,000,005
    (webbase-1M shape).
C4  random-block: 62,500 families of 32 rows; per family 1+Poisson(2) blocks
    of width U{2..10} at random starts; each row copies the family's blocks
    with start jitter U{-2..2} and w.p. 0.10 one extra block of width
    U{8..32}; rows scrambled by a seeded permutation.  m = 2,000,000,
    nnz ~ 40M.  (BAR-aware reordering is applied by the caller, not here.)
C5  3D 27-point stencil on a 200^3 grid, 26 on the diagonal, -1 off it.
    m = 8,000,000, nnz = 598^3 = 213,847,192.

x ~ U[-1, 1) for every config.  All generators are deterministic in `seed`.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np


@dataclass
class Csr:
    """Canonical CSR: row_ptr int64[m+1], col int32[nnz] (strictly increasing
    within each row), vals float64/float32[nnz]."""

    m: int
    n: int
    row_ptr: np.ndarray
    col: np.ndarray
    vals: np.ndarray
    name: str = ""

    @property
    def nnz(self) -> int:
        return int(self.row_ptr[-1])

    def row_lengths(self) -> np.ndarray:
        return np.diff(self.row_ptr)

    def astype(self, dtype) -> "Csr":
        return Csr(self.m, self.n, self.row_ptr, self.col,
                   self.vals.astype(dtype), self.name)


CONFIGS = {
    1: "2D 5-point Laplacian on a 64x64 grid (4,096 rows, ~20K nnz, fp64), BRO-ELL, 1 GPU",
    2: "FEM-like banded matrix, 62K rows, ~4M nnz (cant/pwtk-shaped), BRO-ELL vs ELL, fp64",
    3: "power-law web/circuit-like matrix, 1M rows, ~3M nnz (webbase-shaped), BRO-HYB vs HYB",
    4: "BRO-aware clustering-reordered random-block matrix, 2M rows, ~40M nnz, BRO-HYB fp32 and fp64",
    5: "3D 27-point stencil on a 200^3 grid (8M rows, ~216M nnz), BRO-ELL row-partitioned at 1/2/4/8 B200 with x allgather",
}


# --------------------------------------------------------------------------
# helpers (pure data movement)
# --------------------------------------------------------------------------

def _csr_from_pairs(m: int, n: int, rows: np.ndarray, cols: np.ndarray,
                    vals: np.ndarray, name: str, assume_unique: bool = False) -> Csr:
    """Sort (row, col) pairs into canonical CSR; duplicates are dropped
    (first occurrence kept) unless `assume_unique`."""
    rows = np.asarray(rows, dtype=np.int64)
    cols = np.asarray(cols, dtype=np.int64)
    key = rows * np.int64(n) + cols
    order = np.argsort(key, kind="stable")
    key = key[order]
    if not assume_unique and key.size:
        keep = np.ones(key.size, dtype=bool)
        keep[1:] = key[1:] != key[:-1]
        order = order[keep]
        key = key[keep]
    r = (key // n).astype(np.int64)
    c = (key % n).astype(np.int32)
    v = np.asarray(vals)[order]
    counts = np.bincount(r, minlength=m)
    row_ptr = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    return Csr(m, n, row_ptr, c, v, name)


def _stencil(dims, offsets, diag, off, name) -> Csr:
    """Natural-ordering stencil matrix; `offsets` are sorted so that the
    resulting columns increase within each row."""
    dims = tuple(int(d) for d in dims)
    m = int(np.prod(dims))
    strides = np.ones(len(dims), dtype=np.int64)
    for a in range(len(dims) - 2, -1, -1):
        strides[a] = strides[a + 1] * dims[a + 1]
    coords = np.indices(dims, dtype=np.int32).reshape(len(dims), -1)
    k = len(offsets)
    col2d = np.empty((m, k), dtype=np.int32)
    valid = np.ones((m, k), dtype=bool)
    rowid = np.arange(m, dtype=np.int64)
    for j, off_ in enumerate(offsets):
        ok = np.ones(m, dtype=bool)
        for a, d in enumerate(off_):
            c = coords[a] + d
            ok &= (c >= 0) & (c < dims[a])
        valid[:, j] = ok
        delta = int(sum(int(d) * int(s) for d, s in zip(off_, strides)))
        col2d[:, j] = (rowid + delta).astype(np.int32)
    lens = valid.sum(axis=1)
    row_ptr = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(lens, out=row_ptr[1:])
    col = col2d[valid]
    del col2d
    center = tuple(0 for _ in dims)
    is_diag = np.zeros((m, k), dtype=bool)
    is_diag[:, offsets.index(center)] = True
    vals = np.where(is_diag[valid], float(diag), float(off))
    return Csr(m, m, row_ptr, col, vals.astype(np.float64), name)


# --------------------------------------------------------------------------
# the five configs
# --------------------------------------------------------------------------

def laplacian_2d(g: int = 64) -> Csr:
    """C1: 2D 5-point Laplacian, natural ordering (4 diag, -1 off)."""
    offs = [(-1, 0), (0, -1), (0, 0), (0, 1), (1, 0)]
    return _stencil((g, g), offs, 4.0, -1.0, f"laplace2d_{g}x{g}")


def stencil_27pt(g: int = 200) -> Csr:
    """C5: 3D 27-point stencil on a g^3 grid (26 diag, -1 off)."""
    offs = [(a, b, c) for a in (-1, 0, 1) for b in (-1, 0, 1) for c in (-1, 0, 1)]
    return _stencil((g, g, g), offs, 26.0, -1.0, f"stencil27_{g}^3")


def fem_banded(seed: int = 2, dims=(17, 17, 72), q: float = 0.86, dof: int = 3) -> Csr:
    """C2: FEM-like matrix, 3x3 DOF blocks over a thinned 27-point node graph."""
    rng = np.random.default_rng(seed)
    ni, nj, nk = dims
    nodes = ni * nj * nk
    coords = np.indices(dims).reshape(3, -1)
    fwd = [(a, b, c) for a in (-1, 0, 1) for b in (-1, 0, 1) for c in (-1, 0, 1)
           if (a, b, c) > (0, 0, 0)]
    eu, ev = [], []
    uid = np.arange(nodes, dtype=np.int64)
    for (a, b, c) in fwd:
        i2, j2, k2 = coords[0] + a, coords[1] + b, coords[2] + c
        ok = (i2 >= 0) & (i2 < ni) & (j2 >= 0) & (j2 < nj) & (k2 >= 0) & (k2 < nk)
        keep = ok & (rng.random(nodes) < q)
        u = uid[keep]
        v = (i2[keep] * nj + j2[keep]) * nk + k2[keep]
        eu.append(u)
        ev.append(v)
    eu = np.concatenate(eu)
    ev = np.concatenate(ev)
    nu = np.concatenate([eu, ev, uid])  # both directions + self
    nv = np.concatenate([ev, eu, uid])
    a = np.repeat(np.arange(dof), dof)
    b = np.tile(np.arange(dof), dof)
    rows = (nu[:, None] * dof + a[None, :]).ravel()
    cols = (nv[:, None] * dof + b[None, :]).ravel()
    m = nodes * dof
    vals = rng.uniform(-1.0, 1.0, rows.size)
    return _csr_from_pairs(m, m, rows, cols, vals, "fem_banded", assume_unique=True)


def _distinct_columns(rng, rows_of_entry, draw, n, max_rounds=64):
    """Draw one column per entry with `draw(k)`, re-drawing entries whose
    (row, col) repeats an earlier entry of the same row (sampling without
    replacement per row)."""
    cols = draw(np.arange(rows_of_entry.size))
    todo = np.arange(rows_of_entry.size)
    for _ in range(max_rounds):
        key = rows_of_entry * np.int64(n) + cols
        order = np.argsort(key, kind="stable")
        ks = key[order]
        dup = np.zeros(ks.size, dtype=bool)
        dup[1:] = ks[1:] == ks[:-1]
        todo = order[dup]
        if todo.size == 0:
            return cols
        cols[todo] = draw(todo)
    # last resort: uniform re-draws until unique
    while todo.size:
        cols[todo] = rng.integers(0, n, todo.size)
        key = rows_of_entry * np.int64(n) + cols
        order = np.argsort(key, kind="stable")
        ks = key[order]
        dup = np.zeros(ks.size, dtype=bool)
        dup[1:] = ks[1:] == ks[:-1]
        todo = order[dup]
    return cols


def webbase_like(seed: int = 3, m: int = 1_000_005) -> Csr:
    """C3: power-law row lengths, mostly-local columns with popular hubs."""
    rng = np.random.default_rng(seed)
    n = m
    lens = rng.choice(np.array([1, 2, 3]), size=m, p=[0.05, 0.65, 0.30]).astype(np.int64)
    over = rng.random(m) < 0.015
    u = 1.0 - rng.random(int(over.sum()))  # (0, 1]
    lens[over] = np.clip(np.floor(10.0 * u ** (-1.0 / 1.1)), 10, 4700).astype(np.int64)
    row_ptr = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(lens, out=row_ptr[1:])
    nnz = int(row_ptr[-1])
    rows = np.repeat(np.arange(m, dtype=np.int64), lens)
    hub_perm = rng.permutation(n).astype(np.int64)

    def draw(idx):
        k = idx.size
        r = rows[idx]
        kind = rng.random(k)
        out = np.empty(k, dtype=np.int64)
        loc = kind < 0.7
        off = np.rint(rng.laplace(0.0, 256.0, int(loc.sum()))).astype(np.int64)
        out[loc] = np.clip(r[loc] + off, 0, n - 1)
        pop = (kind >= 0.7) & (kind < 0.85)
        z = rng.zipf(1.8, int(pop.sum())).astype(np.int64)
        out[pop] = hub_perm[(z - 1) % n]
        uni = kind >= 0.85
        out[uni] = rng.integers(0, n, int(uni.sum()))
        return out

    cols = _distinct_columns(rng, rows, draw, n)
    vals = rng.uniform(-1.0, 1.0, nnz)
    return _csr_from_pairs(m, n, rows, cols, vals, "webbase_like", assume_unique=True)


def random_block(seed: int = 4, families: int = 62_500, fam_rows: int = 32,
                 scramble: bool = True) -> Csr:
    """C4: rows in families sharing jittered column blocks; rows scrambled."""
    rng = np.random.default_rng(seed)
    m = families * fam_rows
    n = m
    nb = 1 + rng.poisson(2.0, families)
    fam_of_block = np.repeat(np.arange(families, dtype=np.int64), nb)
    width = rng.integers(2, 11, fam_of_block.size).astype(np.int64)
    start = (rng.random(fam_of_block.size) * (n - width + 1)).astype(np.int64)
    # every row of a family copies each family block with start jitter
    rb_row = (fam_of_block[:, None] * fam_rows + np.arange(fam_rows)[None, :]).ravel()
    rb_w = np.repeat(width, fam_rows)
    rb_s = np.repeat(start, fam_rows) + rng.integers(-2, 3, rb_row.size)
    rb_s = np.clip(rb_s, 0, n - rb_w)
    extra = rng.random(m) < 0.10
    ex_row = np.nonzero(extra)[0].astype(np.int64)
    ex_w = rng.integers(8, 33, ex_row.size).astype(np.int64)
    ex_s = (rng.random(ex_row.size) * (n - ex_w + 1)).astype(np.int64)
    b_row = np.concatenate([rb_row, ex_row])
    b_w = np.concatenate([rb_w, ex_w])
    b_s = np.concatenate([rb_s, ex_s])
    tot = int(b_w.sum())
    rows = np.repeat(b_row, b_w)
    first = np.zeros(b_w.size, dtype=np.int64)
    np.cumsum(b_w[:-1], out=first[1:])
    within = np.arange(tot, dtype=np.int64) - np.repeat(first, b_w)
    cols = np.repeat(b_s, b_w) + within
    if scramble:
        perm = rng.permutation(m).astype(np.int64)  # new row i <- old row perm[i]
        inv = np.empty(m, dtype=np.int64)
        inv[perm] = np.arange(m, dtype=np.int64)
        rows = inv[rows]
    vals = rng.uniform(-1.0, 1.0, tot)
    return _csr_from_pairs(m, n, rows, cols, vals, "random_block")


def random_csr(m: int, n: int, seed: int, max_len: int = 40, empty_frac: float = 0.1,
               long_frac: float = 0.0, long_len: int = 200, wide_cols: bool = False) -> Csr:
    """Small fuzz matrix: random row lengths (some empty, some long), distinct
    columns per row.  `wide_cols` spreads columns over [0, n) uniformly so
    deltas need many bits; otherwise columns cluster near the diagonal."""
    rng = np.random.default_rng(seed)
    lens = rng.integers(0, max_len + 1, m)
    lens[rng.random(m) < empty_frac] = 0
    if long_frac > 0:
        lens[rng.random(m) < long_frac] = long_len
    lens = np.minimum(lens, n)
    rows, cols = [], []
    for i in range(m):
        k = int(lens[i])
        if k == 0:
            continue
        if wide_cols or n <= 4 * k:
            c = rng.choice(n, size=k, replace=False)
        else:
            lo = max(0, min(n - 4 * k, i * n // max(m, 1) - 2 * k))
            c = lo + rng.choice(4 * k, size=k, replace=False)
        rows.append(np.full(k, i, dtype=np.int64))
        cols.append(np.sort(c).astype(np.int64))
    if rows:
        r = np.concatenate(rows)
        c = np.concatenate(cols)
    else:
        r = np.zeros(0, dtype=np.int64)
        c = np.zeros(0, dtype=np.int64)
    vals = rng.uniform(-1.0, 1.0, r.size)
    return _csr_from_pairs(m, n, r, c, vals, f"random_{m}x{n}_s{seed}", assume_unique=True)


def permute_rows(A: Csr, perm: np.ndarray) -> Csr:
    """A' = P.A with row i of A' = row perm[i] of A."""
    perm = np.asarray(perm, dtype=np.int64)
    lens = np.diff(A.row_ptr)[perm]
    row_ptr = np.zeros(A.m + 1, dtype=np.int64)
    np.cumsum(lens, out=row_ptr[1:])
    starts = A.row_ptr[:-1][perm]
    idx = np.repeat(starts - row_ptr[:-1], lens) + np.arange(int(row_ptr[-1]), dtype=np.int64)
    return Csr(A.m, A.n, row_ptr, A.col[idx], A.vals[idx], A.name + "_perm")


def row_block(A: Csr, r0: int, r1: int) -> Csr:
    """Rows [r0, r1) of A with GLOBAL column indices (row-block partition)."""
    a, b = int(A.row_ptr[r0]), int(A.row_ptr[r1])
    return Csr(r1 - r0, A.n, A.row_ptr[r0:r1 + 1] - a, A.col[a:b], A.vals[a:b],
               f"{A.name}[{r0}:{r1}]")


def make_x(n: int, seed: int, dtype=np.float64) -> np.ndarray:
    return np.random.default_rng(seed + 1000).uniform(-1.0, 1.0, n).astype(dtype)


def make_config(i: int, dtype=np.float64) -> Csr:
    """Config i (1..5) of BASELINE.json, seeded with seed i."""
    if i == 1:
        A = laplacian_2d(64)
    elif i == 2:
        A = fem_banded(seed=2)
    elif i == 3:
        A = webbase_like(seed=3)
    elif i == 4:
        A = random_block(seed=4)
    elif i == 5:
        A = stencil_27pt(200)
    else:
        raise ValueError(f"no config {i}")
    A.name = f"C{i}:" + A.name
    return A.astype(dtype) if dtype != np.float64 else A


def dense_band(m: int, k: int = 32, seed: int = 7) -> Csr:
    """Dense m x k matrix (every row holds columns 0..k-1), vals U[-1,1):
    the Fig. 3 workload ('a dense matrix was used ... to avoid
    variations in performance due to cache effects when reading x')."""
    rng = np.random.default_rng(seed)
    row_ptr = np.arange(m + 1, dtype=np.int64) * k
    col = np.tile(np.arange(k, dtype=np.int32), m)
    return Csr(m, k, row_ptr, col, rng.uniform(-1.0, 1.0, m * k), f"dense_{m}x{k}")
