"""BRO-aware reordering, BAR (§3.4).

Test infrastructure only (see oracle/__init__.py).

Objective, Eqn (1):
    Phi({S_t}) = sum_i h/w * ( ceil( sum_j d(S_i, j) / alpha ) + sum_j c(S_i, j) )
Eqn (2): d(S, j) = max{ Gamma(r_aj) : r_a in S }      (delta widths)
Eqn (3) (garbled): c(S, j) = number of unique cachelines of x used by
    the j-th elements of the rows in S.  Reading R20: the union of
    Omega(c_aj), with Omega mapping the COLUMN index c_aj to its 128-byte
    line floor(c_aj * sizeof(value) / 128); padding slots touch no line.
Readings R21/R22: h = w = 32 (factor 1), alpha = sym_len = 32; line 2 sorts by
row length ascending, stable by row id; ties go to the lowest partition index;
a full partition is skipped ("the next available cluster with the lowest
cost").  When h does not divide m the last partition holds the
remaining m - (v-1)h rows (the paper assumes h | m).

Also the signature-clustering order (method 0 of bro_reorder_bar): stable sort
by (row length, jump mask, first column, row id), jump bit j >= 1 set when
Gamma(delta_j) > 2 — a DESIGN.md-defined proxy, not a paper algorithm.
"""
from __future__ import annotations

import math

import numpy as np

from .bro_ell import gamma, row_deltas


def _row(row_ptr, col, i):
    return [int(c) for c in col[int(row_ptr[i]):int(row_ptr[i + 1])]]


def d_term(rows_cols, j):
    """Eqn (2): max Gamma of the j-th delta over the rows (0 past a row's end)."""
    best = 0
    for cols in rows_cols:
        d = row_deltas(cols)
        if j < len(d):
            best = max(best, gamma(d[j]))
    return best


def c_term(rows_cols, j, vsize):
    """Eqn (3), reading R20: distinct 128-byte lines of x used by column j."""
    lines = set()
    for cols in rows_cols:
        if j < len(cols):
            lines.add(cols[j] * vsize // 128)
    return len(lines)


def phi(partitions, row_ptr, col, h=32, w=32, alpha=32, vsize=8):
    """Eqn (1) for a list of partitions (lists of row ids)."""
    total = 0
    for S in partitions:
        rows_cols = [_row(row_ptr, col, i) for i in S]
        k = max((len(c) for c in rows_cols), default=0)
        dsum = sum(d_term(rows_cols, j) for j in range(k))
        csum = sum(c_term(rows_cols, j, vsize) for j in range(k))
        total += h / w * (math.ceil(dsum / alpha) + csum)
    return total


def window_candidates(pos, sizes, cap, h, W):
    """Reading R24 (method 2): the W non-full partitions nearest to the row's
    own partition c = min(pos // h, v - 1) of the sorted sequence, ordered by
    |p - c| then p."""
    v = len(cap)
    c = min(pos // h, v - 1)
    free = [p for p in range(v) if sizes[p] < cap[p]]
    free.sort(key=lambda p: (abs(p - c), p))
    return free[:W]


def algorithm2(row_ptr, col, m, h=32, alpha=32, vsize=8, window=None, w=None, order=None):
    """Algorithm 2, evaluating the full Phi_m of line 9 for every
    candidate partition.  Returns the permutation S_1 ++ S_2 ++ ... .
    window=W restricts line 11 to window_candidates (reading R24); None is
    the paper's algorithm (every non-full partition).  w (warp size, w | h)
    defaults to h: the factor h/w multiplies every partition's term alike and
    cannot change line 11's argmin (reading R21).  order: the row sequence D
    of line 2 (default: the paper's sort by row length); method 3 of
    bro_reorder_bar passes the signature order (reading R27)."""
    w = h if w is None else w
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    if m == 0:
        return np.zeros(0, dtype=np.int64)
    v = -(-m // h)
    cap = [h] * (v - 1) + [m - (v - 1) * h]
    S = [[] for _ in range(v)]                                   # line 1
    lens = np.diff(row_ptr)
    if order is None:
        D = sorted(range(m), key=lambda i: (int(lens[i]), i))     # line 2
    else:
        D = [int(i) for i in order]                               # line 2, reading R27
    seeds = set()
    for t in range(v):                                           # lines 3-6
        S[t].append(D[t * h])
        seeds.add(t * h)
    for pos in range(m):                                         # line 7
        if pos in seeds:
            continue
        r = D[pos]
        if window is None:
            cands = list(range(v))
        else:
            cands = window_candidates(pos, [len(St) for St in S], cap, h, window)
        costs = {}
        for mm in cands:                                         # lines 8-10
            trial = [S[t] + [r] if t == mm else S[t] for t in range(v)]
            costs[mm] = phi(trial, row_ptr, col, h, w, alpha, vsize)
        best = None
        for p in sorted(cands):                                  # line 11
            if len(S[p]) < cap[p] and (best is None or costs[p] < costs[best]):
                best = p
        S[best].append(r)                                        # line 12
    return np.array([i for part in S for i in part], dtype=np.int64)


def signature_order(row_ptr, col, m):
    """Method 0 of bro_reorder_bar."""
    keys = []
    for i in range(m):
        cols = _row(row_ptr, col, i)
        d = row_deltas(cols)
        mask = tuple(1 if gamma(d[j]) > 2 else 0 for j in range(1, len(d)))
        keys.append((len(cols), mask, cols[0] if cols else -1, i))
    return np.array([k[3] for k in sorted(keys)], dtype=np.int64)
