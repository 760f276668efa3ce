"""Value indexing of the BRO-ELL values ("value data compression", the future
work named in the paper's conclusion).

Test infrastructure only (see oracle/__init__.py).  The paper gives no scheme;
reading R28 takes the value-indexing method of the work it cites
for value compression ([16]: "they proposed compressing the values
data in addition to the index data"): a table of the distinct values plus one
short index per stored value.  Written step by step:

  1. D = the distinct BIT PATTERNS of the stored values (so -0.0 and 0.0, or
     two NaN payloads, stay distinct: the scheme is lossless bit for bit),
     sorted ascending as unsigned integers.
  2. code bytes cb = 1 if |D| <= 256, 2 if |D| <= 65536; more distinct values
     and the scheme does not apply (None).
  3. code of a stored value = its position in D.  The codes take the place of
     the values in the BRO-ELL slot layout (R7), grouped per row in 4-byte
     chunks of Vc = 4 / cb codes: slot (r, j) of slice t is code
        vcodes[h * colptr[t] + place(r, j, l_t, Vc, h)]
     (the multiplexing of P:L116 with 4-byte chunks); padding slots hold pz,
     the code of the first FINITE value of D (a padding slot's x is never
     gathered, so its product is a finite value times 0 = 0, reading R30);
     a part with no finite value is not indexed (None).
  4. y_i = sum_j D[code_ij] * x[c_ij] in slot order: the same products as with
     the stored values, bit for bit.
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

from .bro_ell import place


def _bits(vals: np.ndarray) -> np.ndarray:
    vals = np.ascontiguousarray(vals)
    return vals.view(np.uint64 if vals.dtype.itemsize == 8 else np.uint32)


@dataclass
class ValueIndex:
    dict_bits: np.ndarray   # step 1: sorted distinct bit patterns (uint64 / uint32)
    dict_vals: np.ndarray   # the same, as values
    cb: int                 # step 2: bytes per code
    codes: np.ndarray       # step 3: uint8 / uint16[h*colptr[s]] in the 4-byte-chunk slot layout
    pz: int = 0             # step 3: padding code (first finite value of D)


def distinct(vals: np.ndarray):
    """Steps 1-2: (D as bit patterns, D as values, cb) or None if > 65536."""
    vals = np.asarray(vals)
    D = np.unique(_bits(vals))                       # sorted ascending, unsigned
    if D.size <= 256:
        cb = 1
    elif D.size <= 65536:
        cb = 2
    else:
        return None
    return D, D.view(vals.dtype), cb


def padding_code(Dv: np.ndarray):
    """Step 3's pz: index of the first finite value of D (None if none is)."""
    fin = np.nonzero(np.isfinite(Dv))[0]
    return int(fin[0]) if fin.size else (0 if Dv.size == 0 else None)


def encode(row_ptr, vals, m, h, num_col, colptr, cap=None) -> ValueIndex | None:
    """Steps 1-3 for the BRO-ELL part whose slices have num_col / colptr (from
    oracle.bro_ell.encode); row i contributes its first min(len_i, cap) values."""
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    vals = np.asarray(vals)
    lens = np.diff(row_ptr)
    if cap is not None:
        lens = np.minimum(lens, cap)
    stored = np.concatenate([vals[row_ptr[i]:row_ptr[i] + lens[i]] for i in range(m)]) if m else vals[:0]
    got = distinct(stored)
    if got is None:
        return None
    D, Dv, cb = got
    pz = padding_code(Dv)
    if pz is None:
        return None
    Vc = 4 // cb
    codes = np.full(h * int(colptr[-1]), pz, dtype=np.uint8 if cb == 1 else np.uint16)
    pos = {int(b): k for k, b in enumerate(D)}
    bits = _bits(vals)
    s = len(num_col)
    for t in range(s):
        l = int(num_col[t])
        base = h * int(colptr[t])
        for r in range(h):
            row = t * h + r
            if row >= m:
                continue
            a = int(row_ptr[row])
            for j in range(int(lens[row])):
                codes[base + place(r, j, l, Vc, h)] = pos[int(bits[a + j])]
    return ValueIndex(D, Dv, cb, codes, pz)


def slot_values(V: ValueIndex, h, num_col, colptr, Vv) -> np.ndarray:
    """Step 4's lookup, re-laid out in the value slot layout (chunks of Vv):
    D[code] of every slot (padding slots: D[pz]).  Equal, bit for bit, to the
    BRO-ELL values at every non-padding slot (round-trip pin)."""
    out = np.zeros(h * int(colptr[-1]), dtype=V.dict_vals.dtype)
    Vc = 4 // V.cb
    for t in range(len(num_col)):
        l = int(num_col[t])
        base = h * int(colptr[t])
        for r in range(h):
            for j in range(l):
                out[base + place(r, j, l, Vv, h)] = V.dict_vals[int(V.codes[base + place(r, j, l, Vc, h)])]
    return out
