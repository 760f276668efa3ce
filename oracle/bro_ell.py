"""BRO-ELL encoder and Algorithm-1 decoder (§3.1).

Test infrastructure only (see oracle/__init__.py).  Written step by step in
the paper's order and notation; the readings R1-R11 it relies on are listed
in DESIGN.md ("Readings of the paper").

Encoder steps:
  1. delta encoding   delta_{i,j} = c_{i,j} - c_{i,j-1}, c_{i,-1} = 0, with the
     paper's 1-based column indices; 0 marks an invalid (padding) slot.
     With 0-based columns this is delta_{i,0} = c_{i,0} + 1 (reading R1).
  2. slices of height h, each compressed independently.
  3. num_col: l_t = number of columns holding valid data in slice t (
     R9: the longest row of the slice).
  4. bit_alloc_t = [b_1 .. b_l, b_p]: b_j = max over the slice's rows of
     Gamma(delta) (Gamma(u) = bit length, Gamma(0) = 0, R2).
  5. padding b_p so that sym_len divides sum_j b_j, placed at the end
     of every row stream (R8).
  6. each row stream is the concatenation of its b_j-bit fields, most
     significant bit first (R3: Alg. 1 consumes `sym << b` from the top),
     cut into S_t = (sum_j b_j + b_p) / sym_len symbols.
  7. multiplexing: symbol q of row r of slice t is stored at
        words[h * symptr[t] + place(r, q, S_t, V, h)]
     (R11).  V = 1 is exactly the paper's comp_str_i[q*h + tid]
     (Alg. 1 line 12 with the per-row symbol counter of R4); V = 4 groups
     4 consecutive symbols of one row into one 16-byte chunk.
  8. values are slot-indexed (R7) in the same interleaved way with
     Vv = 16 / sizeof(value) slots per chunk; padding slots hold 0.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

_POW2 = np.array([1 << k for k in range(64)], dtype=np.uint64)


def gamma(u: int) -> int:
    """Gamma(u): number of bits needed to pack the unsigned integer u
    (P:L200).  Reading R2: the bit length, Gamma(0) = 0."""
    u = int(u)
    assert u >= 0
    return u.bit_length()


def gamma_np(a: np.ndarray) -> np.ndarray:
    """Vectorised Gamma: number of powers of two <= u (exact integer method)."""
    a = np.asarray(a, dtype=np.uint64)
    return np.searchsorted(_POW2, a, side="right").astype(np.int64)


def row_deltas(cols) -> list:
    """Step 1 for one row: 1-based c with c_{-1} = 0  ==>  delta_0 = c_0 + 1."""
    out = []
    prev = 0  # c_{i,-1}, 1-based
    for c in cols:
        c1 = int(c) + 1  # the paper's 1-based column index
        out.append(c1 - prev)
        prev = c1
    return out


def place(r: int, q: int, S: int, V: int, h: int) -> int:
    """Position of item q of row r inside a slice block of h*S items, when
    each row's items are grouped into chunks of V (last chunk V' = S - V*F)."""
    F = S // V
    Vp = S - V * F
    if q // V < F:
        return h * V * (q // V) + r * V + (q % V)
    return h * V * F + r * Vp + (q - V * F)


def value_chunk(itemsize: int) -> int:
    """Vv: value slots per 16-byte chunk (2 for fp64, 4 for fp32)."""
    return 16 // int(itemsize)


@dataclass
class SliceCode:
    l: int                 # num_col
    widths: list           # bit_alloc without b_p
    b_p: int               # padding bits
    S: int                 # symbols per row
    deltas: list           # h lists of length l
    symbols: list          # h lists of S ints


def encode_slice(rows_cols, h: int, sym_len: int, min_bits: int = 0) -> SliceCode:
    """Steps 1-6 for one slice.  rows_cols: h column lists (0-based, sorted
    strictly increasing); rows past the matrix end are empty lists.
    min_bits > 0 forces every width up to min_bits: the simulated compression
    ratios of the Fig. 3 experiment ("the number of bits allocated to each
    index value of a non-zero entry was varied")."""
    assert len(rows_cols) == h
    l = max((len(c) for c in rows_cols), default=0)                # step 3
    deltas = []
    for cols in rows_cols:                                          # step 1
        d = row_deltas(cols)
        deltas.append(d + [0] * (l - len(d)))                       # 0 = invalid
    widths = [max([min_bits] + [gamma(deltas[r][j]) for r in range(h)]) for j in range(l)]  # step 4
    L = sum(widths)
    S = -(-L // sym_len)                                            # step 5
    b_p = sym_len * S - L
    symbols = []
    for r in range(h):                                              # step 6
        stream = 0
        for j in range(l):
            assert deltas[r][j] < (1 << widths[j])
            stream = (stream << widths[j]) | deltas[r][j]          # MSB first
        stream <<= b_p
        mask = (1 << sym_len) - 1
        symbols.append([(stream >> (sym_len * (S - 1 - q))) & mask for q in range(S)])
    return SliceCode(l, widths, b_p, S, deltas, symbols)


@dataclass
class BroEll:
    m: int
    n: int
    h: int
    sym_len: int
    V: int
    Vv: int
    num_col: np.ndarray          # int64[s]
    S: np.ndarray                # int64[s]
    bit_alloc: np.ndarray        # uint8[colptr[s]] (b_j of every slice, b_p implied)
    colptr: np.ndarray           # uint64[s+1]
    symptr: np.ndarray           # uint64[s+1]
    words: np.ndarray            # uint32[h*symptr[s]] (or uint64 if sym_len = 64)
    vals: np.ndarray             # value dtype[h*colptr[s]]
    slices: dict = field(default_factory=dict)  # t -> SliceCode (encoded slices)

    @property
    def s(self) -> int:
        return int(self.num_col.size)

    def stream_bytes(self) -> int:
        """C of P:L246 for BRO-ELL: size of the compressed stream."""
        return int(self.h * int(self.symptr[-1]) * self.sym_len // 8)


def _slice_rows(row_ptr, col, t, h, m):
    out = []
    for r in range(t * h, t * h + h):
        if r < m:
            out.append([int(c) for c in col[int(row_ptr[r]):int(row_ptr[r + 1])]])
        else:
            out.append([])
    return out


def slice_shapes(row_ptr, col, m, h=32, sym_len=32, min_bits=0):
    """(num_col, S, widths-flat) for ALL slices, vectorised over the matrix.
    Same rules as encode_slice (steps 1, 3-5); a separate code path used to
    place sampled slices of full-size matrices (pinned against encode_slice
    by tests/test_oracle_bro_ell.py)."""
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    lens = np.diff(row_ptr)
    s = -(-m // h)
    lens_p = np.zeros(s * h, dtype=np.int64)
    lens_p[:m] = lens
    num_col = lens_p.reshape(s, h).max(axis=1) if s else np.zeros(0, np.int64)
    colptr = np.zeros(s + 1, dtype=np.int64)
    np.cumsum(num_col, out=colptr[1:])
    nnz = int(row_ptr[-1])
    rows = np.repeat(np.arange(m, dtype=np.int64), lens)
    pos = np.arange(nnz, dtype=np.int64) - np.repeat(row_ptr[:-1], lens)
    c = np.asarray(col, dtype=np.int64)
    prev = np.empty(nnz, dtype=np.int64)
    prev[1:] = c[:-1] + 1
    if nnz:
        prev[0] = 0
    prev[pos == 0] = 0
    delta = (c + 1) - prev
    g = gamma_np(delta)
    widths = np.zeros(int(colptr[-1]), dtype=np.int64)
    np.maximum.at(widths, colptr[rows // h] + pos, g)
    widths = np.maximum(widths, min_bits)
    cw = np.zeros(widths.size + 1, dtype=np.int64)
    np.cumsum(widths, out=cw[1:])
    L = cw[colptr[1:]] - cw[colptr[:-1]]          # sum_j b_j per slice (exact ints)
    S = -(-L // sym_len)
    return num_col, S, widths


def encode(row_ptr, col, vals, m, n, h=32, sym_len=32, V=4, Vv=None, slices=None,
           min_bits=0) -> BroEll:
    """BRO-ELL of the CSR matrix.  `slices=None` encodes every slice; a list
    encodes only those slices (placed at their global offsets, other words
    left 0) so full-size matrices can be checked on samples."""
    row_ptr = np.asarray(row_ptr, dtype=np.int64)
    vals = np.asarray(vals)
    if Vv is None:
        Vv = value_chunk(vals.dtype.itemsize)
    s = -(-m // h)
    num_col, S, widths_flat = slice_shapes(row_ptr, col, m, h, sym_len, min_bits)
    colptr = np.zeros(s + 1, dtype=np.uint64)
    np.cumsum(num_col, out=colptr[1:])
    symptr = np.zeros(s + 1, dtype=np.uint64)
    np.cumsum(S, out=symptr[1:])
    wdt = np.uint32 if sym_len == 32 else np.uint64
    words = np.zeros(h * int(symptr[-1]), dtype=wdt)
    vsl = np.zeros(h * int(colptr[-1]), dtype=vals.dtype)
    bit_alloc = widths_flat.astype(np.uint8)
    todo = range(s) if slices is None else slices
    codes = {}
    for t in todo:
        sc = encode_slice(_slice_rows(row_ptr, col, t, h, m), h, sym_len, min_bits)
        assert sc.l == num_col[t] and sc.S == S[t]
        bit_alloc[int(colptr[t]):int(colptr[t + 1])] = sc.widths
        wb = h * int(symptr[t])
        for r in range(h):                                           # step 7
            for q in range(sc.S):
                words[wb + place(r, q, sc.S, V, h)] = sc.symbols[r][q]
        vb = h * int(colptr[t])
        for r in range(h):                                           # step 8
            row = t * h + r
            if row >= m:
                continue
            a, b = int(row_ptr[row]), int(row_ptr[row + 1])
            for j in range(b - a):
                vsl[vb + place(r, j, sc.l, Vv, h)] = vals[a + j]
        codes[t] = sc
    return BroEll(m, n, h, sym_len, V, Vv, num_col.astype(np.int64), S.astype(np.int64),
                  bit_alloc, colptr, symptr, words, vsl, codes)


# ---------------------------------------------------------------------------
# decoder: Algorithm 1, transcribed line by line
# ---------------------------------------------------------------------------

def _top(sym: int, q: int, sym_len: int) -> int:
    """sym[0:q]: the q leading bits of the sym_len-bit buffer; zero if q <= 0
    (Definition)."""
    if q <= 0:
        return 0
    return sym >> (sym_len - q)


def alg1_slice(E: BroEll, i: int, x=None, strict=True):
    """Run Algorithm 1 for every thread tid of slice (block) i.

    Returns (cols, y): cols[tid] = decoded 0-based column list of row
    i*h + tid; y[tid] = the row's dot product with x (None if x is None).

    strict=True keeps line 5's printed 'b < rb'; reading R5: when a field ends
    exactly at a symbol boundary this loads the next symbol eagerly (reading
    past the row stream on its last symbol, guarded here to return 0); the
    decoded values are identical to the 'b <= rb' variant (strict=False) the
    kernel uses — tests assert both agree.
    """
    h, sym_len = E.h, E.sym_len
    l_i = int(E.num_col[i])
    bit_alloc_i = E.bit_alloc[int(E.colptr[i]):int(E.colptr[i + 1])]
    S_i = int(E.S[i])
    mask = (1 << sym_len) - 1
    cols_out, y_out = [], []
    for tid in range(h):                                   # 1: tid, h, i
        row_idx = i * h + tid                              # 2
        col_idx = rb = sym = decoded = 0                   # 3
        acc = 0.0
        q = 0                                              # R4: symbol counter
        mine = []

        def comp_str(qq):
            # comp_str_i[qq*h + tid] with multiplexing generalised by place()
            if qq >= S_i:
                return 0  # R5 guard: never used for a decoded value
            return int(E.words[h * int(E.symptr[i]) + place(tid, qq, S_i, E.V, h)])

        for c in range(l_i):
            b = int(bit_alloc_i[c])                        # 4
            if (b < rb) if strict else (b <= rb):          # 5
                decoded = _top(sym, b, sym_len)            # 6
                rb = rb - b                                # 7
            else:                                          # 9
                decoded = _top(sym, rb, sym_len)           # 10
                b = b - rb                                 # 11
                sym = comp_str(q)                          # 12
                q += 1
                decoded = (decoded << b) + _top(sym, b, sym_len)  # 13
                rb = sym_len - b                           # 14
            sym = (sym << b) & mask                        # 16 (R6)
            if decoded != 0:                               # 17
                col_idx = col_idx + decoded                # 18 (1-based)
                mine.append(col_idx - 1)
                if x is not None and row_idx < E.m:        # 19 (R7: slot vals)
                    v = E.vals[h * int(E.colptr[i]) + place(tid, c, l_i, E.Vv, h)]
                    acc = acc + float(v) * float(x[col_idx - 1])
        cols_out.append(mine)
        y_out.append(acc if x is not None else None)      # 22
    return cols_out, y_out


def decode(E: BroEll, strict=True):
    """Decode every row's column list (round trip of encode)."""
    out = []
    for i in range(E.s):
        cols, _ = alg1_slice(E, i, None, strict)
        out.extend(cols)
    return out[:E.m]


def spmv(E: BroEll, x, strict=True):
    """y = A.x through Algorithm 1 (plain float arithmetic, slot order)."""
    y = []
    for i in range(E.s):
        _, yy = alg1_slice(E, i, x, strict)
        y.extend(yy)
    return np.array(y[:E.m])


def decoded_slots(E: BroEll, slices=None):
    """Decoded column per slot in V=1 slot order (slot = h*colptr[t] + h*j + r),
    -1 for padding — the layout bro_decode_indices() returns."""
    out = np.full(E.h * int(E.colptr[-1]), -1, dtype=np.int64)
    todo = range(E.s) if slices is None else slices
    for t in todo:
        sc = E.slices.get(t)
        base = E.h * int(E.colptr[t])
        cols, _ = alg1_slice(E, t, None, strict=False)
        for r, lst in enumerate(cols):
            for j, c in enumerate(lst):
                out[base + E.h * j + r] = c
        del sc
    return out
