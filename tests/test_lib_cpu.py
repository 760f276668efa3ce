"""CPU tests of libbro.so (no GPU): symbol exports, input validation, and the
C++ host encoder byte-exact against the independent oracle encoder, through
host-only handles (BRO_DEVICE_HOST_ONLY: encoded, exportable, never run)."""
import os
import re
import subprocess

import numpy as np
import pytest

from gen import Csr, laplacian_2d, make_config, random_csr, random_block, row_block
from oracle import bar, bro_coo, bro_ell, hyb, spmv

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HOST = -1


def header_functions():
    src = open(os.path.join(ROOT, "include", "bro.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(bro_[A-Za-z_0-9]+)\s*\(", src)))


def test_exports_every_header_symbol(lib):
    names = header_functions()
    assert "bro_spmv" in names and "bro_create_hyb" in names
    out = subprocess.run(["nm", "-D", "--defined-only", lib.bro._LIB_PATH], capture_output=True,
                         text=True).stdout
    exported = set(re.findall(r"\bT (bro_\w+)", out))
    missing = [n for n in names if n not in exported]
    assert not missing, missing
    assert sorted(lib.EXPORTED_SYMBOLS) == names  # the binding declares exactly the header's calls
    assert lib.bro_version() == 1


def _ell_parts(lib, A, V=4, dtype=np.float64):
    o = lib.bro_opts_default(vec_words=V)
    h = lib.bro_create_ell(HOST, A.m, A.n, A.row_ptr, A.col, A.vals.astype(dtype), o)
    try:
        return {p: lib.bro_export_encoded(h, p, dtype) for p in
                ("ell_words", "ell_bit_alloc", "ell_colptr", "ell_symptr", "ell_vals")}, lib.bro_get_info(h)
    finally:
        lib.bro_destroy(h)


def _assert_ell_equal(parts, E):
    assert np.array_equal(parts["ell_colptr"], E.colptr.astype(np.uint64))
    assert np.array_equal(parts["ell_symptr"], E.symptr.astype(np.uint64))
    assert np.array_equal(parts["ell_bit_alloc"], E.bit_alloc)
    assert np.array_equal(parts["ell_words"], E.words)
    assert np.array_equal(parts["ell_vals"], E.vals)


@pytest.mark.parametrize("V", [1, 2, 4])
@pytest.mark.parametrize("seed", range(4))
def test_bro_ell_bytes_match_oracle_random(lib, V, seed):
    A = random_csr(150 + 37 * seed, 4000 if seed % 2 else 300, seed, max_len=45, empty_frac=0.15,
                   wide_cols=seed >= 2)
    parts, info = _ell_parts(lib, A, V)
    E = bro_ell.encode(A.row_ptr, A.col, A.vals, A.m, A.n, V=V)
    _assert_ell_equal(parts, E)
    assert info["ell_stream_bytes"] == E.stream_bytes()


def test_bro_ell_bytes_extreme_columns(lib):
    """n = 2^31 - 1: first deltas of 31 bits, a 31-bit jump, empty rows."""
    n = 2**31 - 1
    rows = [[0, 1, n - 1], [], [n - 2, n - 1], [2**30], [5, 2**30 + 5, n - 1]] * 9
    rp = np.zeros(len(rows) + 1, dtype=np.int64)
    rp[1:] = np.cumsum([len(r) for r in rows])
    col = np.array([c for r in rows for c in r], dtype=np.int64)
    A = Csr(len(rows), n, rp, col, np.arange(col.size, dtype=np.float64), "extreme")
    for dt in (np.float64, np.float32):
        parts, _ = _ell_parts(lib, A, 4, dt)
        E = bro_ell.encode(A.row_ptr, A.col, A.vals.astype(dt), A.m, A.n, V=4)
        _assert_ell_equal(parts, E)


def test_bro_ell_c1_closed_form(lib):
    A = laplacian_2d(64)
    parts, info = _ell_parts(lib, A)
    assert info["n_slices"] == 128 and info["ell_stream_bytes"] == 16384
    assert info["eta_stream"] == pytest.approx(0.8)  # closed form (tests/test_oracle_bro.py)
    _assert_ell_equal(parts, bro_ell.encode(A.row_ptr, A.col, A.vals, A.m, A.n))


def test_bro_ell_c2_full_fp32(lib):
    A = make_config(2, np.float32)
    parts, info = _ell_parts(lib, A, 4, np.float32)
    E = bro_ell.encode(A.row_ptr, A.col, A.vals, A.m, A.n, V=4)
    _assert_ell_equal(parts, E)
    assert 0.8 < info["eta_stream"] < 0.95  # cant-like savings (Table 3: 85.9%)


def _coo_of(A):
    rows, cols, vals = spmv.csr_to_coo(A.row_ptr, A.col, A.vals)
    return rows.astype(np.int32), cols.astype(np.int32), vals


@pytest.mark.parametrize("V", [1, 4])
def test_bro_coo_bytes_match_oracle(lib, V):
    A = random_csr(500, 700, 11, max_len=60, empty_frac=0.4, long_frac=0.03, long_len=600)
    r, c, v = _coo_of(A)
    h = lib.bro_create_coo(HOST, A.m, A.n, r, c, v, lib.bro_opts_default(vec_words=V))
    try:
        C = bro_coo.encode(r, c, v, T=32, V=V)
        assert np.array_equal(lib.bro_export_encoded(h, "coo_words"), C.words)
        assert np.array_equal(lib.bro_export_encoded(h, "coo_base_row"), C.base_row)
        assert np.array_equal(lib.bro_export_encoded(h, "coo_width"), C.width)
        assert np.array_equal(lib.bro_export_encoded(h, "coo_symptr"), C.symptr)
        assert np.array_equal(lib.bro_export_encoded(h, "coo_col"), c)
        assert np.array_equal(lib.bro_export_encoded(h, "coo_vals", np.float64), v)
    finally:
        lib.bro_destroy(h)


def test_hyb_split_and_parts_match_oracle_c3(lib):
    A = make_config(3)
    K = hyb.hyb_K(A.row_ptr)
    assert lib.bro_hyb_K(A.row_ptr) == K == 2
    h = lib.bro_create_hyb(HOST, A.m, A.n, A.row_ptr, A.col, A.vals)
    try:
        info = lib.bro_get_info(h)
        ep, ec, ev, cr, cc, cv = hyb.hyb_split(A.row_ptr, A.col, A.vals, K)
        assert info["nnz_ell"] == ec.size and info["nnz_coo"] == cc.size
        assert 0.6 < ec.size / A.nnz < 0.7  # webbase-1M: 64.2% in BRO-ELL (Table 4)
        assert info["vec_words"] == 1  # auto layout for fp64: the paper's multiplexing
        E = bro_ell.encode(ep, ec, ev, A.m, A.n, V=1, slices=[0, 1, 777, 31250])
        words = lib.bro_export_encoded(h, "ell_words")
        assert np.array_equal(lib.bro_export_encoded(h, "ell_colptr"), E.colptr)
        assert np.array_equal(lib.bro_export_encoded(h, "ell_symptr"), E.symptr)
        assert np.array_equal(lib.bro_export_encoded(h, "ell_bit_alloc"), E.bit_alloc)
        for t in (0, 1, 777, 31250):
            a, b = 32 * int(E.symptr[t]), 32 * int(E.symptr[t + 1])
            assert np.array_equal(words[a:b], E.words[a:b])
        # COO part: sampled intervals through the oracle encoder
        C = bro_coo.encode(cr[:32 * 1024 * 3], cc[:32 * 1024 * 3], cv[:32 * 1024 * 3], V=1)
        cw = lib.bro_export_encoded(h, "coo_words")
        sp = lib.bro_export_encoded(h, "coo_symptr")
        assert np.array_equal(sp[:C.symptr.size], C.symptr)
        assert np.array_equal(cw[:C.words.size], C.words)
        assert np.array_equal(lib.bro_export_encoded(h, "coo_width")[:C.width.size], C.width)
    finally:
        lib.bro_destroy(h)


def test_plain_ell_layout_matches_oracle(lib):
    A = random_csr(70, 90, 2, max_len=12, empty_frac=0.2)
    h = lib.bro_create_ell(HOST, A.m, A.n, A.row_ptr, A.col, A.vals, lib.bro_opts_default(codec=0))
    try:
        info = lib.bro_get_info(h)
        Cm, Vm = hyb.ell_arrays(A.row_ptr, A.col, A.vals)
        K, pitch = Cm.shape[1], info["ell_pitch"]
        assert info["K"] == K and pitch == 96
        col = lib.bro_export_encoded(h, "pell_col").reshape(K, pitch)
        vals = lib.bro_export_encoded(h, "pell_vals", np.float64).reshape(K, pitch)
        assert np.array_equal(col[:, :A.m].T, Cm)
        assert np.array_equal(vals[:, :A.m].T, Vm)
        assert np.all(col[:, A.m:] == -1)
    finally:
        lib.bro_destroy(h)


def test_c5_sampled_slices_match_oracle(lib):
    """Full-size C5 (8M rows, 213.8M nnz): C++ encoder vs oracle on sampled
    slices, and the closed-form nnz 598^3."""
    A = make_config(5)
    assert A.nnz == 598**3
    h = lib.bro_create_ell(HOST, A.m, A.n, A.row_ptr, A.col, A.vals)
    try:
        info = lib.bro_get_info(h)
        assert info["nnz"] == 598**3 and info["n_slices"] == 250000
        sample = [0, 1, 6249, 6250, 124999, 187500, 249999]
        sub = row_block(A, 0, A.m)
        assert info["vec_words"] == 1
        E = bro_ell.encode(sub.row_ptr, sub.col, sub.vals, A.m, A.n, V=1, slices=sample)
        assert np.array_equal(lib.bro_export_encoded(h, "ell_colptr"), E.colptr)
        assert np.array_equal(lib.bro_export_encoded(h, "ell_symptr"), E.symptr)
        words = lib.bro_export_encoded(h, "ell_words")
        vals = lib.bro_export_encoded(h, "ell_vals", np.float64)
        for t in sample:
            a, b = 32 * int(E.symptr[t]), 32 * int(E.symptr[t + 1])
            assert np.array_equal(words[a:b], E.words[a:b])
            a, b = 32 * int(E.colptr[t]), 32 * int(E.colptr[t + 1])
            assert np.array_equal(vals[a:b], E.vals[a:b])
        assert 0.8 < info["eta_stream"] < 0.87
    finally:
        lib.bro_destroy(h)


# ---------------------------------------------------------------- validation

def test_validation_errors(lib):
    rp = np.array([0, 2, 3], dtype=np.int64)
    good_c = np.array([0, 2, 1], dtype=np.int32)
    v = np.ones(3)
    h = lib.bro_create_ell(HOST, 2, 3, rp, good_c, v)
    lib.bro_destroy(h)
    cases = [
        (np.array([1, 2, 3]), good_c, 3, "BRO_ERR_INDEX"),            # row_ptr[0] != 0
        (rp, np.array([2, 0, 1]), 3, "BRO_ERR_INDEX"),                # unsorted
        (rp, np.array([1, 1, 1]), 3, "BRO_ERR_INDEX"),                # repeated column
        (rp, np.array([0, 3, 1]), 3, "BRO_ERR_INDEX"),                # col >= n
        (rp, np.array([0, -1, 1]), 3, "BRO_ERR_INDEX"),               # col < 0
        (np.array([0, 2, 1]), good_c, 3, "BRO_ERR_INDEX"),            # decreasing row_ptr
        (rp, good_c, 2**31, "BRO_ERR_SHAPE"),                         # n too large
    ]
    for rpx, cx, n, want in cases:
        with pytest.raises(lib.BroError) as ei:
            lib.bro_create_ell(HOST, 2, n, rpx, cx, v)
        assert want in str(ei.value), (rpx, cx, n, str(ei.value))
    with pytest.raises(lib.BroError, match="UNSUPPORTED"):
        lib.bro_create_ell(HOST, 2, 3, rp, good_c, v, lib.bro_opts_default(slice_h=64))
    with pytest.raises(lib.BroError, match="ARG"):
        lib.bro_create_ell(HOST, 2, 3, rp, good_c, v, lib.bro_opts_default(vec_words=3))
    with pytest.raises(lib.BroError, match="INDEX"):   # COO not sorted by row
        lib.bro_create_coo(HOST, 2, 3, np.array([1, 0]), np.array([0, 0]), np.ones(2))


def test_host_only_handle_has_no_cpu_spmv(lib):
    A = random_csr(40, 40, 0)
    h = lib.bro_create_hyb(HOST, A.m, A.n, A.row_ptr, A.col, A.vals)
    try:
        with pytest.raises(lib.BroError, match="UNSUPPORTED"):
            lib.bro_spmv(h, 1, 2, 0)
        with pytest.raises(lib.BroError, match="UNSUPPORTED"):
            lib.bro_spmv_host(h, np.zeros(A.n), np.zeros(A.m))
    finally:
        lib.bro_destroy(h)


def test_export_unknown_part_and_small_buffer(lib):
    A = random_csr(40, 40, 1)
    h = lib.bro_create_ell(HOST, A.m, A.n, A.row_ptr, A.col, A.vals)
    try:
        with pytest.raises(lib.BroError, match="ARG"):
            lib.bro_export_encoded(h, 99)
        assert lib.bro_export_encoded(h, "coo_words").size == 0  # absent part
    finally:
        lib.bro_destroy(h)


# ---------------------------------------------------------------- BAR

def test_bar_signature_order_matches_oracle(lib):
    A = random_block(seed=9, families=40, fam_rows=32)
    perm = lib.bro_reorder_bar(A.m, A.n, A.row_ptr, A.col, method=0)
    assert np.array_equal(np.sort(perm), np.arange(A.m))
    assert np.array_equal(perm, bar.signature_order(A.row_ptr, A.col, A.m))


@pytest.mark.parametrize("seed", [0, 1])
def test_bar_algorithm2_matches_oracle(lib, seed):
    A = random_block(seed=seed, families=3, fam_rows=32)   # 96 rows, 3 partitions
    Ab = row_block(A, 0, 90)                                # h does not divide m
    for M in (A, Ab):
        perm = lib.bro_reorder_bar(M.m, M.n, M.row_ptr, M.col, method=1)
        ref = bar.algorithm2(M.row_ptr, M.col, M.m, h=32)
        assert np.array_equal(perm, ref)


@pytest.mark.parametrize("min_bits", [3, 9, 31])
def test_forced_widths_bytes_match_oracle(lib, min_bits):
    """min_bits (Fig. 3 forced widths): C++ bytes == oracle bytes."""
    A = random_csr(120, 700, 4, max_len=40, empty_frac=0.1)
    o = lib.bro_opts_default(min_bits=min_bits)
    h = lib.bro_create_ell(HOST, A.m, A.n, A.row_ptr, A.col, A.vals, o)
    try:
        parts = {p: lib.bro_export_encoded(h, p, np.float64) for p in
                 ("ell_words", "ell_bit_alloc", "ell_colptr", "ell_symptr", "ell_vals")}
    finally:
        lib.bro_destroy(h)
    E = bro_ell.encode(A.row_ptr, A.col, A.vals, A.m, A.n, V=1, min_bits=min_bits)  # auto V for fp64
    _assert_ell_equal(parts, E)
    assert bro_ell.decode(E) == [A.col[A.row_ptr[i]:A.row_ptr[i + 1]].tolist() for i in range(A.m)]


def test_dense_band_eta_closed_form(lib):
    """Dense 32-column rows with every width forced to b: each row stream is
    exactly b symbols of 32 bits, so eta = 1 - b/32."""
    from gen import dense_band
    A = dense_band(320, 32)
    for b in (1, 4, 16, 31):
        h = lib.bro_create_ell(HOST, A.m, A.n, A.row_ptr, A.col, A.vals, lib.bro_opts_default(min_bits=b))
        try:
            info = lib.bro_get_info(h)
        finally:
            lib.bro_destroy(h)
        assert info["eta_stream"] == pytest.approx(1 - b / 32)


@pytest.mark.parametrize("seed,m", [(3, None), (4, 300)])
def test_bar_window_matches_oracle(lib, seed, m, monkeypatch):
    """Method 2 (Algorithm 2 with a candidate window, reading R24; window
    forced to 8 through the library's tuning variable) == the oracle's
    transcription with window=8; 10 partitions, so the window excludes some
    (and h does not divide m in the second case)."""
    monkeypatch.setenv("BRO_BAR_WINDOW", "8")
    A = random_block(seed=seed, families=10, fam_rows=32)
    if m is not None:
        A = row_block(A, 0, m)
    perm = lib.bro_reorder_bar(A.m, A.n, A.row_ptr, A.col, method=2)
    assert np.array_equal(perm, bar.algorithm2(A.row_ptr, A.col, A.m, h=32, window=8))


def test_bar_window_improves_eta_over_scrambled(lib):
    """On scrambled random-block rows (C4's generator at 1/100 size) the
    windowed greedy recovers compressibility: eta_stream of BRO-ELL rises."""
    from gen import permute_rows
    A = random_block(seed=11, families=625, fam_rows=32)
    etas = {}
    for name, method in (("scrambled", None), ("m0", 0), ("m2", 2)):
        B = A if method is None else permute_rows(A, lib.bro_reorder_bar(A.m, A.n, A.row_ptr, A.col,
                                                                          method=method))
        h = lib.bro_create_ell(HOST, B.m, B.n, B.row_ptr, B.col, B.vals)
        try:
            etas[name] = lib.bro_get_info(h)["eta_stream"]
        finally:
            lib.bro_destroy(h)
    assert etas["m2"] > etas["scrambled"] + 0.05, etas
