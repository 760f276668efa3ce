"""CPU tests of libbro.so (no GPU): symbol exports, input validation, and the
C++ host encoder byte-exact against the independent oracle encoder, through
host-only handles (BRO_DEVICE_HOST_ONLY: encoded, exportable, never run)."""
import os
import re
import subprocess

import numpy as np
import pytest

from gen import Csr, laplacian_2d, make_config, random_csr, random_block, row_block
from oracle import bar, bro_coo, bro_ell, hyb, metrics, spmv

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


def _ell_parts(lib, A, V=4, dtype=np.float64, h=32):
    o = lib.bro_opts_default(vec_words=V, slice_h=h)
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


@pytest.mark.parametrize("h", [32, 64])
@pytest.mark.parametrize("V", [1, 4])
@pytest.mark.parametrize("seed", range(4))
def test_bro_ell_bytes_match_oracle_random(lib, h, V, seed):
    A = random_csr(150 + 37 * seed, 4000 if seed % 2 else 300, seed, max_len=45, empty_frac=0.15,
                   wide_cols=seed >= 2)
    for dt in (np.float64, np.float32):
        parts, info = _ell_parts(lib, A, V, dt, h)
        E = bro_ell.encode(A.row_ptr, A.col, A.vals.astype(dt), A.m, A.n, h=h, V=V)
        _assert_ell_equal(parts, E)
        assert info["ell_stream_bytes"] == E.stream_bytes() and info["slice_h"] == h


def test_bro_ell_bytes_extreme_columns(lib):
    """n = 2^31 - 1: first deltas of 31 bits, a 31-bit jump, empty rows."""
    n = 2**31 - 1
    rows = [[0, 1, n - 1], [], [n - 2, n - 1], [2**30], [5, 2**30 + 5, n - 1]] * 9
    rp = np.zeros(len(rows) + 1, dtype=np.int64)
    rp[1:] = np.cumsum([len(r) for r in rows])
    col = np.array([c for r in rows for c in r], dtype=np.int64)
    A = Csr(len(rows), n, rp, col, np.arange(col.size, dtype=np.float64), "extreme")
    for dt in (np.float64, np.float32):
        for h in (32, 64):
            parts, _ = _ell_parts(lib, A, 4, dt, h)
            E = bro_ell.encode(A.row_ptr, A.col, A.vals.astype(dt), A.m, A.n, h=h, V=4)
            _assert_ell_equal(parts, E)


def test_bro_ell_c1_closed_form(lib):
    A = laplacian_2d(64)
    parts, info = _ell_parts(lib, A)
    assert info["n_slices"] == 128 and info["ell_stream_bytes"] == 16384
    assert info["eta_stream"] == pytest.approx(0.8)  # closed form (tests/test_oracle_bro.py)
    _assert_ell_equal(parts, bro_ell.encode(A.row_ptr, A.col, A.vals, A.m, A.n))


@pytest.mark.parametrize("h", [32, 64])
def test_bro_ell_c2_full_fp32(lib, h):
    A = make_config(2, np.float32)
    parts, info = _ell_parts(lib, A, 4, np.float32, h)
    E = bro_ell.encode(A.row_ptr, A.col, A.vals, A.m, A.n, h=h, V=4)
    _assert_ell_equal(parts, E)
    assert 0.8 < info["eta_stream"] < 0.95  # cant-like savings (Table 3: 85.9%)


def _coo_of(A):
    rows, cols, vals = spmv.csr_to_coo(A.row_ptr, A.col, A.vals)
    return rows.astype(np.int32), cols.astype(np.int32), vals


def _coo_parts_equal(lib, h, C, r, c, v, codec=1):
    if codec:
        assert np.array_equal(lib.bro_export_encoded(h, "coo_words"), C.words)
        assert np.array_equal(lib.bro_export_encoded(h, "coo_base_row"), C.base_row)
        assert np.array_equal(lib.bro_export_encoded(h, "coo_width"), C.width)
        assert np.array_equal(lib.bro_export_encoded(h, "coo_symptr"), C.symptr)
    else:
        assert np.array_equal(lib.bro_export_encoded(h, "coo_row"), bro_coo.plain_rows(r, C.T))
    assert np.array_equal(lib.bro_export_encoded(h, "coo_col"), C.col)
    assert np.array_equal(lib.bro_export_encoded(h, "coo_vals", v.dtype), C.vals)


@pytest.mark.parametrize("T", [8, 16, 32])
@pytest.mark.parametrize("V", [1, 4])
@pytest.mark.parametrize("codec", [1, 0])
def test_bro_coo_bytes_match_oracle(lib, T, V, codec):
    A = random_csr(500, 700, 11, max_len=60, empty_frac=0.4, long_frac=0.03, long_len=600)
    r, c, v = _coo_of(A)
    for dt in (np.float64, np.float32):
        vv = v.astype(dt)
        h = lib.bro_create_coo(HOST, A.m, A.n, r, c, vv, lib.bro_opts_default(vec_words=V, coo_T=T, codec=codec))
        try:
            info = lib.bro_get_info(h)
            assert info["coo_T"] == T and info["n_intervals"] == -(-A.nnz // (32 * T))
            C = bro_coo.encode(r, c, vv, T=T, V=1)  # COO words: V = 1 whatever vec_words says
            _coo_parts_equal(lib, h, C, r, c, vv, codec)
        finally:
            lib.bro_destroy(h)


def test_coo_auto_T():
    """coo_T = 0 resolves to 8 whatever the size."""
    import paper_conf_sc_tangtrwckgtw13_b200 as P
    for nnz, want in ((100, 8), (32 * 32 * 4736, 8)):
        rows = np.zeros(nnz, np.int32)
        cols = np.arange(nnz, dtype=np.int32)
        h = P.bro_create_coo(HOST, 1, nnz, rows, cols, np.zeros(nnz, np.float32))
        try:
            assert P.bro_get_info(h)["coo_T"] == want
        finally:
            P.bro_destroy(h)


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
        H, T = info["slice_h"], info["coo_T"]
        assert H == 32 and T == 8  # auto: ELL part rows <= K = 2 (tiny); auto T = 8
        sample = [0, 1, 777, 15624]
        E = bro_ell.encode(ep, ec, ev, A.m, A.n, h=H, V=1, slices=sample)
        words = lib.bro_export_encoded(h, "ell_words")
        assert np.array_equal(lib.bro_export_encoded(h, "ell_colptr"), E.colptr)
        assert np.array_equal(lib.bro_export_encoded(h, "ell_symptr"), E.symptr)
        assert np.array_equal(lib.bro_export_encoded(h, "ell_bit_alloc"), E.bit_alloc)
        for t in sample:
            a, b = H * int(E.symptr[t]), H * int(E.symptr[t + 1])
            assert np.array_equal(words[a:b], E.words[a:b])
        # COO part: the first intervals through the oracle encoder
        I = 32 * T
        n3 = 3 * I
        C = bro_coo.encode(cr[:n3], cc[:n3], cv[:n3], T=T, V=1)
        cw = lib.bro_export_encoded(h, "coo_words")
        sp = lib.bro_export_encoded(h, "coo_symptr")
        assert np.array_equal(sp[:C.symptr.size], C.symptr)
        assert np.array_equal(cw[:C.words.size], C.words)
        assert np.array_equal(lib.bro_export_encoded(h, "coo_width")[:C.width.size], C.width)
        assert np.array_equal(lib.bro_export_encoded(h, "coo_col")[:n3], C.col)
        assert np.array_equal(lib.bro_export_encoded(h, "coo_vals", np.float64)[:n3], C.vals)
        # HYB space savings (Table 4 analog) from the oracle's own
        # shapes and metrics (reading R19)
        _, S, _ = bro_ell.slice_shapes(ep, ec, A.m, H, 32)
        _, _, Sc = bro_coo.interval_shapes(cr, T)
        Cb = metrics.bro_hyb_stream_bytes(4 * H * int(S.sum()), 4 * 32 * int(Sc.sum()), cr.size)
        assert info["eta_stream"] == pytest.approx(metrics.eta(Cb, metrics.hyb_index_bytes(A.m, K, cr.size)),
                                                   rel=0, abs=1e-12)
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


@pytest.mark.parametrize("H", [32, 64])
def test_c5_sampled_slices_match_oracle(lib, H):
    """Full-size C5 (8M rows, 213.8M nnz): C++ encoder vs oracle on sampled
    slices, the closed-form nnz 598^3, and at h = 32 the survey's regression
    eta_stream (0.8378, tests/golden/survey_c5_layout.json)."""
    A = make_config(5)
    assert A.nnz == 598**3
    h = lib.bro_create_ell(HOST, A.m, A.n, A.row_ptr, A.col, A.vals, lib.bro_opts_default(slice_h=H))
    try:
        info = lib.bro_get_info(h)
        s = A.m // H
        assert info["nnz"] == 598**3 and info["n_slices"] == s
        sample = [0, 1, s // 40 - 1, s // 40, s // 2 - 1, 3 * s // 4, s - 1]
        assert info["vec_words"] == 1
        E = bro_ell.encode(A.row_ptr, A.col, A.vals, A.m, A.n, h=H, V=1, slices=sample)
        assert np.array_equal(lib.bro_export_encoded(h, "ell_colptr"), E.colptr)
        assert np.array_equal(lib.bro_export_encoded(h, "ell_symptr"), E.symptr)
        words = lib.bro_export_encoded(h, "ell_words")
        vals = lib.bro_export_encoded(h, "ell_vals", np.float64)
        for t in sample:
            a, b = H * int(E.symptr[t]), H * int(E.symptr[t + 1])
            assert np.array_equal(words[a:b], E.words[a:b])
            a, b = H * int(E.colptr[t]), H * int(E.colptr[t + 1])
            assert np.array_equal(vals[a:b], E.vals[a:b])
        if H == 32:
            assert round(info["eta_stream"], 4) == 0.8378
        else:
            assert 0.8 < info["eta_stream"] < 0.8378
    finally:
        lib.bro_destroy(h)


@pytest.mark.slow
def test_c4_encoding_bytes_sampled_every_S(lib):
    """C4 (2M rows, BAR method 0, BRO-HYB): the C++ encoder's bytes against
    the oracle encoder on >= 1% of the ELL slices, chosen to cover every
    symbols-per-row value S that occurs, plus the COO part's first and last
    intervals (C4's encoding was never byte-compared)."""
    from gen import permute_rows
    A0 = make_config(4)
    A = permute_rows(A0, lib.bro_reorder_bar(A0.m, A0.n, A0.row_ptr, A0.col, method=0))
    for dt, V in ((np.float64, 1), (np.float32, 4)):
        vals = A.vals.astype(dt)
        h = lib.bro_create_hyb(HOST, A.m, A.n, A.row_ptr, A.col, vals, lib.bro_opts_default(vec_words=V))
        try:
            info = lib.bro_get_info(h)
            H, T, K = info["slice_h"], info["coo_T"], info["K"]
            ep, ec, ev, cr, cc, cv = hyb.hyb_split(A.row_ptr, A.col, vals, K)
            sym = lib.bro_export_encoded(h, "ell_symptr").astype(np.int64)
            S = np.diff(sym)
            rng = np.random.default_rng(4)
            sample = set(rng.choice(S.size, S.size // 100, replace=False).tolist())
            for sv in np.unique(S):       # every S value, first and last occurrence
                idx = np.nonzero(S == sv)[0]
                sample.update([int(idx[0]), int(idx[-1])])
            sample = sorted(sample)
            assert len(sample) >= S.size // 100
            E = bro_ell.encode(ep, ec, ev, A.m, A.n, h=H, V=V, slices=sample)
            assert np.array_equal(S, E.S)
            assert np.array_equal(lib.bro_export_encoded(h, "ell_bit_alloc"), E.bit_alloc)
            assert np.array_equal(lib.bro_export_encoded(h, "ell_colptr"), E.colptr)
            words = lib.bro_export_encoded(h, "ell_words")
            ev_lib = lib.bro_export_encoded(h, "ell_vals", dt)
            for t in sample:
                a, b = H * int(E.symptr[t]), H * int(E.symptr[t + 1])
                assert np.array_equal(words[a:b], E.words[a:b]), t
                a, b = H * int(E.colptr[t]), H * int(E.colptr[t + 1])
                assert np.array_equal(ev_lib[a:b], E.vals[a:b]), t
            # COO part: first two and last interval (prefix / suffix encodes)
            I = 32 * T
            nI = info["n_intervals"]
            C = bro_coo.encode(cr[:2 * I], cc[:2 * I], cv[:2 * I], T=T, V=1)
            cw = lib.bro_export_encoded(h, "coo_words")
            assert np.array_equal(cw[:C.words.size], C.words)
            assert np.array_equal(lib.bro_export_encoded(h, "coo_vals", dt)[:2 * I], C.vals)
            e0 = (nI - 1) * I
            Cl = bro_coo.encode(cr[e0:], cc[e0:], cv[e0:], T=T, V=1)
            sp = lib.bro_export_encoded(h, "coo_symptr").astype(np.int64)
            assert np.array_equal(cw[32 * sp[nI - 1]:], Cl.words)
            assert np.array_equal(lib.bro_export_encoded(h, "coo_col")[e0:], Cl.col)
            assert int(lib.bro_export_encoded(h, "coo_base_row")[-1]) == int(Cl.base_row[0])
            # HYB eta (Table 4 analog) recomputed from the oracle's shapes
            _, Ss, _ = bro_ell.slice_shapes(ep, ec, A.m, H, 32)
            _, _, Sc = bro_coo.interval_shapes(cr, T)
            Cb = metrics.bro_hyb_stream_bytes(4 * H * int(Ss.sum()), 4 * 32 * int(Sc.sum()), cr.size)
            assert info["eta_stream"] == pytest.approx(
                metrics.eta(Cb, metrics.hyb_index_bytes(A.m, K, cr.size)), rel=0, abs=1e-12)
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
        lib.bro_create_ell(HOST, 2, 3, rp, good_c, v, lib.bro_opts_default(slice_h=48))
    with pytest.raises(lib.BroError, match="UNSUPPORTED"):
        lib.bro_create_ell(HOST, 2, 3, rp, good_c, v, lib.bro_opts_default(coo_T=12))
    for V in (2, 3):
        with pytest.raises(lib.BroError, match="ARG"):
            lib.bro_create_ell(HOST, 2, 3, rp, good_c, v, lib.bro_opts_default(vec_words=V))
    with pytest.raises(lib.BroError, match="ARG"):  # tiny instance: every slice <= 4 columns
        A = random_csr(64, 64, 0, max_len=9)
        lib.bro_create_ell(HOST, A.m, A.n, A.row_ptr, A.col, A.vals, lib.bro_opts_default(ell_kernel=1))
    with pytest.raises(lib.BroError, match="ARG"):
        lib.bro_create_ell(HOST, 2, 3, rp, good_c, v, lib.bro_opts_default(ell_kernel=11))
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


def test_instance_choice(lib):
    """Kernel instance resolved at create (bro_info_t.ell_kernel): tiny for
    slices <= 4 columns, few-slice for short h = 32 matrices, else small /
    mid / general window by the longest row stream (its symbol count from
    the oracle's slice shapes); forced instances are honoured."""
    def auto(A, h):
        _, S, _ = bro_ell.slice_shapes(A.row_ptr, A.col, A.m, h, 32)
        return 3 if S.max() < 10 else 4 if S.max() < 18 else 5
    short, mid, long_ = (random_csr(5000, 5000, 1, max_len=k) for k in (4, 12, 90))
    cases = [(short, {}, 1), (mid, {}, 2), (long_, {}, 2),
             (mid, {"slice_h": 64}, auto(mid, 64)), (long_, {"slice_h": 64}, auto(long_, 64)),
             (long_, {"slice_h": 64, "ell_kernel": 5}, 5), (mid, {"ell_kernel": 5}, 5)]
    assert auto(mid, 64) == 3 and auto(long_, 64) > 3
    for A, kw, want in cases:
        h = lib.bro_create_ell(HOST, A.m, A.n, A.row_ptr, A.col, A.vals, lib.bro_opts_default(**kw))
        try:
            assert lib.bro_get_info(h)["ell_kernel"] == want, (kw, want)
        finally:
            lib.bro_destroy(h)


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
def test_bar_window_matches_oracle(lib, seed, m):
    """Method 2 (Algorithm 2 with a candidate window, reading R24; window
    forced to 8 through bro_reorder_bar's window argument) == the oracle's
    transcription with window=8; 10 partitions, so the window excludes some
    (and h does not divide m in the second case)."""
    A = random_block(seed=seed, families=10, fam_rows=32)
    if m is not None:
        A = row_block(A, 0, m)
    perm = lib.bro_reorder_bar(A.m, A.n, A.row_ptr, A.col, method=2, window=8)
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


@pytest.mark.slow
def test_auto_slice_height(lib):
    """slice_h = 0: 64 only for big matrices (>= 303,104 rows) that are not
    tiny and whose h = 32 row streams fit the mid window (< 18 symbols,
    the oracle's slice shapes): C5 -> 64; C4 (up to 14 symbols) -> 64; C3
    (ELL part of <= 2 entries per row) -> 32; C2 (62K rows) -> 32."""
    from gen import permute_rows
    for cfg, fmt, want in ((5, "ell", 64), (4, "hyb", 64), (3, "hyb", 32), (2, "ell", 32)):
        A = make_config(cfg)
        if cfg == 4:
            A = permute_rows(A, lib.bro_reorder_bar(A.m, A.n, A.row_ptr, A.col, method=0))
        K = hyb.hyb_K(A.row_ptr) if fmt == "hyb" else int(A.row_lengths().max())
        ep, ec, _, _, _, _ = hyb.hyb_split(A.row_ptr, A.col, A.vals, K)
        l, S, _ = bro_ell.slice_shapes(ep, ec, A.m, 32, 32)
        expect = 64 if (A.m >= 303104 and l.max() > 4 and S.max() < 18) else 32
        assert expect == want, (cfg, l.max(), S.max())
        create = lib.bro_create_hyb if fmt == "hyb" else lib.bro_create_ell
        h = create(HOST, A.m, A.n, A.row_ptr, A.col, A.vals)
        try:
            assert lib.bro_get_info(h)["slice_h"] == want, cfg
        finally:
            lib.bro_destroy(h)


@pytest.mark.parametrize("seed,m", [(5, None), (6, 290)])
def test_bar_method3_matches_oracle(lib, seed, m):
    """Method 3 (windowed Algorithm 2 over the signature order, R27) ==
    the oracle's algorithm2(window=8, order=signature_order)."""
    A = random_block(seed=seed, families=10, fam_rows=32)
    if m is not None:
        A = row_block(A, 0, m)
    perm = lib.bro_reorder_bar(A.m, A.n, A.row_ptr, A.col, method=3, window=8)
    order = bar.signature_order(A.row_ptr, A.col, A.m)
    assert np.array_equal(perm, bar.algorithm2(A.row_ptr, A.col, A.m, h=32, window=8, order=order))


@pytest.mark.parametrize("h", [32, 64])
@pytest.mark.parametrize("nd", [2, 200, 3000])
@pytest.mark.parametrize("fmt", ["ell", "hyb"])
def test_value_index_bytes_match_oracle(lib, h, nd, fmt):
    """value_codec 1 (reading R28): the table and the 1-byte (<= 256 distinct)
    or 2-byte codes are byte-exact against oracle/value_index.py, for the ELL
    part only in a HYB handle; sizes reported in bro_info_t."""
    from oracle import value_index
    A = random_csr(700, 900, 11 + nd, max_len=30, empty_frac=0.1, long_frac=0.05, long_len=120)
    rng = np.random.default_rng(nd)
    pool = rng.uniform(-1, 1, nd)
    for dt in (np.float64, np.float32):
        vals = pool.astype(dt)[rng.integers(0, nd, A.nnz)]
        K = hyb.hyb_K(A.row_ptr) if fmt == "hyb" else None
        create = lib.bro_create_hyb if fmt == "hyb" else lib.bro_create_ell
        hd = create(HOST, A.m, A.n, A.row_ptr, A.col, vals, lib.bro_opts_default(slice_h=h, value_codec=1))
        try:
            info = lib.bro_get_info(hd)
            codes = lib.bro_export_encoded(hd, "ell_vcodes")
            D = lib.bro_export_encoded(hd, "ell_vdict", dt)
        finally:
            lib.bro_destroy(hd)
        E = bro_ell.encode(A.row_ptr, A.col, vals, A.m, A.n, h=h, V=1) if K is None else None
        if K is not None:
            ep, ec, ev, _, _, _ = hyb.hyb_split(A.row_ptr, A.col, vals, K)
            E = bro_ell.encode(ep, ec, ev, A.m, A.n, h=h, V=1)
        Vx = value_index.encode(A.row_ptr, vals, A.m, h, E.num_col, E.colptr, cap=K)
        assert info["value_code_bytes"] == Vx.cb and info["value_dict_size"] == Vx.dict_bits.size
        assert np.array_equal(D.view(Vx.dict_bits.dtype), Vx.dict_bits)
        assert np.array_equal(codes.view(Vx.codes.dtype), Vx.codes)
        assert info["value_bytes"] >= Vx.codes.nbytes + Vx.dict_bits.nbytes


def test_value_index_errors(lib):
    """More than 65,536 distinct values: BRO_ERR_UNSUPPORTED; value_codec with
    the uncompressed baseline or out of range: BRO_ERR_ARG."""
    A = random_csr(4000, 3000, 5, max_len=40)
    vals = np.arange(A.nnz, dtype=np.float64)
    assert A.nnz > 65536
    with pytest.raises(lib.BroError, match="UNSUPPORTED"):
        lib.bro_create_ell(HOST, A.m, A.n, A.row_ptr, A.col, vals, lib.bro_opts_default(value_codec=1))
    with pytest.raises(lib.BroError, match="ARG"):
        lib.bro_create_ell(HOST, A.m, A.n, A.row_ptr, A.col, A.vals, lib.bro_opts_default(value_codec=1, codec=0))
    with pytest.raises(lib.BroError, match="ARG"):
        lib.bro_create_ell(HOST, A.m, A.n, A.row_ptr, A.col, A.vals, lib.bro_opts_default(value_codec=2))
    with pytest.raises(lib.BroError, match="UNSUPPORTED"):  # no finite value for the padding code
        lib.bro_create_ell(HOST, A.m, A.n, A.row_ptr, A.col, np.full(A.nnz, np.inf), lib.bro_opts_default(value_codec=1))
    rows = np.repeat(np.arange(A.m, dtype=np.int32), np.diff(A.row_ptr))
    with pytest.raises(lib.BroError, match="ARG"):  # COO handles have no BRO-ELL values to index
        lib.bro_create_coo(HOST, A.m, A.n, rows, A.col, A.vals, lib.bro_opts_default(value_codec=1))
