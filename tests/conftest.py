import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def _build_lib():
    """Build libbro.so in-tree if missing or stale (nvcc cross-compiles here)."""
    import importlib.util
    spec = importlib.util.spec_from_file_location(
        "_bro_build", os.path.join(ROOT, "paper_conf_sc_tangtrwckgtw13_b200", "_build.py"))
    mod = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mod)
    mod.build()


def pytest_configure(config):
    _build_lib()
    config.addinivalue_line("markers", "gpu: needs a CUDA B200 (run via gpurun)")
    config.addinivalue_line("markers", "slow: long CPU test (full-size configs)")


@pytest.fixture(scope="session")
def golden_A():
    import json
    with open(os.path.join(ROOT, "tests", "golden", "paper_matrix_A.json")) as f:
        return json.load(f)


@pytest.fixture(scope="session")
def matrix_A(golden_A):
    """Matrix A of P:L63 as 0-based CSR (from the paper's COO arrays)."""
    import numpy as np
    from gen.matrices import Csr
    g = golden_A["coo"]
    rows = np.array(g["row_idx"]) - 1
    cols = np.array(g["col_idx"]) - 1
    vals = np.array(g["vals"], dtype=np.float64)
    m, n = golden_A["m"], golden_A["n"]
    counts = np.bincount(rows, minlength=m)
    row_ptr = np.zeros(m + 1, dtype=np.int64)
    np.cumsum(counts, out=row_ptr[1:])
    return Csr(m, n, row_ptr, cols.astype(np.int32), vals, "paper_A")


@pytest.fixture(scope="session")
def lib():
    """Build (if stale) and load libbro.so through the Python binding."""
    _build_lib()
    import paper_conf_sc_tangtrwckgtw13_b200 as P
    return P
