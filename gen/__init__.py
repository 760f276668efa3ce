"""Seeded synthetic inputs shared by the oracle, the tests and bench.py.

This package holds NO arithmetic of the BRO method (no deltas, widths, bit
packing, HYB split or SpMV).  It only builds canonical CSR matrices
(row_ptr int64[m+1], col int32[nnz] strictly increasing per row, vals) and
dense x vectors, following the recipes in DESIGN.md §"Input recipe"
(SURVEY.md §8(d)).  Both sides (oracle/ and the CUDA library) consume the
same arrays; neither side's code lives here.
"""
from .matrices import (  # noqa: F401
    CONFIGS,
    Csr,
    make_config,
    make_x,
    laplacian_2d,
    stencil_27pt,
    fem_banded,
    webbase_like,
    random_block,
    random_csr,
    dense_band,
    permute_rows,
    row_block,
)
