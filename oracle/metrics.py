"""Space savings and compression ratio (§4.2.1).

Test infrastructure only (see oracle/__init__.py).

  eta   = 1 - C/O      C = compressed size of the index data, O = original
  kappa = 1 / (1 - eta)

Reading R19: C counts the compressed stream only (P:L116 counts
"the final size of the compressed stream"); O is the padded ELLPACK col_idx
(4 bytes per slot: 80 bytes for the 4x5 col_idx of matrix A), plus
2 x 4 bytes per entry for the COO part of a HYB matrix ("2nnz").
"""
from __future__ import annotations


def eta(C: float, O: float) -> float:
    return 1.0 - float(C) / float(O)


def kappa(eta_value: float) -> float:
    return 1.0 / (1.0 - float(eta_value))


def ell_index_bytes(m: int, K: int) -> int:
    """O for ELLPACK: m x K int32 col_idx."""
    return 4 * m * K


def hyb_index_bytes(m: int, K: int, nnz_coo: int) -> int:
    """O for HYB: ELL col_idx plus COO row_idx and col_idx."""
    return 4 * m * K + 8 * nnz_coo


def bro_hyb_stream_bytes(ell_stream: int, coo_row_stream: int, nnz_coo: int) -> int:
    """C for BRO-HYB: BRO-ELL stream + BRO-COO row stream + raw COO col_idx."""
    return ell_stream + coo_row_stream + 4 * nnz_coo
