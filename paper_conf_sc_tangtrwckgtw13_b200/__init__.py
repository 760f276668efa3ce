"""B200-native BRO SpMV (Tang et al., SC'13): libbro.so + a thin Python binding.

Hot path: y = A.x over BRO-ELL / BRO-COO / BRO-HYB with the index streams
decoded inside sm_100a kernels (csrc/kernels.cuh) behind the C ABI of
include/bro.h.  `dist` adds the row-block multi-GPU iteration x_{k+1} = A.x_k
(allgather, overlapped allgather, or the fused P2P scatter of y into every
rank's x replica).
"""
from .bro import (  # noqa: F401
    BroError,
    BroMatrix,
    EXPORTED_SYMBOLS,
    bro_create_coo,
    bro_create_ell,
    bro_create_hyb,
    bro_decode_indices,
    bro_destroy,
    bro_export_encoded,
    bro_get_info,
    bro_hyb_K,
    bro_last_error,
    bro_opts_default,
    bro_reorder_bar,
    bro_spmv,
    bro_spmv_host,
    bro_spmv_scatter,
    BRO_MAX_DST,
    bro_status_str,
    bro_version,
    BRO_DEVICE_HOST_ONLY,
)
