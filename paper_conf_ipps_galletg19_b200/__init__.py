"""B200-native eps-grid similarity self-join (Gallet & Gowanlock, IPDPSW 2019).

Thin Python binding of ``libsj.so`` (``include/sj.h``).  Every function here only
marshals arguments for the C ABI of the same name; every step of the hot path runs
in the CUDA kernels of ``csrc/``.  There is no CPU fallback: importing this package
without the built library, or calling it without a CUDA device, raises.

PyTorch is used only as a holder of device / pinned memory (``torch.Tensor`` data
pointers are passed straight through) and, in :mod:`.dist`, for process groups.
"""
from ._lib import (  # noqa: F401
    SJ_OK, SJ_MORE, SJ_EINVAL, SJ_ENOMEM, SJ_ECUDA, SJ_EGRID, SJ_ESTATE,
    SJ_PATTERN_LID_UNICOMP, SJ_PATTERN_GCG, SJ_PATTERN_UNICOMP, SJ_ORDER_WORKLOAD, SJ_ORDER_CELL, SJ_ORDER_INPUT,
    PATTERNS, ORDERS,
    SJ_OPT_K, SJ_OPT_BATCH_PAIRS, SJ_OPT_STREAMS, SJ_OPT_SAMPLE_PPM, SJ_OPT_GRAB,
    SJ_OPT_COUNT_CALCS, SJ_OPT_BLOCKS_PER_SM, SJ_OPT_FAST_PATH, SJ_OPT_EXACT, SJ_OPT_QUEUE,
    SJError, SJStats, lib_path, header_functions,
    sj_abi_version, sj_kernel_launches, sj_last_error, sj_create, sj_create_ex, sj_create_part, sj_create_from_index, sj_create_from_index_view, sj_self_join, sj_destroy,
    sj_set_option, sj_set_slice, sj_get_stats, sj_export_index, sj_forward_offsets,
    sj_slice_chunks, sj_batch_chunks, sj_measure_fp64, sj_measure_atomics, sj_neighbor_csr, sj_set_stream,
    sj_part_bounds, sj_part_columns, sj_part_histogram, sj_part_pack,
    Handle, self_join_pairs,
)

__all__ = [n for n in dir() if n.startswith(("sj_", "SJ", "Handle", "self_join_pairs", "PATTERNS", "ORDERS"))]
