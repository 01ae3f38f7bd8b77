"""B200-native DTC-SpMM hot path: thin Python binding over libdtc.so (include/dtc.h).

Every step of the path runs in the CUDA kernels of ``csrc/``; this module only
marshals arguments (torch tensors -> raw device pointers, streams) through the
C ABI.  There is no CPU fallback: if ``libdtc.so`` is missing, importing the
binding's entry points raises.

    from paper_conf_asplos_fan0024_b200 import Format
    fmt = Format.build(rowptr, colidx, vals, M, K, dtype="tf32")   # F0-F4 on the GPU
    C = fmt.spmm(B)                                                 # S1-S5, C = A @ B
"""
from ._binding import (  # noqa: F401
    DTC_OK, DTC_ERR_INVALID, DTC_ERR_UNSORTED, DTC_ERR_DUPLICATE, DTC_ERR_RANGE, DTC_ERR_OOM,
    DTC_ERR_CUDA, DTC_ERR_NCCL, DTC_ERR_UNSUPPORTED, DTC_TF32, DTC_FP16,
    DtcError, Format, Dist, lib, library_path, exported_symbols, partition_windows, nccl_unique_id, tca_reorder,
    selector_ar, launches_per_call, version, OPTIONS, KERNELS, sched_model, make_model, selector_plan,
    selector_simulate, selector_report, SchedModel, softmax_xent, sgd_update, GCN2, tca_reorder_checked, dist_chunks,
)

__all__ = ["Format", "Dist", "DtcError", "lib", "partition_windows", "nccl_unique_id"]
