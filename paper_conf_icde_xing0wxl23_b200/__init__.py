"""B200-native LightTraffic walk-update path (Xing et al., ICDE 2023).

The product is liblt.so (C ABI in include/lt.h, CUDA kernels for sm_100a in csrc/); this package
is its thin Python binding. Importing it fails loudly when the CUDA extension is missing.
"""
from .lt import (DEEPWALK, EMPTY, INSERT_DIRECT, INSERT_WARP_AGGREGATED, LAYOUT_ADJ, LAYOUT_ADJ12, LAYOUT_AUTO,  # noqa: F401
                 LAYOUT_CSR, POLICY_PREEMPTIVE_ONLY, POLICY_ROUND_ROBIN, POLICY_SELECTIVE,
                 POLICY_SELECTIVE_ONLY, PPR, PAGERANK, LT_OK, LT_ERR_INVALID, LT_ERR_STATE, LT_ERR_OOM, LT_ERR_CUDA,
                 LT_ERR_NCCL, Engine, LTError, ipc_handle, partition_bounds, philox_device, compress_columns)

__all__ = ["Engine", "LTError", "partition_bounds", "ipc_handle", "DEEPWALK", "PPR", "PAGERANK", "EMPTY", "POLICY_SELECTIVE",
           "POLICY_ROUND_ROBIN", "INSERT_WARP_AGGREGATED", "INSERT_DIRECT", "LAYOUT_AUTO", "LAYOUT_CSR", "LAYOUT_ADJ", "LAYOUT_ADJ12",
           "POLICY_SELECTIVE_ONLY", "POLICY_PREEMPTIVE_ONLY", "LT_OK", "LT_ERR_INVALID", "LT_ERR_STATE", "LT_ERR_OOM",
           "LT_ERR_CUDA", "LT_ERR_NCCL", "philox_device", "compress_columns"]
