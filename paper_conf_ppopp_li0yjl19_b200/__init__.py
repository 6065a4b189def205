"""B200-native variable-size batched GEMM with coordinated tiling and batching.

Reimplements the method of Li, Liang, Yan, Jia, Li, "A Coordinated Tiling and Batching
Framework for Efficient GEMM on GPUs" (PPoPP'19) for sm_100a:

* host planner (C++): tiling engine (§4.2.3), batching engine (§5), five-array encoding (§6)
* device kernels (CUDA, sm_100a): tcgen05/TMEM/TMA persistent kernel for bf16/fp16,
  FFMA kernel for fp32, both walking the batching engine's work lists (Fig. 7)
* C-ABI ``include/vbgemm.h``; this package is its thin ctypes binding.

The compute path is libvbgemm.so only; importing without it raises ImportError.
"""
from ._native import (  # noqa: F401
    Plan, VbError, check, device_info, fill_alpha_beta, fill_uniform_batch, header_symbols, lib, plan_from_schedule,
    plan_conv, plan_tune, plan_vbatched, shard_lpt, version,
    VB_BATCH_AUTO, VB_BATCH_BINARY, VB_BATCH_NONE, VB_BATCH_THRESHOLD,
    VB_TABLE_B200_FFMA, VB_TABLE_B200_TC, VB_TABLE_DEFAULT, VB_TABLE_V100,
    VB_OK, VB_ERR_ALIGNMENT, VB_ERR_CUDA, VB_ERR_INTERNAL, VB_ERR_INVALID_ARG, VB_ERR_OOM, VB_ERR_UNSUPPORTED,
)

POLICIES = {"threshold": VB_BATCH_THRESHOLD, "binary": VB_BATCH_BINARY, "none": VB_BATCH_NONE, "auto": VB_BATCH_AUTO}
