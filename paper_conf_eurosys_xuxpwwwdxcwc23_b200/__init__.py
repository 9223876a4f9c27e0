"""ALT's hot path on B200 (sm_100a): conv2d / GEMM executed directly on
tensors stored in ALT layouts, the conversion kernels between layouts, layout
propagation and a bounded on-device tuner.  See DESIGN.md.

The compute lives in ``libalt.so`` (C-ABI ``include/alt.h``); this package is
its ctypes binding plus plain helpers (layout builders, synthetic inputs,
network layer tables, the batch-sharded chain runner).
"""
from ._alt import (ACT, ALT_BF16, ALT_F32, AltError, ConvParams, KernelCfg, Layout, PATH_AUTO,
                   PATH_DW, PATH_SIMT, PATH_TC, conv2d, conv_params, last_plan, launch_count,
                   decouple_at, lib_path, matmul, matmul_store_at, plan_chain, store_at, pool2d, relayout, tune)

__all__ = ["ACT", "ALT_BF16", "ALT_F32", "AltError", "ConvParams", "KernelCfg", "Layout",
           "PATH_AUTO", "PATH_DW", "PATH_SIMT", "PATH_TC", "conv2d", "conv_params", "last_plan",
           "launch_count", "lib_path", "matmul", "matmul_store_at", "store_at", "decouple_at", "plan_chain", "pool2d", "relayout", "tune"]
