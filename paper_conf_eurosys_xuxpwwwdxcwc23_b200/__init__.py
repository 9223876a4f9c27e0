"""ALT's hot path on B200 (sm_100a): conv2d / GEMM executed directly on
tensors stored in ALT layouts, the conversion kernels between layouts, layout
propagation and a bounded on-device tuner.  See DESIGN.md.

The compute lives in ``libalt.so`` (C-ABI ``include/alt.h``); this package is
its ctypes binding plus plain helpers (layout builders, synthetic inputs,
network layer tables, the batch-sharded chain runner).

The binding is loaded on first use of any of its names (PEP 562), so the
plain helpers (``nets``, ``synth``, ``layouts``, ``tunecache``) can be
imported without mapping ``libalt.so`` — the oracle arm of bench.py does
that.  Using the binding without the library raises ImportError: there is no
CPU fallback.
"""
import importlib

__all__ = ["ACT", "ALT_BF16", "ALT_F32", "AltError", "ConvParams", "KernelCfg", "Layout",
           "PATH_AUTO", "PATH_DW", "PATH_SIMT", "PATH_TC", "conv2d", "conv_params", "conv3d", "conv3d_params",
           "last_plan",
           "launch_count", "lib_path", "matmul", "matmul_store_at", "store_at", "decouple_at", "plan_chain",
           "pool2d", "relayout", "tune"]


def __getattr__(name):
    if name == "_alt":
        return importlib.import_module("._alt", __name__)
    if name in __all__:
        mod = importlib.import_module("._alt", __name__)
        val = getattr(mod, name)
        globals()[name] = val
        return val
    raise AttributeError(f"module {__name__!r} has no attribute {name!r}")
