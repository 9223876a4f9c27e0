"""Run test_gpu_store_at's GEMM parity cases in one process, repeatedly, to
catch the intermittent failure of the 384x192x256 pad-7 TC case."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from tests import test_gpu_store_at as T  # noqa: E402

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 20
fails = {}
for r in range(reps):
    for case in T.GEMM_CASES:
        for dt in (torch.bfloat16, torch.float32):
            try:
                T.test_matmul_store_at_parity(case, dt)
            except AssertionError as e:
                k = (case, str(dt))
                fails[k] = fails.get(k, 0) + 1
                print("rep", r, case, dt, str(e)[:100], flush=True)
print("fails", fails)
