"""Stress the randomized parity tests over many more seeds than the suite
runs (developer tool): usage: stress_random.py CONV_SEEDS GEMM_SEEDS RELAYOUT_SEEDS [ANY_PATH_SEEDS [C3D_SEEDS [STORE_AT_SEEDS [POOL_SEEDS [CHAIN_SEEDS [TUNE_SEEDS]]]]]]"""
import os
import sys
import traceback
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import pytest  # noqa: E402
from tests import test_gpu_conv as TC, test_gpu_conv3d as T3, test_gpu_relayout as TR  # noqa: E402
from tests import test_gpu_store_at as TS  # noqa: E402
from tests import test_gpu_chain as TCH  # noqa: E402

nc, ng, nr = (int(v) for v in sys.argv[1:4])
na = int(sys.argv[4]) if len(sys.argv) > 4 else 0
n3 = int(sys.argv[5]) if len(sys.argv) > 5 else 0
ns = int(sys.argv[6]) if len(sys.argv) > 6 else 0
npool = int(sys.argv[7]) if len(sys.argv) > 7 else 0
nch = int(sys.argv[8]) if len(sys.argv) > 8 else 0
ntu = int(sys.argv[9]) if len(sys.argv) > 9 else 0
off = int(os.environ.get("STRESS_SEED_OFFSET", "0"))  # explore seeds past the ones already run
fails = []
for name, fn, n, base in (("conv", TC.test_tc_conv_random, nc, 300), ("gemm", TC.test_tc_gemm_random, ng, 150),
                          ("relayout", TR.test_relayout_random_layout_pairs, nr, 240),
                          ("template", TR.test_relayout_random_conv_templates, nr // 4, 60),
                          ("any_path", TC.test_conv_random_any_path, na, 200),
                          ("c3d", T3.test_c3d_random, n3, 120),
                          ("store_at", TS.test_store_at_random, ns, 100),
                          ("pool", TCH.test_pool_random, npool, 80),
                          ("chain", TCH.test_chain_random, nch, 40),
                          ("tune", TCH.test_tune_random, ntu, 30)):
    ok = skip = 0
    for seed in range(base + off, base + off + n):
        try:
            fn(seed)
            ok += 1
        except pytest.skip.Exception:
            skip += 1
        except (Exception, pytest.fail.Exception) as e:  # noqa: BLE001
            fails.append((name, seed, repr(e)[:300]))
            traceback.print_exc(limit=2)
    print(f"{name}: {ok} ok, {skip} skipped, {len([f for f in fails if f[0] == name])} failed", flush=True)
for f in fails:
    print("FAIL", f)
