"""Re-run one randomized conv seed with its drawn arguments printed (developer tool)."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from tests import test_gpu_conv as TC  # noqa: E402

orig = TC.run_conv


def traced(name, N, C, H, W, K, R, S, V, pad, xp, wp, yp, dtype, **kw):
    print("ARGS", dict(N=N, C=C, H=H, W=W, K=K, R=R, S=S, V=V, pad=pad, g=kw.get("groups"), dil=kw.get("dil")),
          "\n  x", xp, "\n  w", wp, "\n  y", yp,
          "\n ", dtype, kw.get("cfg"), "res" if kw.get("res_p") is not None else "", flush=True)
    return orig(name, N, C, H, W, K, R, S, V, pad, xp, wp, yp, dtype, **kw)


TC.run_conv = traced
for s in sys.argv[1:]:
    try:
        TC.test_tc_conv_random(int(s))
        print("seed", s, "ok", flush=True)
    except AssertionError as e:
        print("seed", s, "FAIL", str(e)[:80], TC.alt.last_plan(), flush=True)
