"""compute-sanitizer probe of the peer-memory path at one rank (racecheck, TMA push vs register push)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import numpy as np  # noqa: E402,F401
from tests.test_gpu_p2p import _run as run_p2p  # noqa: E402

import tests._parity as par  # noqa: E402

_orig = par.rel_err


def _loud(gpu, ref):  # print every comparison's error (stage/rank come from the assertion message)
    e = _orig(gpu, ref)
    if e > par.TOL:
        import numpy as np
        g, r = np.asarray(gpu, dtype=np.float64), np.asarray(ref, dtype=np.float64)
        j = int(np.argmax(np.abs(g - r)))
        print(f"  c13 {e:.3e} at element {j} of {len(r)}: gpu {g[j]:.9g} oracle {r[j]:.9g}", flush=True)
    return e


import tests.test_gpu_p2p as tp  # noqa: E402
tp.rel_err = _loud
for opt in ("sgd", "adam"):
    for steps in (1, 2):
        try:
            run_p2p(1, [70_003, 17], steps, "combined", opt)
            print(f"p2p {opt} steps={steps} ok", os.environ.get("AVGPIPE_EA_P2P_PUSH", "bulk"), flush=True)
        except AssertionError as e:
            print(f"p2p {opt} steps={steps} PARITY FAIL", os.environ.get("AVGPIPE_EA_P2P_PUSH", "bulk"), repr(e),
                  flush=True)
