"""compute-sanitizer probe of the peer-memory path at one rank (racecheck, TMA push vs register push)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402,F401
from tests.test_gpu_p2p import _run as run_p2p  # noqa: E402

for opt in ("sgd", "adam"):
    try:
        run_p2p(1, [70_003, 17], 2, "combined", opt)
        print(f"p2p {opt} ok", os.environ.get("AVGPIPE_EA_P2P_PUSH", "bulk"), flush=True)
    except AssertionError as e:
        print(f"p2p {opt} PARITY FAIL", os.environ.get("AVGPIPE_EA_P2P_PUSH", "bulk"), repr(e), flush=True)
