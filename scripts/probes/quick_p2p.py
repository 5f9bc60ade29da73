"""Fast sanity check of the fused peer-memory exchange with virtual ranks (run under `timeout`)."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
os.environ.setdefault("AVGPIPE_EA_P2P_TIMEOUT_MS", "5000")
from tests.test_gpu_p2p import _run  # noqa: E402

for n in (1, 2, 4):
    _run(n, [100_003, 64], 3, "combined")
    print(f"p2p N={n} ok", flush=True)
print("quick_p2p ok")
