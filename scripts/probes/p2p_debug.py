"""Debug driver for the peer-memory exchange with N virtual ranks on one GPU (short timeouts, one line per case)."""
import os
import sys

os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")   # 2N streams of N virtual ranks (ea.h)
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
os.environ.setdefault("AVGPIPE_EA_P2P_TIMEOUT_MS", "5000")
from tests.test_gpu_p2p import _run  # noqa: E402

cases = [(8, [200_003, 64, 1_000_000], 10, "combined")]
if len(sys.argv) > 1 and sys.argv[1] == "all":
    cases = [(3, [200_003, 64, 1_000_000], 10, "paper"), (4, [200_003, 64, 1_000_000], 10, "paper"),
             (8, [200_003, 64, 1_000_000], 10, "combined"), (4, [1_000_000, 1_000_003], 100, "paper")]
print({k: v for k, v in os.environ.items() if k.startswith("AVGPIPE_EA") or k.startswith("CUDA_DEVICE")}, flush=True)
for n, sizes, steps, mode in cases:
    t0 = time.time()
    try:
        _run(n, sizes, steps, mode)
        print("ok", n, sizes, steps, mode, f"{time.time() - t0:.1f}s", flush=True)
    except Exception as e:
        print("FAIL", n, sizes, steps, mode, repr(e)[:300], flush=True)
