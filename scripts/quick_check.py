"""Fast GPU sanity check of one kernel variant (run under `timeout` before the full suites)."""
import sys
import os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from tests.test_gpu_parity import _run_colocated  # noqa: E402

variant = sys.argv[1] if len(sys.argv) > 1 else "bulkpipe"
for n in (1, 2, 4, 8):
    e = _run_colocated(n, [100_003, 7, 250_000], 3, "combined", variants=(variant,), many=True)
    print(f"{variant} N={n} many ok worst={e:.2e}", flush=True)
    e = _run_colocated(n, [100_003], 3, "paper", variants=(variant,))
    print(f"{variant} N={n} single ok worst={e:.2e}", flush=True)
print("quick_check ok")
