"""Small runs of every kernel changed in round 1 session 2, for compute-sanitizer
(memcheck / racecheck / synccheck): the bulk-copy pipeline with copies issued
from all producer lanes (SGD, Adam), the register loop with Adam, the spread
bulk pipeline (SGD, Adam; ragged tail + zero padding), the stale center with
Adam.  Each run is checked against the float64 oracle as well."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from tests.test_gpu_parity import _run_colocated, test_spread_decomposition_virtual_ranks  # noqa: E402

sizes = [20_003, 7, 4096]
for n in (1, 4, 5):
    _run_colocated(n, sizes, 2, "combined", variants=("bulkpipe",), many=True)
    _run_colocated(n, sizes, 2, "combined", variants=("bulkpipe",), many=True, optimizer="adam", lr=1e-3, wd=1e-2)
    print(f"bulkpipe N={n} ok", flush=True)
for n in (2, 3, 5, 8):
    _run_colocated(n, sizes, 2, "combined", variants=("regloop",), many=True, optimizer="adamw", lr=1e-3, wd=1e-2)
    print(f"regloop adamw N={n} ok", flush=True)
for opt in ("sgd", "adam"):
    test_spread_decomposition_virtual_ranks(2, "combined", opt, sizes=(20_003, 64), steps=2)
    print(f"spread bulk {opt} ok", flush=True)
_run_colocated(3, sizes, 3, "combined", variants=("auto",), staleness=1, many=True, optimizer="adam", lr=1e-3)
print("stale adam ok")
print("sanitize_check ok")
