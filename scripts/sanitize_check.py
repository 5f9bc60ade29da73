"""Small runs of the kernels added or changed in round 2 (and the round-1 shared-memory kernels), for
compute-sanitizer (memcheck / racecheck / synccheck): the stale center on the lane kernel (x~_{t-1} tile as a
second bulk copy on the same mbarrier; SGD / ASGD / Adam) and on the bulk-copy pipeline (x~_{t-1} as one more
stream; N = 1 and 5..8), ASGD on the lane / register / bulk kernels, the spread bulk pipeline, the peer-memory
push kernel (bulk-copy ring) + the ticket-ordered exchange kernel at one rank.
Each run is also checked against the float64 oracle."""
import os
import sys

os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")   # virtual ranks (include/ea.h)
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from tests.test_gpu_p2p import _run as run_p2p  # noqa: E402
from tests.test_gpu_parity import _run_colocated, test_spread_decomposition_virtual_ranks  # noqa: E402

sizes = [20_003, 7, 4096]
for n, opt, lr in ((2, "sgd", 0.05), (3, "asgd", 0.05), (4, "adam", 1e-3), (1, "sgd", 0.05), (5, "asgd", 0.05),
                   (6, "adamw", 1e-3), (8, "sgd", 0.05)):
    _run_colocated(n, sizes, 3, "combined", variants=("auto",), staleness=1, many=True, optimizer=opt, lr=lr)
    print(f"stale {opt} N={n} ok", flush=True)
for v in ("laneshfl", "regloop", "bulkpipe"):
    _run_colocated(4, sizes, 2, "combined", variants=(v,), many=True, optimizer="asgd")
    print(f"asgd {v} ok", flush=True)
for opt in ("sgd", "adam"):
    test_spread_decomposition_virtual_ranks(2, "combined", opt, sizes=(20_003, 64), steps=2)
    print(f"spread bulk {opt} ok", flush=True)
# one rank only: the sanitizers serialise kernels, and with N > 1 virtual ranks rank 0's exchange kernel would
# wait for rank 1's push, which is queued behind it
for opt in ("sgd", "adam"):
    run_p2p(1, [70_003, 17], 2, "combined", opt)
    print(f"p2p push+exchange {opt} ok", flush=True)
print("sanitize_check ok")
