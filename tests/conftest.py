import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# N virtual ranks of the peer-memory exchange on ONE device drive 2N streams; the device multiplexes streams onto
# CUDA_DEVICE_MAX_CONNECTIONS hardware queues (default 8), and a spinning exchange kernel must never sit in a queue
# ahead of a push it waits for.  Set before any CUDA context exists (include/ea.h, ea_p2p_connect).
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)


def pytest_configure(config):
    config.addinivalue_line("markers", "gpu: needs a CUDA device (B200, sm_100a)")
    config.addinivalue_line("markers", "slow: long-running")


@pytest.fixture(scope="session")
def root():
    return ROOT


@pytest.fixture(autouse=True)
def _parity_margin(request):
    """Record the worst c13 error (tests/_parity.rel_err) of every GPU test in a JSON-lines log, so the margin
    to the 1e-5 gate is kept, not just pass/fail (profiles/r02_parity_margins.jsonl is a copy of one run)."""
    if request.node.get_closest_marker("gpu") is None:
        yield
        return
    from tests import _parity
    _parity.WORST["err"] = None
    yield
    err = _parity.WORST["err"]
    if err is None:
        return
    import json
    path = os.environ.get("AVGPIPE_PARITY_LOG", os.path.join(ROOT, "gpurun_out", "parity_margins.jsonl"))
    try:
        os.makedirs(os.path.dirname(path), exist_ok=True)
        with open(path, "a") as f:
            f.write(json.dumps({"test": request.node.nodeid, "worst_c13": err, "tol": _parity.TOL,
                                "margin": _parity.TOL / err if err > 0 else None}) + "\n")
    except OSError:
        pass
