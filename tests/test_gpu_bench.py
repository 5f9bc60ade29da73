"""bench.py end to end on the GPU (short runs): exactly one JSON line, the
driver's keys, a live roofline from our own kernel, e2e through the host API,
and the spread layout's code path at world 1 (its local kernel's roofline and
its e2e line).  Guards the round-end bench against crashes, not a perf gate."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
        "vs_baseline", "dtype", "data", "config", "roofline", "gpu_launches", "clocks", "e2e"}


def _bench(*args):
    r = subprocess.run([sys.executable, "bench.py", "--steps", "5", "--warmup", "3", "--e2e-steps", "2",
                        "--no-cpu-baseline", *args], cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.strip()]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert KEYS <= set(d), KEYS - set(d)
    assert d["value"] > 0 and d["gpu_launches"] > 0
    return d


def test_bench_default_line():
    d = _bench()
    assert d["config"]["workload"].startswith("C2") and d["config"]["layout"] == "colocated"
    r = d["roofline"]
    assert r["bound"] == "hbm" and 0.3 < r["frac"] < 1.3 and r["peak"] > 0
    assert d["e2e"]["h2d_bytes_per_step"] == 4 * 4 * 25_000_000 and d["e2e"]["value"] > 0


@pytest.mark.parametrize("opt", ["adam", "sgd"])
def test_bench_spread_world1_line(opt):
    d = _bench("--layout", "spread", "--config", "C1", "--optimizer", opt)
    assert d["config"]["layout"] == "spread" and d["n_gpus"] == 1
    r = d["roofline"]     # world 1: the local kernel's HBM roofline
    assert r["bound"] == "hbm" and r["kernel"].startswith("spread_bulkpipe") and r["frac"] > 0
    assert d["e2e"]["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] == 4 * 2_000_000
