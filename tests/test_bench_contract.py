"""bench.py's JSON contract, checked on CPU: the reference arm (the float64
oracle on host cores) prints exactly one JSON line with the driver's keys,
and under torchrun only rank 0 prints.  Also the algorithmic byte counts the
roofline divides by ((20N+8)P co-located SGD, 28P spread)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402

KEYS = {"metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better", "scaling",
        "vs_baseline", "dtype", "data", "config", "impl", "cpu_baseline", "e2e", "gpu_launches"}


def _json_lines(out: str):
    return [json.loads(l) for l in out.splitlines() if l.strip().startswith("{")]


def test_reference_arm_one_json_line():
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--steps", "3", "--warmup", "3"],
                       cwd=ROOT, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr
    lines = [l for l in r.stdout.splitlines() if l.strip()]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert KEYS <= set(d), KEYS - set(d)
    assert d["impl"] == "reference" and d["unit"] == bench.UNIT and d["metric"] == bench.METRIC
    assert d["config"]["workload"].startswith("C2")
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["value"] == d["value"]
    assert d["value"] > 0 and d["steps"] == 3


def test_reference_arm_under_torchrun_rank0_only():
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
                        "--master-addr", "127.0.0.1", "--master-port", "29617", "bench.py", "--impl", "reference",
                        "--gpus", "2", "--steps", "3", "--warmup", "3"],
                       cwd=ROOT, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = _json_lines(r.stdout)
    assert len(lines) == 1, r.stdout
    assert lines[0]["n_gpus"] == 2 and lines[0]["config"]["n_pipelines"] == 2


@pytest.mark.parametrize("n", [1, 2, 4, 8, 12])
def test_algorithmic_bytes(n):
    p = 1000
    # read x~ + N x (x, g, m); write N x (x, m) + x~
    assert bench.bytes_colocated(n, p) == 4 * p * ((1 + 3 * n) + (2 * n + 1))
    # Adam: + v read and written per replica
    assert bench.bytes_colocated(n, p, "adam") == 4 * p * ((1 + 4 * n) + (3 * n + 1))
    # spread: read x, g, m, x~; write x, m, r
    assert bench.bytes_spread_local(p) == 4 * p * 7
    assert bench.bytes_spread_local(p, "adam") == 4 * p * 9


def test_default_workload_is_configs1():
    assert bench.workload_key(1, None) == "C2"
    assert bench.workload_key(8, None) == "C4"


@pytest.mark.parametrize("optimizer", ["sgd", "adam"])
def test_traffic_is_keyed_by_kernel(optimizer):
    """roofline.traffic comes from an ncu capture of the SAME kernel: within 5% below the algorithmic
    bytes (dirty L2 lines at the end of an isolated launch are not yet written back), never another
    kernel's number."""
    wl = "C2-resnet50-25M-N4-K4"
    t = bench.traffic_from_profiles(wl, bench.kernel_name("auto", optimizer, 4))
    alg = bench.bytes_colocated(4, 25_000_000, optimizer)
    assert t is not None and 0.95 * alg <= t <= alg * 1.01
    assert bench.traffic_from_profiles(wl, "no_such_kernel") is None


def test_stale_kernel_name_and_launches(monkeypatch):
    """Row f4: the lane kernel for 2 <= N <= 4 and the bulk-copy pipeline for N = 1, 5..8 (Adam(W) to 6), one
    launch per <= 8 stages; the replica loop otherwise and under the AVGPIPE_EA_FORCE_WIDE knob (one launch per
    stage) -- the dispatch in ea_api.cu."""
    import argparse
    monkeypatch.delenv("AVGPIPE_EA_FORCE_WIDE", raising=False)
    assert bench.kernel_name("auto", "sgd", 4, 1) == "colocated_laneshfl<stale>"
    assert bench.kernel_name("auto", "asgd", 2, 1) == "colocated_warprep<stale,asgd>"
    assert bench.kernel_name("auto", "adam", 2, 1) == "colocated_laneshfl<stale,adam>"
    assert bench.kernel_name("auto", "sgd", 1, 1) == "colocated_bulkpipe<stale>"
    assert bench.kernel_name("auto", "sgd", 5, 1) == "colocated_warprep<stale>"
    assert bench.kernel_name("auto", "adam", 1, 1) == "colocated_warpspec<stale,adam>"
    assert bench.kernel_name("auto", "adam", 7, 1) == "colocated_warpspec<stale,adam>"
    assert bench.kernel_name("auto", "sgd", 7, 1) == "colocated_wide<stale>"
    assert bench.kernel_name("auto", "sgd", 1, 1) == "colocated_bulkpipe<stale>"
    assert bench.kernel_name("auto", "adam", 5, 1) == "colocated_warpspec<stale,adam>"
    assert bench.kernel_name("auto", "adam", 12, 1) == "colocated_wide<stale>"
    assert bench.kernel_name("auto", "sgd", 6, 1) == "colocated_wide<stale>"
    assert bench.kernel_name("auto", "sgd", 12, 1) == "colocated_wide<stale>"
    args = argparse.Namespace(optimizer="sgd", variant="auto", staleness=1)
    assert bench.colocated_launches(4, 4, args, True) == 1
    assert bench.colocated_launches(5, 4, args, True) == 1
    assert bench.colocated_launches(8, 4, args, True) == 4
    assert bench.colocated_launches(12, 4, args, True) == 4
    monkeypatch.setenv("AVGPIPE_EA_FORCE_WIDE", "1")
    assert bench.kernel_name("auto", "sgd", 4, 1) == "colocated_wide<stale>"
    assert bench.colocated_launches(4, 4, args, True) == 4
