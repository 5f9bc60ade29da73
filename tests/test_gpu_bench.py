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


def _bench(*args, cpu=False):
    extra = ["--cpu-seconds", "1"] if cpu else ["--no-cpu-baseline"]
    r = subprocess.run([sys.executable, "bench.py", "--steps", "5", "--warmup", "3", "--e2e-steps", "2",
                        *extra, *args], cwd=ROOT, capture_output=True, text=True, timeout=600)
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


@pytest.mark.parametrize("opt,exchange", [("adam", "nccl"), ("sgd", "nccl"), ("sgd", "p2p")])
def test_bench_spread_world1_line(opt, exchange):
    d = _bench("--layout", "spread", "--config", "C1", "--optimizer", opt, "--exchange", exchange, cpu=True)
    assert d["config"]["layout"] == "spread" and d["n_gpus"] == 1
    r = d["roofline"]     # world 1: the local kernel's HBM roofline
    kern = "spread_bulkpipe" if exchange == "nccl" else "p2p_push"
    assert r["bound"] == "hbm" and r["kernel"].startswith(kern) and r["frac"] > 0 and "traffic" in r
    assert r["peak_source"]
    assert d["e2e"]["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] == 4 * 2_000_000
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    if exchange == "nccl":
        assert isinstance(d["config"]["nccl"], list)      # NCCL_DEBUG=INFO summary of the library's communicator


def test_bench_world2_line_on_one_gpu():
    """bench.py's N>1 path (torchrun, 2 ranks, spread layout, max over ranks, rank-0 JSON line, e2e)
    on a one-GPU box: both ranks on cuda:0 with the P2P exchange over CUDA IPC and a gloo control
    group (AVGPIPE_BENCH_SHARED_GPU=1; NCCL refuses two ranks on one device).  Crash guard only:
    the two ranks' kernels are time-sliced."""
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = str(sk.getsockname()[1])
    env = dict(os.environ, AVGPIPE_BENCH_SHARED_GPU="1", AVGPIPE_EA_P2P_TIMEOUT_MS="120000")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", port, "bench.py", "--gpus", "2", "--exchange", "p2p",
           "--config", "C1", "--steps", "3", "--warmup", "3", "--e2e-steps", "2", "--cpu-seconds", "1"]
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=900, env=env)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.strip().startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert KEYS <= set(d), KEYS - set(d)
    assert d["n_gpus"] == 2 and d["config"]["layout"] == "spread" and d["config"]["exchange"] == "p2p"
    r = d["roofline"]
    assert r["bound"] == "nvlink" and d["value"] > 0 and d["e2e"]["value"] > 0
    assert "B200_PROFILING" in r["peak_source"] and "traffic" in r
    loc = d["local_kernel_roofline"]          # the push kernel on each rank's caller stream
    assert loc["bound"] == "hbm" and loc["kernel"] == "p2p_push" and "traffic" in loc and loc["frac"] > 0
    cb = d["cpu_baseline"]                    # rank 0 times one stage-shard of the oracle, extrapolated
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and "extrapolated" in cb
