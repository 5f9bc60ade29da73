"""Spread layout with one process per rank under torchrun, against the float64
oracle (tests/spread_parity_worker.py; north-star gate: C1 sizes + the tail
stage, 100 steps, c13 <= 1e-5 on every rank's replica, optimizer state and
center).

* NCCL exchange: world = min(#GPUs, 8) ranks on distinct GPUs, N in {2, 4, 8}
  as far as the box allows; at one GPU, world 1 (the reduce-scatter /
  all-gather degenerate to copies but run through NCCL).
* P2P exchange: the same on distinct GPUs; on a one-GPU box, 2 ranks on cuda:0
  time-sliced (AVGPIPE_BENCH_SHARED_GPU=1, IPC handles over gloo).
"""
import json
import os
import socket
import subprocess
import sys

import pytest
import torch

from tests._parity import TOL

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        return str(sk.getsockname()[1])


def _torchrun(nproc, *args, env_extra=None, timeout=1500):
    env = dict(os.environ, AVGPIPE_EA_P2P_TIMEOUT_MS="120000", **(env_extra or {}))
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(nproc),
           "--master-addr", "127.0.0.1", "--master-port", _free_port(),
           os.path.join(ROOT, "tests", "spread_parity_worker.py"), *args]
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=timeout, env=env)
    assert r.returncode == 0, r.stderr[-4000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    return json.loads(lines[0])


def _worlds():
    g = torch.cuda.device_count()
    return [w for w in (2, 4, 8) if w <= g] or [1]


@pytest.mark.parametrize("exchange", ["nccl", "p2p"])
def test_spread_multirank_c1_100_steps(exchange):
    for w in _worlds():
        d = _torchrun(w, "--exchange", exchange)
        assert d["world"] == w and d["max_rel_err"] <= TOL, d


@pytest.mark.parametrize("optimizer", ["adamw", "asgd"])
def test_spread_multirank_optimizers(optimizer):
    w = _worlds()[-1]
    d = _torchrun(w, "--exchange", "nccl", "--optimizer", optimizer, "--steps", "30", "--sizes", "300001,17")
    assert d["max_rel_err"] <= TOL, d


@pytest.mark.skipif(torch.cuda.device_count() > 1, reason="covered on distinct GPUs")
def test_spread_p2p_two_processes_one_gpu():
    """2 ranks on one GPU (time-sliced), the fused P2P kernel across processes, 20 steps."""
    d = _torchrun(2, "--exchange", "p2p", "--steps", "20", "--sizes", "200003,64",
                  env_extra={"AVGPIPE_BENCH_SHARED_GPU": "1"})
    assert d["world"] == 2 and d["max_rel_err"] <= TOL, d
