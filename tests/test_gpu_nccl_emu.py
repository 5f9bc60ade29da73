"""The NCCL spread exchange (rows a6/a7/e) at world 2/4/8 on ONE GPU.

The library's own EA_SPREAD + EA_XCHG_NCCL code path -- local kernel on the
caller's stream, ncclReduceScatter -> spread_apply -> in-place ncclAllGather on
the side stream, per stage in the global order K-1..0 -- runs with N ranks as N
threads of one process, NCCL replaced by the in-process emulation
tests/nccl_emu/libnccl_emu.so (LD_PRELOAD).  Checked: every rank's replica,
optimizer state and center against the float64 oracle after 100 steps (c13
<= 1e-5), the zero padding, and every collective's arguments against
parallel.shard_bounds (reduce-scatter count P_pad/N, all-gather in place from
center + rank * P_pad/N).  What the emulation does NOT cover is NCCL itself
(its transport and algorithms); the library's call sequence, counts, offsets,
aliasing and stream ordering are what is under test.
"""
import json
import os
import subprocess
import sys
import tempfile

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _emu_lib():
    from paper_conf_ppopp_chen0qz23_b200.build import build_nccl_emu
    return build_nccl_emu()


def run_emu(world, *extra, timeout=900, env_extra=None):
    lib = _emu_lib()
    with tempfile.TemporaryDirectory() as d:
        log = os.path.join(d, "calls.log")
        env = dict(os.environ, LD_PRELOAD=lib, NCCL_EMU_LOG=log, NCCL_EMU_TIMEOUT_S="300", **(env_extra or {}))
        out = subprocess.run([sys.executable, os.path.join(ROOT, "tests", "nccl_emu_worker.py"), "--world",
                              str(world), *extra], capture_output=True, text=True, timeout=timeout, env=env, cwd=ROOT)
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("{")]
    assert out.returncode == 0 and lines, out.stdout[-3000:] + out.stderr[-3000:]
    return json.loads(lines[-1])


def _check(d, steps=100, stages=2, pieces=1):
    assert "error" not in d, d
    assert d["max_err"] <= 1e-5, d
    assert d["padding_zero"], d
    c = d["collectives"]
    assert not c["bad"], c
    assert c["rs"] == c["ag"] == d["world"] * steps * stages * pieces, c


@pytest.mark.parametrize("world", [2, 4, 8])
def test_nccl_spread_path_world_n_one_gpu(world):
    """C1 sizes + the 1,000,003 tail stage, 100 steps, SGD-momentum (the north-star gate, spread layout)."""
    _check(run_emu(world))


@pytest.mark.parametrize("world,optimizer", [(2, "adam"), (4, "adamw"), (3, "asgd")])
def test_nccl_spread_path_other_optimizers(world, optimizer):
    _check(run_emu(world, "--optimizer", optimizer, "--steps", "30", "--sizes", "300001,17"), steps=30)


@pytest.mark.parametrize("world,mode", [(2, "paper"), (4, "easgd"), (3, "combined")])
def test_nccl_spread_path_modes(world, mode):
    _check(run_emu(world, "--mode", mode, "--steps", "40", "--sizes", "200003,64,1000"), steps=40, stages=3)


@pytest.mark.parametrize("world,optimizer", [(2, "sgd"), (4, "sgd"), (8, "sgd"), (3, "adam"), (2, "asgd")])
def test_stale_center_spread_world_n(world, optimizer):
    """Row f4 in EA_SPREAD: the local step of iteration t dilutes with x~_{t-1} (the snapshot the previous
    exchange took) while that exchange is still in flight (reading c28), against the stale oracle."""
    steps = 100 if optimizer == "sgd" else 30
    _check(run_emu(world, "--staleness", "1", "--optimizer", optimizer, "--steps", str(steps)), steps=steps)


@pytest.mark.parametrize("world,chunks", [(2, 3), (4, 5), (8, 2)])
def test_intra_stage_pipelining(world, chunks):
    """AVGPIPE_EA_SPREAD_CHUNKS: each stage cut into pieces whose local kernel runs while the previous piece's
    reduce-scatter / shard update / all-gather run on the side stream; every piece's calls
    checked (rank r owns block r of each piece), parity after 60 steps."""
    d = run_emu(world, "--steps", "60", env_extra={"AVGPIPE_EA_SPREAD_CHUNKS": str(chunks)})
    _check(d, steps=60, pieces=chunks)
