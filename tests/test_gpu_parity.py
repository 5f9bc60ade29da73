"""GPU parity: the CUDA path through the C ABI vs the float64 oracle.

Element by element on seeded synthetic inputs (paper_conf_ppopp_chen0qz23_b200.synth),
c13 metric <= 1e-5 on every x_i, m_i and x~ (tests/_parity.py):
  * C1 (2 pipelines x 2 stages, 1M params per stage) + the ragged-tail stage
    P_s = 1,000,003, 100 steps, all three modes, both co-located kernels;
  * N in {1, 3, 5, 8, 12}, ragged/tiny/empty-vector sizes, Nesterov, weight
    decay, alpha in {0, 1};
  * the spread decomposition (local kernel -> reduce-scatter -> shard update
    -> all-gather) with N virtual ranks on one GPU, and the integrated NCCL
    path at world = 1;
  * optimizer-state get/set (checkpoint/resume) and set_hyper.
"""
import numpy as np
import pytest
import torch

from paper_conf_ppopp_chen0qz23_b200 import synth
from paper_conf_ppopp_chen0qz23_b200.binding import EAError, ElasticAveraging, get_unique_id
from tests._parity import TOL, OracleStage, asgd_kw, hyper, rel_err, to_np

pytestmark = pytest.mark.gpu

VARIANTS = ("regloop", "laneshfl", "bulkpipe")  # Adam(W): lane kernel whatever the variant


def _run_colocated(n, sizes, steps, mode, variants=VARIANTS, alpha=None, nesterov=False, wd=0.0, lr=synth.LR,
                   momentum=synth.MOMENTUM, seed=0, many=False, optimizer="sgd", staleness=0):
    hp = hyper(n, mode, alpha=alpha, lr=lr, momentum=momentum, wd=wd, nesterov=nesterov)
    dev = torch.device("cuda:0")
    oracle, gstreams = [], []
    gpu = {v: [] for v in variants}
    handles = {}
    for s, p in enumerate(sizes):
        reps, c = synth.host_state(n, p, seed=synth.WEIGHT_SEED + 97 * seed + s)
        oracle.append(OracleStage(reps, c, optimizer, staleness))
        gstreams.append(synth.GradStream(n, p, seed=synth.GRAD_SEED + 97 * seed + s))
        for v in variants:
            gpu[v].append(([torch.from_numpy(x).to(dev) for x in reps], torch.from_numpy(c).to(dev)))
    for v in variants:
        handles[v] = ElasticAveraging(sizes, n, alpha=hp.alpha, beta=hp.beta, rho=hp.rho, lr=hp.lr,
                                      momentum=hp.momentum, weight_decay=hp.weight_decay, nesterov=hp.nesterov,
                                      kernel_variant=v, optimizer=optimizer, betas=(hp.beta1, hp.beta2), eps=hp.eps,
                                      staleness=staleness, **asgd_kw(hp))
    gbuf = [[torch.empty(p, device=dev) for _ in range(n)] for p in sizes]
    order = list(reversed(range(len(sizes))))
    for t in range(steps):
        for s in range(len(sizes)):
            g = gstreams[s].next()
            for i in range(n):
                gbuf[s][i].copy_(torch.from_numpy(g[i]))
            if not many:
                for v in variants:
                    reps, c = gpu[v][s]
                    handles[v].step(s, reps, gbuf[s], c)
            oracle[s].step(g, hp)
        if many:      # every stage in one ea_step_many call (one launch per <= 8 stages)
            for v in variants:
                handles[v].step_many(order, [gpu[v][s][0] for s in order], [gbuf[s] for s in order],
                                     [gpu[v][s][1] for s in order])
    torch.cuda.synchronize()
    worst = 0.0
    for v in variants:
        for s in range(len(sizes)):
            reps, c = gpu[v][s]
            o = oracle[s]
            errs = [rel_err(to_np(c), o.c)]
            for i in range(n):
                errs.append(rel_err(to_np(reps[i]), o.xs[i]))
                errs.append(rel_err(to_np(handles[v].momentum(s, i)), o.ms[i]))
                if optimizer in ("adam", "adamw"):
                    errs.append(rel_err(to_np(handles[v].state(s, i, 1)), o.vs[i]))
            if optimizer != "sgd":
                assert handles[v].get_step(s) == steps
            e = max(errs)
            worst = max(worst, e)
            assert e <= TOL, f"variant={v} stage={s} (P={sizes[s]}) rel err {e:.3e} > {TOL}"
        handles[v].close()
    return worst


@pytest.mark.parametrize("mode", synth.MODES)
def test_c1_100_steps_with_ragged_tail(mode):
    """C1 sizes, the P_s = 1,000,003 tail stage, 100 steps (north-star gate)."""
    _run_colocated(2, [1_000_000, 1_000_003], 100, mode)


@pytest.mark.parametrize("mode", synth.MODES)
def test_c1_step_many_one_launch(mode):
    """C1 + tail stage, all stages in ONE launch per step (ea_step_many)."""
    _run_colocated(2, [1_000_000, 1_000_003], 100, mode, many=True)


@pytest.mark.parametrize("n", [1, 2, 3, 4, 8, 12])
def test_step_many_mixed_sizes_and_chunks(n):
    """10 stages of mixed/ragged sizes: > kMaxLaunchStages (8) -> 2 launches;
    tiny stages shorter than one tile or one float4."""
    sizes = [100_003, 64, 3, 65_536, 7, 1, 4099, 250_000, 33, 12_345]
    _run_colocated(n, sizes, 12, "combined", many=True)


def test_step_many_rejects_duplicates_and_bad_stage():
    h = ElasticAveraging([1000, 1000], 2)
    x = [torch.zeros(1000, device="cuda:0") for _ in range(2)]
    c = torch.zeros(1000, device="cuda:0")
    with pytest.raises(EAError, match="twice"):
        h.step_many([0, 0], [x, x], [x, x], [c, c])
    with pytest.raises(EAError, match="EA_EINVAL"):
        h.step_many([0, 2], [x, x], [x, x], [c, c])
    h.step_many([], [], [], [])
    h.close()


# ------------------------------------------------------------------ Adam / AdamW (row f1)
@pytest.mark.parametrize("optimizer", ["adam", "adamw"])
@pytest.mark.parametrize("mode", synth.MODES)
def test_adam_c1_100_steps(optimizer, mode):
    """C1 + tail stage, 100 steps, Adam(W) as the local optimizer (all stages in one launch)."""
    _run_colocated(2, [1_000_000, 1_000_003], 100, mode, optimizer=optimizer, lr=1e-3, wd=1e-2, many=True,
                   variants=("auto",))


@pytest.mark.parametrize("optimizer", ["adam", "adamw"])
@pytest.mark.parametrize("n", [1, 3, 4, 8, 12])
def test_adam_replica_counts_and_sizes(optimizer, n):
    sizes = [100_003, 7, 4096, 33]
    _run_colocated(n, sizes, 20, "combined", optimizer=optimizer, lr=1e-3, wd=1e-2, many=True, variants=("auto",))
    _run_colocated(n, sizes[:1], 10, "paper", optimizer=optimizer, lr=1e-3, variants=("auto",))


@pytest.mark.parametrize("optimizer", ["adam", "adamw"])
@pytest.mark.parametrize("n", [1, 2, 4, 5, 8])
def test_adam_bulk_pipeline(optimizer, n):
    """Adam/AdamW through the bulk-copy pipeline (x, g, m, v of every replica in the slot)."""
    sizes = [100_003, 7, 4096]
    _run_colocated(n, sizes, 12, "combined", optimizer=optimizer, lr=1e-3, wd=1e-2, many=True,
                   variants=("bulkpipe",))


@pytest.mark.parametrize("optimizer", ["adam", "adamw"])
@pytest.mark.parametrize("n", [1, 2, 3, 5, 7, 8])
def test_adam_register_loop(optimizer, n):
    """Adam/AdamW through the register-loop kernel (all (4N+1) float4 loads of a thread hoisted)."""
    sizes = [100_003, 7, 4096, 1_000_001]
    _run_colocated(n, sizes, 12, "combined", optimizer=optimizer, lr=1e-3, wd=1e-2, many=True,
                   variants=("regloop",))
    _run_colocated(n, sizes[:1], 8, "paper", optimizer=optimizer, lr=1e-3, variants=("regloop",))


# ------------------------------------------------------------------ ASGD (row f1, reading c29)
@pytest.mark.parametrize("mode", synth.MODES)
def test_asgd_c1_100_steps(mode):
    """C1 + tail stage, 100 steps, ASGD as the local optimizer (averaging from step t0 + 2 = 7 on): the
    iterate, the average ax and the center, every kernel variant, all stages in one launch."""
    _run_colocated(2, [1_000_000, 1_000_003], 100, mode, optimizer="asgd", wd=1e-3, many=True,
                   variants=("auto", "regloop", "laneshfl", "bulkpipe"))


@pytest.mark.parametrize("n", [1, 3, 4, 5, 8, 12])
def test_asgd_replica_counts_and_sizes(n):
    sizes = [100_003, 7, 4096, 33]
    _run_colocated(n, sizes, 20, "combined", optimizer="asgd", many=True)
    _run_colocated(n, sizes[:2], 12, "paper", optimizer="asgd", variants=("auto",))


# ------------------------------------------------------------------ stale center (row f4)
@pytest.mark.parametrize("n", [1, 2, 3, 4, 8, 12])
@pytest.mark.parametrize("mode", synth.MODES)
def test_stale_center(n, mode):
    """staleness 1 (reading c28): replicas dilute with x~_{t-1}, the center moves from x~_t."""
    _run_colocated(n, [100_003, 7, 4096], 40, mode, variants=("auto",), staleness=1, many=True)
    _run_colocated(n, [65_537], 20, mode, variants=("auto",), staleness=1, nesterov=True, wd=1e-3)


@pytest.mark.parametrize("optimizer", ["adam", "adamw"])
@pytest.mark.parametrize("n", [1, 2, 3, 4, 8, 12])
def test_stale_center_adam(optimizer, n):
    """staleness 1 with Adam / AdamW as the local optimizer (readings c28 + c21)."""
    _run_colocated(n, [100_003, 7, 4096], 30, "combined", variants=("auto",), staleness=1, many=True,
                   optimizer=optimizer, lr=1e-3, wd=1e-2)
    _run_colocated(n, [65_537], 15, "paper", variants=("auto",), staleness=1, optimizer=optimizer, lr=1e-3)


@pytest.mark.parametrize("n", [1, 2, 3, 4, 8, 12])
def test_stale_center_asgd(n):
    """staleness 1 with ASGD as the local optimizer (readings c28 + c29; averaging from step 7 on)."""
    _run_colocated(n, [100_003, 7, 4096], 30, "combined", variants=("auto",), staleness=1, many=True,
                   optimizer="asgd", wd=1e-3)
    _run_colocated(n, [65_537], 15, "paper", variants=("auto",), staleness=1, optimizer="asgd")


def test_stale_center_c1_100_steps():
    _run_colocated(2, [1_000_000, 1_000_003], 100, "combined", variants=("auto",), staleness=1, many=True)


@pytest.mark.parametrize("n,optimizer", [(3, "sgd"), (4, "adamw"), (2, "asgd")])
def test_stale_center_many_stage_batches(n, optimizer):
    """11 stages in one ea_step_many: the stale lane kernel (2 <= N <= 4) splits them into launches of 8 + 3."""
    sizes = [4096 * (k + 1) + k for k in range(11)]
    _run_colocated(n, sizes, 12, "combined", variants=("auto",), staleness=1, many=True, optimizer=optimizer,
                   lr=1e-3 if optimizer in ("adam", "adamw") else synth.LR)


def test_stale_center_replica_loop_knob():
    """AVGPIPE_EA_FORCE_WIDE=1 sends 2 <= N <= 4 back to the replica-loop kernel (the A/B knob): same parity."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    code = ("from tests.test_gpu_parity import _run_colocated\n"
            "for n in (2, 3, 4):\n"
            "    for opt, lr in (('sgd', 0.05), ('adamw', 1e-3), ('asgd', 0.05)):\n"
            "        _run_colocated(n, [100_003, 7, 4096], 12, 'combined', variants=('auto',), staleness=1,\n"
            "                       many=True, optimizer=opt, lr=lr)\n"
            "print('knob ok')\n")
    env = dict(os.environ, AVGPIPE_EA_FORCE_WIDE="1")
    r = subprocess.run([sys.executable, "-c", code], env=env, cwd=root, capture_output=True, text=True,
                       timeout=900)
    assert r.returncode == 0 and "knob ok" in r.stdout, r.stdout[-3000:] + r.stderr[-3000:]
