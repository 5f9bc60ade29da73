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
import os

import numpy as np
import pytest
import torch

from paper_conf_ppopp_chen0qz23_b200 import synth
from paper_conf_ppopp_chen0qz23_b200.binding import EAError, ElasticAveraging, get_unique_id
from tests._parity import TOL, OracleStage, asgd_kw, hyper, rel_err, to_np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

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
@pytest.mark.parametrize("n", [1, 2, 3, 4, 5, 6, 7, 8, 12])
@pytest.mark.parametrize("mode", synth.MODES)
def test_stale_center(n, mode):
    """staleness 1 (reading c28): replicas dilute with x~_{t-1}, the center moves from x~_t."""
    _run_colocated(n, [100_003, 7, 4096], 40, mode, variants=("auto",), staleness=1, many=True)
    _run_colocated(n, [65_537], 20, mode, variants=("auto",), staleness=1, nesterov=True, wd=1e-3)


@pytest.mark.parametrize("optimizer", ["adam", "adamw"])
@pytest.mark.parametrize("n", [1, 2, 3, 4, 5, 6, 8, 12])
def test_stale_center_adam(optimizer, n):
    """staleness 1 with Adam / AdamW as the local optimizer (readings c28 + c21)."""
    _run_colocated(n, [100_003, 7, 4096], 30, "combined", variants=("auto",), staleness=1, many=True,
                   optimizer=optimizer, lr=1e-3, wd=1e-2)
    _run_colocated(n, [65_537], 15, "paper", variants=("auto",), staleness=1, optimizer=optimizer, lr=1e-3)


@pytest.mark.parametrize("n", [1, 2, 3, 4, 6, 8, 12])
def test_stale_center_asgd(n):
    """staleness 1 with ASGD as the local optimizer (readings c28 + c29; averaging from step 7 on)."""
    _run_colocated(n, [100_003, 7, 4096], 30, "combined", variants=("auto",), staleness=1, many=True,
                   optimizer="asgd", wd=1e-3)
    _run_colocated(n, [65_537], 15, "paper", variants=("auto",), staleness=1, optimizer="asgd")


def test_stale_center_c1_100_steps():
    _run_colocated(2, [1_000_000, 1_000_003], 100, "combined", variants=("auto",), staleness=1, many=True)


@pytest.mark.parametrize("n,optimizer", [(3, "sgd"), (4, "adamw"), (2, "asgd"), (1, "sgd"), (6, "adam"), (8, "asgd")])
def test_stale_center_many_stage_batches(n, optimizer):
    """11 stages in one ea_step_many: the stale lane kernel (2 <= N <= 4) / bulk-copy pipeline (N = 1, 5..8)
    splits them into launches of 8 + 3."""
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


@pytest.mark.parametrize("optimizer", ["sgd", "adam", "adamw", "asgd"])
@pytest.mark.parametrize("n", [1, 3, 5, 6, 7, 8])
def test_split_register_loop(n, optimizer):
    """Variant 4 (two lanes per center column, N/2 replicas each, shuffle reduction): C1-sized stages + ragged
    ones in one launch, every optimizer."""
    lr = 1e-3 if optimizer in ("adam", "adamw") else synth.LR
    _run_colocated(n, [100_003, 7, 4096, 1_000_001], 12, "combined", variants=("split",), many=True,
                   optimizer=optimizer, lr=lr, wd=0.0 if optimizer == "sgd" else 1e-2)


@pytest.mark.parametrize("optimizer", ["sgd", "adam", "adamw", "asgd"])
@pytest.mark.parametrize("n", [1, 2, 5, 6, 7, 8])
def test_warp_per_replica(n, optimizer):
    """Variant 5 (warp per replica, contributions reduced through shared memory): C1-sized and ragged stages in
    one launch, every optimizer."""
    lr = 1e-3 if optimizer in ("adam", "adamw") else synth.LR
    _run_colocated(n, [100_003, 7, 4096, 1_000_001], 12, "combined", variants=("warprep",), many=True,
                   optimizer=optimizer, lr=lr, wd=0.0 if optimizer == "sgd" else 1e-2)


@pytest.mark.parametrize("optimizer", ["sgd", "adam", "asgd"])
@pytest.mark.parametrize("n", [1, 3, 4, 6, 8])
def test_warp_per_replica_stale(n, optimizer):
    """Variant 5 with the stale center (row f4): the replicas read x~_{t-1}, the reduction writes x~_{t+1} and
    rolls x~_{t-1} <- x~_t; several stages per launch."""
    lr = 1e-3 if optimizer in ("adam", "adamw") else synth.LR
    _run_colocated(n, [100_003, 7, 4096], 20, "combined", variants=("warprep",), many=True, optimizer=optimizer,
                   lr=lr, staleness=1)


@pytest.mark.parametrize("knobs", ["AVGPIPE_EA_WARPREP_U=2"])
def test_warp_per_replica_knobs(knobs):
    """The U = 2 geometry of the warp-per-replica kernel behind its measurement knob: every optimizer, N = 1..8,
    ragged stages in one launch, and the stale center (the knob is read once per process: a subprocess)."""
    import subprocess
    import sys
    code = ("import tests.test_gpu_parity as t\n"
            "for opt in ('sgd', 'adam', 'adamw', 'asgd'):\n"
            "    lr = 1e-3 if opt in ('adam', 'adamw') else t.synth.LR\n"
            "    for n in range(1, 9):\n"
            "        t._run_colocated(n, [100_003, 7, 4096, 300_001], 8, 'combined', variants=('warprep',), many=True,"
            " optimizer=opt, lr=lr, wd=0.0 if opt == 'sgd' else 1e-2)\n"
            "    for n in (2, 5, 8):\n"
            "        t._run_colocated(n, [100_003, 7, 4096], 8, 'combined', variants=('warprep',), many=True,"
            " optimizer=opt, lr=lr, staleness=1)\n")
    env = dict(os.environ)
    for kv in knobs.split():
        k, v = kv.split("=")
        env[k] = v
    r = subprocess.run([sys.executable, "-c", code], cwd=ROOT, env=env, capture_output=True, text=True, timeout=1200)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]


@pytest.mark.parametrize("optimizer", ["sgd", "adam", "adamw", "asgd"])
@pytest.mark.parametrize("n", [1, 2, 3, 5, 6, 7, 8])
def test_warp_specialised(n, optimizer):
    """Variant 6 (N replica warps + a reducer warp over an mbarrier ring of contribution tiles): C1-sized and
    ragged stages in one launch (ring wrap-around, ragged last tiles, scalar tails), every optimizer."""
    lr = 1e-3 if optimizer in ("adam", "adamw") else synth.LR
    _run_colocated(n, [100_003, 7, 4096, 1_000_001], 12, "combined", variants=("warpspec",), many=True,
                   optimizer=optimizer, lr=lr, wd=0.0 if optimizer == "sgd" else 1e-2)


@pytest.mark.parametrize("optimizer", ["sgd", "adam", "asgd"])
@pytest.mark.parametrize("n", [1, 2, 4, 8])
def test_warp_specialised_stale(n, optimizer):
    """Variant 6 with the stale center (row f4): replica warps read x~_{t-1}, the reducer writes x~_{t+1} and
    x~_{t-1} <- x~_t."""
    lr = 1e-3 if optimizer in ("adam", "adamw") else synth.LR
    _run_colocated(n, [100_003, 7, 4096], 20, "combined", variants=("warpspec",), many=True, optimizer=optimizer,
                   lr=lr, staleness=1)


@pytest.mark.parametrize("n,optimizer,staleness", [(8, "adam", 0), (8, "adamw", 0), (5, "sgd", 0), (5, "asgd", 0),
                                                   (3, "adam", 1), (3, "adamw", 1), (7, "adam", 0), (6, "adamw", 0),
                                                   (1, "adam", 1), (5, "adamw", 1), (6, "adam", 1), (8, "adam", 1)])
def test_library_default_kernel(n, optimizer, staleness):
    """The library's own per-N choice (kernel_variant "auto") where sessions o/v/x moved it: Adam(W) N = 6, 7 (U = 3)
    and 8 (U = 2) and SGD/ASGD N = 5 to the warp-specialised kernel, the stale Adam(W) N = 1, 3, 5-8 likewise; 30
    steps, several stages per call."""
    lr = 1e-3 if optimizer in ("adam", "adamw") else synth.LR
    _run_colocated(n, [100_003, 7, 4096, 1_000_001], 30, "combined", variants=("auto",), many=True,
                   optimizer=optimizer, lr=lr, wd=0.0 if optimizer == "sgd" else 1e-2, staleness=staleness)


def test_warp_specialised_u2_and_100_steps():
    """The U = 2 / 3 / 4 geometries behind AVGPIPE_EA_WARPSPEC_U (subprocesses: the knob is read once) and the
    100-step C1 gate with Adam at N = 8."""
    import subprocess
    import sys
    code = ("import tests.test_gpu_parity as t\n"
            "for opt in ('sgd', 'adam', 'asgd'):\n"
            "    lr = 1e-3 if opt == 'adam' else t.synth.LR\n"
            "    for n in (1, 4, 6, 7, 8):\n"
            "        t._run_colocated(n, [100_003, 7, 4096, 300_001], 8, 'combined', variants=('warpspec',), many=True,"
            " optimizer=opt, lr=lr, wd=0.0 if opt == 'sgd' else 1e-2)\n")
    for u in ("2", "3", "4"):   # (3 applies to Adam(W) only; the others run their default)
        r = subprocess.run([sys.executable, "-c", code], cwd=ROOT, env=dict(os.environ, AVGPIPE_EA_WARPSPEC_U=u),
                           capture_output=True, text=True, timeout=1200)
        assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]
    _run_colocated(8, [1_000_000, 1_000_003], 100, "combined", variants=("warpspec",), many=True, optimizer="adam",
                   lr=1e-3, wd=1e-2)


def test_warp_per_replica_c1_100_steps():
    _run_colocated(8, [1_000_000, 1_000_003], 100, "combined", variants=("warprep",), many=True, optimizer="adam",
                   lr=1e-3, wd=1e-2)


def test_split_register_loop_c1_100_steps():
    _run_colocated(8, [1_000_000, 1_000_003], 100, "combined", variants=("split",), many=True, optimizer="adam",
                   lr=1e-3, wd=1e-2)


@pytest.mark.parametrize("n,optimizer", [(33, "sgd"), (64, "sgd"), (64, "adamw")])
def test_maximum_replica_count(n, optimizer):
    """EA_MAX_REPLICAS = 64 co-located replicas (the replica-loop kernel's pointer table)."""
    _run_colocated(n, [20_003, 5], 6, "combined", optimizer=optimizer, lr=1e-3 if optimizer != "sgd" else synth.LR,
                   many=True, variants=("auto",))


@pytest.mark.parametrize("n", [1, 3, 5, 6, 7, 8, 12])
@pytest.mark.parametrize("mode", synth.MODES)
def test_replica_counts(n, mode):
    _run_colocated(n, [65_539, 4097], 30, mode)


@pytest.mark.parametrize("p", [1, 2, 3, 4, 5, 7, 31, 127, 1029, 4096 * 8 + 3])
def test_tiny_and_ragged_sizes(p):
    _run_colocated(3, [p], 12, "combined")
    _run_colocated(4, [p], 5, "paper")


@pytest.mark.parametrize("nesterov,wd", [(True, 0.0), (False, 1e-2), (True, 5e-3)])
def test_nesterov_and_weight_decay(nesterov, wd):
    _run_colocated(4, [300_001], 40, "combined", nesterov=nesterov, wd=wd)


@pytest.mark.parametrize("alpha", [0.0, 1.0, 0.37])
def test_alpha_edges(alpha):
    _run_colocated(3, [100_003], 25, "easgd", alpha=alpha)
    _run_colocated(3, [100_003], 25, "paper", alpha=alpha)


def test_plain_sgd_momentum_zero():
    _run_colocated(2, [10_000], 20, "paper", momentum=0.0)


# ------------------------------------------------------------------ spread
def _placement(rank, stage, n):
    from paper_conf_ppopp_chen0qz23_b200.parallel import replica_of
    return replica_of(rank, stage, n)


@pytest.mark.parametrize("n,optimizer", [(2, "sgd"), (3, "sgd"), (4, "sgd"), (8, "sgd"), (2, "adam"), (4, "adamw"),
                                         (3, "asgd")])
@pytest.mark.parametrize("mode", synth.MODES)
def test_spread_decomposition_virtual_ranks(n, mode, optimizer, sizes=(200_003, 64), steps=20):
    """N ranks on one GPU, external-collective mode: the real local and shard
    kernels, with the reduce-scatter / all-gather done by the test."""
    sizes = list(sizes)
    hp = hyper(n, mode, lr=synth.LR if optimizer in ("sgd", "asgd") else 1e-3, wd=0.0 if optimizer == "sgd" else 1e-2)
    dev = torch.device("cuda:0")
    hs = [ElasticAveraging(sizes, n, alpha=hp.alpha, beta=hp.beta, rho=hp.rho, lr=hp.lr, momentum=hp.momentum,
                           weight_decay=hp.weight_decay, layout="spread", rank=r, world=n, optimizer=optimizer,
                           **asgd_kw(hp))
          for r in range(n)]
    oracle, gstreams, xs, centers = [], [], [], []
    for s, p in enumerate(sizes):
        reps, c = synth.host_state(n, p, seed=synth.WEIGHT_SEED + s)
        oracle.append(OracleStage(reps, c, optimizer))
        gstreams.append(synth.GradStream(n, p, seed=synth.GRAD_SEED + s))
        cap = hs[0].center_capacity(s)
        assert cap % (32 * n) == 0 and cap >= p
        assert hs[0].shard_elems(s) * n == cap
        cs = []
        for r in range(n):
            cr = torch.zeros(cap, device=dev)
            cr[:p] = torch.from_numpy(c)
            cs.append(cr)
        centers.append(cs)
        xs.append([torch.from_numpy(reps[_placement(r, s, n)]).to(dev) for r in range(n)])
    for t in range(steps):
        for s in reversed(range(len(sizes))):   # global stage order K-1 .. 0
            p = sizes[s]
            cap = hs[0].center_capacity(s)
            shard = cap // n
            g = gstreams[s].next()
            contribs = []
            for r in range(n):
                gr = torch.from_numpy(g[_placement(r, s, n)]).to(dev)
                cb = torch.full((cap,), float("nan"), device=dev)    # padding must be written as 0
                hs[r].spread_local(s, xs[s][r], gr, centers[s][r], cb)
                contribs.append(cb)
            total = torch.stack(contribs).sum(0)                     # reduce-scatter (sum)
            for r in range(n):
                hs[r].spread_apply(s, centers[s][r][r * shard:(r + 1) * shard], total[r * shard:(r + 1) * shard])
            for r in range(n):                                        # all-gather
                for q in range(n):
                    if q != r:
                        centers[s][q][r * shard:(r + 1) * shard].copy_(centers[s][r][r * shard:(r + 1) * shard])
            oracle[s].step(g, hp)
    torch.cuda.synchronize()
    for s, p in enumerate(sizes):
        o = oracle[s]
        for r in range(n):
            i = _placement(r, s, n)
            assert rel_err(to_np(xs[s][r]), o.xs[i]) <= TOL
            assert rel_err(to_np(hs[r].momentum(s, 0)), o.ms[i]) <= TOL
            if optimizer in ("adam", "adamw"):
                assert rel_err(to_np(hs[r].state(s, 0, 1)), o.vs[i]) <= TOL
            assert rel_err(to_np(centers[s][r][:p]), o.c) <= TOL
            assert torch.all(centers[s][r][p:] == 0), "center padding must stay zero"
    for h in hs:
        h.close()


@pytest.mark.parametrize("kernel", ["reg"])
@pytest.mark.parametrize("optimizer", ["sgd", "adam", "asgd"])
def test_spread_local_kernel_variants(kernel, optimizer):
    """The spread local step on the register kernel behind AVGPIPE_EA_SPREAD_KERNEL=reg (the contribution to the
    exchange buffer, the padding zeroed), 4 virtual ranks (the knob is read once per process: a subprocess)."""
    import subprocess
    import sys
    code = ("import tests.test_gpu_parity as t; "
            f"t.test_spread_decomposition_virtual_ranks(4, 'combined', '{optimizer}', sizes=(1_000_003, 200_003, 64), "
            "steps=12)")
    env = dict(os.environ, AVGPIPE_EA_SPREAD_KERNEL=kernel)
    r = subprocess.run([sys.executable, "-c", code], cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-4000:]


@pytest.mark.parametrize("n,mode", [(2, m) for m in synth.MODES] + [(4, m) for m in synth.MODES] + [(8, "combined")])
def test_spread_decomposition_c1_100_steps(n, mode):
    """North-star gate for the NCCL layout's kernels: C1 + tail stage, 100 steps, N = 2/4/8 virtual ranks."""
    test_spread_decomposition_virtual_ranks(n, mode, "sgd", sizes=(1_000_000, 1_000_003), steps=100)


def test_spread_nccl_world1_and_stream_order():
    """Integrated EA_SPREAD path (NCCL reduce-scatter / all-gather on the
    library's side stream) at world = 1, driven from a non-default stream."""
    sizes = [100_003, 5]
    hp = hyper(1, "combined")
    dev = torch.device("cuda:0")
    h = ElasticAveraging(sizes, 1, alpha=hp.alpha, beta=hp.beta, rho=hp.rho, lr=hp.lr, momentum=hp.momentum,
                         layout="spread", rank=0, world=1, nccl_id=get_unique_id())
    stream = torch.cuda.Stream()
    oracle, gstreams, xs, cs = [], [], [], []
    for s, p in enumerate(sizes):
        reps, c = synth.host_state(1, p, seed=synth.WEIGHT_SEED + s)
        oracle.append(OracleStage(reps, c))
        gstreams.append(synth.GradStream(1, p, seed=synth.GRAD_SEED + s))
        cap = h.center_capacity(s)
        cc = torch.zeros(cap, device=dev)
        cc[:p] = torch.from_numpy(c)
        cs.append(cc)
        xs.append(torch.from_numpy(reps[0]).to(dev))
    with torch.cuda.stream(stream):
        for t in range(15):
            for s in reversed(range(len(sizes))):
                g = gstreams[s].next()
                gd = torch.from_numpy(g[0]).to(dev, non_blocking=False)
                h.step(s, [xs[s]], [gd], cs[s], stream=stream)
                oracle[s].step(g, hp)
        h.sync(stream)
    stream.synchronize()
    for s, p in enumerate(sizes):
        assert rel_err(to_np(xs[s]), oracle[s].xs[0]) <= TOL
        assert rel_err(to_np(cs[s][:p]), oracle[s].c) <= TOL
        assert rel_err(to_np(h.momentum(s, 0)), oracle[s].ms[0]) <= TOL
    buf = torch.zeros(sizes[0] + 4, device=dev)
    with pytest.raises(EAError):
        h.step(0, [buf[1:sizes[0] + 1]], [buf[1:sizes[0] + 1]], cs[0])   # misaligned pointers -> EA_EINVAL
    h.close()


def test_spread_external_mode_rejects_ea_step():
    h = ElasticAveraging([1000], 2, layout="spread", rank=0, world=2)
    x = torch.zeros(1000, device="cuda:0")
    c = torch.zeros(h.center_capacity(0), device="cuda:0")
    with pytest.raises(EAError, match="EA_ESTATE"):
        h.step(0, [x], [x], c)
    h.close()


# ------------------------------------------------------------------ state & errors
def test_state_roundtrip_and_set_hyper():
    """Checkpoint the library-owned momentum, resume in a fresh handle, and
    change the learning rate mid-run: must equal an uninterrupted oracle run."""
    n, p = 3, 50_001
    dev = torch.device("cuda:0")
    hp1 = hyper(n, "combined")
    hp2 = hyper(n, "combined", lr=0.01)
    reps, c = synth.host_state(n, p)
    o = OracleStage(reps, c)
    gs = synth.GradStream(n, p)
    xs = [torch.from_numpy(x).to(dev) for x in reps]
    cc = torch.from_numpy(c).to(dev)
    kw = dict(alpha=hp1.alpha, beta=hp1.beta, rho=hp1.rho, momentum=hp1.momentum)
    h = ElasticAveraging([p], n, lr=hp1.lr, **kw)
    for t in range(5):
        g = gs.next()
        h.step(0, xs, [torch.from_numpy(a).to(dev) for a in g], cc)
        o.step(g, hp1)
    saved = [h.momentum(0, i).clone() for i in range(n)]
    h.close()
    h2 = ElasticAveraging([p], n, lr=hp1.lr, **kw)
    for i in range(n):
        h2.set_momentum(0, i, saved[i])
    h2.set_hyper(alpha=hp2.alpha, beta=hp2.beta, rho=hp2.rho, lr=hp2.lr, momentum=hp2.momentum)
    for t in range(5):
        g = gs.next()
        h2.step(0, xs, [torch.from_numpy(a).to(dev) for a in g], cc)
        o.step(g, hp2)
    torch.cuda.synchronize()
    assert rel_err(to_np(cc), o.c) <= TOL
    for i in range(n):
        assert rel_err(to_np(xs[i]), o.xs[i]) <= TOL
        assert rel_err(to_np(h2.momentum(0, i)), o.ms[i]) <= TOL
    h2.close()


def test_adam_checkpoint_resume():
    """Both Adam moments and the step count (bias correction) survive a
    checkpoint into a fresh handle; the resumed run equals an uninterrupted one."""
    n, p = 3, 70_001
    dev = torch.device("cuda:0")
    hp = hyper(n, "combined", lr=1e-3, wd=1e-2)
    reps, c = synth.host_state(n, p)
    o = OracleStage(reps, c, "adamw")
    gs = synth.GradStream(n, p)
    xs = [torch.from_numpy(x).to(dev) for x in reps]
    cc = torch.from_numpy(c).to(dev)
    kw = dict(alpha=hp.alpha, beta=hp.beta, rho=hp.rho, lr=hp.lr, weight_decay=hp.weight_decay, optimizer="adamw")
    h = ElasticAveraging([p], n, **kw)
    for t in range(4):
        g = gs.next()
        h.step(0, xs, [torch.from_numpy(a).to(dev) for a in g], cc)
        o.step(g, hp)
    saved = [(h.state(0, i, 0).clone(), h.state(0, i, 1).clone()) for i in range(n)]
    t_saved = h.get_step(0)
    assert t_saved == 4
    h.close()
    h2 = ElasticAveraging([p], n, **kw)
    for i in range(n):
        h2.set_state(0, i, saved[i][0], slot=0)
        h2.set_state(0, i, saved[i][1], slot=1)
    h2.set_step(0, t_saved)
    for t in range(4):
        g = gs.next()
        h2.step(0, xs, [torch.from_numpy(a).to(dev) for a in g], cc)
        o.step(g, hp)
    torch.cuda.synchronize()
    assert rel_err(to_np(cc), o.c) <= TOL
    for i in range(n):
        assert rel_err(to_np(xs[i]), o.xs[i]) <= TOL
        assert rel_err(to_np(h2.state(0, i, 1)), o.vs[i]) <= TOL
    with pytest.raises(EAError):
        ElasticAveraging([p], n).state(0, 0, 1)       # SGD has one state slot
    h2.close()


def test_bad_pointers_rejected_before_enqueue():
    n, p = 2, 1000
    h = ElasticAveraging([p], n)
    x = [torch.zeros(p + 4, device="cuda:0") for _ in range(n)]
    c = torch.zeros(p, device="cuda:0")
    with pytest.raises(EAError, match="EA_EINVAL"):
        h.step(0, [t[1:p + 1] for t in x], [t[:p] for t in x], c)     # 4-byte offset -> misaligned
    with pytest.raises(EAError, match="EA_EINVAL"):
        h.step(1, [t[:p] for t in x], [t[:p] for t in x], c)          # stage out of range
    with pytest.raises(ValueError, match="elements"):
        h.step(0, [t[:p - 4] for t in x], [t[:p] for t in x], c)      # undersized replica: never reaches the ABI
    with pytest.raises(ValueError, match="elements"):
        h.step(0, [t[:p] for t in x], [t[:p] for t in x], c[:p - 4])  # undersized center
    host = torch.zeros(p).pin_memory()
    import ctypes
    from paper_conf_ppopp_chen0qz23_b200 import binding
    lib = binding.load_library()
    arr = (ctypes.c_void_p * 2)(host.data_ptr(), host.data_ptr())
    st = lib.ea_step(h._h, 0, arr, arr, c.data_ptr(), None)
    assert st == binding.EA_EINVAL                                     # host memory is not device memory
    h.sync()
    h.close()


# ------------------------------------------------------------------ host-buffer path
@pytest.mark.parametrize("optimizer,n", [("sgd", 2), ("sgd", 4), ("adamw", 3), ("sgd", 12), ("asgd", 4)])
def test_step_many_host_pipelined(optimizer, n):
    """ea_step_many_host: gradients from pinned host memory in 4 Mi-element
    chunks (a 9,000,003-element stage spans 3 ragged chunks), centers copied
    back to host; must equal the oracle and the device-resident center."""
    sizes = [9_000_003, 1_000, 5] if n <= 4 else [4_500_001, 77]
    steps = 3
    lr = synth.LR if optimizer in ("sgd", "asgd") else 1e-3
    hp = hyper(n, "combined", lr=lr, wd=0.0 if optimizer == "sgd" else 1e-2)
    dev = torch.device("cuda:0")
    h = ElasticAveraging(sizes, n, alpha=hp.alpha, beta=hp.beta, rho=hp.rho, lr=hp.lr, momentum=hp.momentum,
                         weight_decay=hp.weight_decay, optimizer=optimizer, **asgd_kw(hp))
    oracle, gstreams, xs, cs, host_out = [], [], [], [], []
    for s, p in enumerate(sizes):
        reps, c = synth.host_state(n, p, seed=synth.WEIGHT_SEED + s)
        oracle.append(OracleStage(reps, c, optimizer))
        gstreams.append(synth.GradStream(n, p, seed=synth.GRAD_SEED + s))
        xs.append([torch.from_numpy(x).to(dev) for x in reps])
        cs.append(torch.from_numpy(c).to(dev))
        host_out.append(torch.empty(p, dtype=torch.float32).pin_memory())
    order = list(reversed(range(len(sizes))))
    stream = torch.cuda.Stream()
    for t in range(steps):
        hg = {}
        for s in range(len(sizes)):
            g = gstreams[s].next()
            hg[s] = [torch.from_numpy(a).pin_memory() for a in g]
            oracle[s].step(g, hp)
        h.step_many_host(order, [xs[s] for s in order], [hg[s] for s in order], [cs[s] for s in order],
                         [host_out[s] for s in order], stream=stream)
        stream.synchronize()
        for s in range(len(sizes)):
            assert torch.equal(host_out[s], cs[s].cpu()), "host copy of the center differs from the device center"
    for s, p in enumerate(sizes):
        o = oracle[s]
        assert rel_err(host_out[s].numpy(), o.c) <= TOL
        for i in range(n):
            assert rel_err(to_np(xs[s][i]), o.xs[i]) <= TOL
            assert rel_err(to_np(h.momentum(s, i)), o.ms[i]) <= TOL
        assert h.get_step(s) == steps
    with pytest.raises(TypeError):
        h.step_many_host([0], [xs[0]], [[a.to(dev) for a in hg[0]]], [cs[0]], [host_out[0]])
    h.close()


# ------------------------------------------------------------------ CUDA graphs
@pytest.mark.parametrize("optimizer", ["sgd", "adam", "adamw", "asgd"])
def test_step_many_captured_in_a_cuda_graph(optimizer):
    """ea_step_many is stream-ordered work only -- including Adam's step
    counter and bias corrections, which live on the device -- so a whole EA
    step can be captured once and replayed.  Replays must equal the oracle run
    step by step, and the step counter must count replays."""
    n, sizes, steps = 3, [100_003, 4096, 7], 6
    lr = synth.LR if optimizer in ("sgd", "asgd") else 1e-3
    hp = hyper(n, "combined", lr=lr, wd=0.0 if optimizer == "sgd" else 1e-2)
    dev = torch.device("cuda:0")
    h = ElasticAveraging(sizes, n, alpha=hp.alpha, beta=hp.beta, rho=hp.rho, lr=hp.lr, momentum=hp.momentum,
                         weight_decay=hp.weight_decay, optimizer=optimizer, **asgd_kw(hp))
    oracle, gstreams, xs, cs, gb = [], [], [], [], []
    for s, p in enumerate(sizes):
        reps, c = synth.host_state(n, p, seed=synth.WEIGHT_SEED + s)
        oracle.append(OracleStage(reps, c, optimizer))
        gstreams.append(synth.GradStream(n, p, seed=synth.GRAD_SEED + s))
        xs.append([torch.from_numpy(x).to(dev) for x in reps])
        cs.append(torch.from_numpy(c).to(dev))
        gb.append([torch.zeros(p, device=dev) for _ in range(n)])
    order = list(reversed(range(len(sizes))))
    graph = torch.cuda.CUDAGraph()
    side = torch.cuda.Stream()
    side.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(side):
        with torch.cuda.graph(graph, stream=side):
            h.step_many(order, [xs[s] for s in order], [gb[s] for s in order], [cs[s] for s in order], stream=side)
    torch.cuda.synchronize()
    for t in range(steps):
        for s in range(len(sizes)):
            g = gstreams[s].next()
            for i in range(n):
                gb[s][i].copy_(torch.from_numpy(g[i]))
            oracle[s].step(g, hp)
        graph.replay()
    torch.cuda.synchronize()
    for s in range(len(sizes)):
        assert rel_err(to_np(cs[s]), oracle[s].c) <= TOL
        for i in range(n):
            assert rel_err(to_np(xs[s][i]), oracle[s].xs[i]) <= TOL
            assert rel_err(to_np(h.state(s, i, 0)), oracle[s].ms[i]) <= TOL
            if optimizer in ("adam", "adamw"):
                assert rel_err(to_np(h.state(s, i, 1)), oracle[s].vs[i]) <= TOL
        if optimizer != "sgd":
            assert h.get_step(s) == steps          # device counter: replays, not the one capture
    h.close()
