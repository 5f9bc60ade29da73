"""Full-size parity on sampled outputs (the oracle is elementwise over j, so it
can compute any sample of elements one by one).

* C2 (BASELINE configs[1]: 25M params, K=4, N=4) in bench.py's launch
  configuration (ea_step_many, default kernel): 3 steps, 200k sampled
  elements per stage plus the first/last elements, checked after every step.
* A stage larger than 2^31 elements (int64 indexing) with N=1 and N=2.
"""
import numpy as np
import pytest
import torch

from oracle.ea_oracle import Hyper, ea_step, ea_step_adam
from paper_conf_ppopp_chen0qz23_b200 import synth
from paper_conf_ppopp_chen0qz23_b200.binding import ElasticAveraging
from tests._parity import TOL, OracleStage, asgd_kw, hyper, rel_err

pytestmark = pytest.mark.gpu


def _sample_idx(p, k, rng):
    idx = rng.choice(p, size=min(k, p), replace=False)
    edge = np.r_[np.arange(min(8, p)), np.arange(max(p - 8, 0), p)]
    return torch.from_numpy(np.unique(np.r_[idx, edge]).astype(np.int64))


def _run_sampled(n, sizes, steps, variant, mode="combined", many=True, k=200_000, optimizer="sgd"):
    dev = torch.device("cuda:0")
    a, b, r = synth.mode_coeffs(mode, n)
    lr = synth.LR if optimizer == "sgd" else 1e-3
    hp = hyper(n, mode, lr=lr, wd=0.0 if optimizer == "sgd" else 1e-2)
    h = ElasticAveraging(sizes, n, alpha=a, beta=b, rho=r, lr=lr, momentum=synth.MOMENTUM,
                         weight_decay=0.0 if optimizer == "sgd" else 1e-2, kernel_variant=variant, optimizer=optimizer)
    gen = torch.Generator(device=dev)
    gen.manual_seed(7)
    rng = np.random.default_rng(0)
    state = []
    for s, p in enumerate(sizes):
        reps, c, grads = synth.device_state(n, p, dev, seed=s)
        state.append((reps, c, grads, _sample_idx(p, k, rng).to(dev)))
    order = list(reversed(range(len(sizes))))
    f64 = lambda t, idx: t[idx].double().cpu().numpy()
    for t in range(steps):
        before = []
        for s, (reps, c, grads, idx) in enumerate(state):
            for g in grads:
                g.normal_(0.0, synth.GRAD_STD, generator=gen)
            vs = [f64(h.state(s, i, 1), idx) for i in range(n)] if optimizer != "sgd" else None
            before.append(([f64(x, idx) for x in reps], [f64(h.momentum(s, i), idx) for i in range(n)],
                           f64(c, idx), [f64(g, idx) for g in grads], vs))
        if many:
            h.step_many(order, [state[s][0] for s in order], [state[s][2] for s in order],
                        [state[s][1] for s in order])
        else:
            for s in order:
                h.step(s, state[s][0], state[s][2], state[s][1])
        torch.cuda.synchronize()
        for s, (reps, c, grads, idx) in enumerate(state):
            xs, ms, cc, gs, vs = before[s]
            if optimizer == "sgd":
                ox, om, oc = ea_step(xs, ms, cc, gs, hp)
            else:
                ox, om, ov, oc = ea_step_adam(xs, ms, vs, cc, gs, hp, t + 1, decoupled=optimizer == "adamw")
                for i in range(n):
                    assert rel_err(f64(h.state(s, i, 1), idx), ov[i]) <= TOL, (s, t, i)
            assert rel_err(f64(c, idx), oc) <= TOL, (s, t)
            for i in range(n):
                assert rel_err(f64(reps[i], idx), ox[i]) <= TOL, (s, t, i)
                assert rel_err(f64(h.momentum(s, i), idx), om[i]) <= TOL, (s, t, i)
    h.close()


def _run_trajectory(n, sizes, steps, optimizer, mode="combined", k=100_000, graph=True, checkpoints=(1, 10, 50)):
    """100-step ACCUMULATED parity at full size: the oracle evolves only the sampled elements (the update is
    elementwise over j), from the same initial state and with the same gradients gathered at those indices every
    step; the GPU runs the whole stages exactly as bench.py times them (ea_step_many, default kernel, replayed as
    one captured CUDA graph).  Compared at the checkpoints and after the last step (c13 <= 1e-5)."""
    dev = torch.device("cuda:0")
    lr = 1e-3 if optimizer in ("adam", "adamw") else synth.LR
    hp = hyper(n, mode, lr=lr, wd=0.0 if optimizer == "sgd" else 1e-2)
    h = ElasticAveraging(sizes, n, alpha=hp.alpha, beta=hp.beta, rho=hp.rho, lr=hp.lr, momentum=hp.momentum,
                         weight_decay=hp.weight_decay, optimizer=optimizer, betas=(hp.beta1, hp.beta2), eps=hp.eps,
                         **asgd_kw(hp))
    gen = torch.Generator(device=dev)
    gen.manual_seed(11)
    rng = np.random.default_rng(1)
    state, oracle = [], []
    f64 = lambda t_, idx: t_[idx].double().cpu().numpy()
    for s, p in enumerate(sizes):
        reps, c, grads = synth.device_state(n, p, dev, seed=s)
        idx = _sample_idx(p, k, rng).to(dev)
        state.append((reps, c, grads, idx))
        oracle.append(OracleStage([f64(x, idx) for x in reps], f64(c, idx), optimizer))
    order = list(reversed(range(len(sizes))))
    run = lambda st=None: h.step_many(order, [state[s][0] for s in order], [state[s][2] for s in order],
                                      [state[s][1] for s in order], stream=st)
    if graph:
        g = torch.cuda.CUDAGraph()
        side = torch.cuda.Stream()
        side.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(side):
            with torch.cuda.graph(g, stream=side):
                run(side)
        torch.cuda.synchronize()
        run = g.replay
    worst = 0.0
    for t in range(1, steps + 1):
        for s, (reps, c, grads, idx) in enumerate(state):
            for gr in grads:
                gr.normal_(0.0, synth.GRAD_STD, generator=gen)
            oracle[s].step([f64(gr, idx) for gr in grads], hp)
        run()
        if t in checkpoints or t == steps:
            torch.cuda.synchronize()
            for s, (reps, c, grads, idx) in enumerate(state):
                o = oracle[s]
                errs = [rel_err(f64(c, idx), o.c)]
                for i in range(n):
                    errs.append(rel_err(f64(reps[i], idx), o.xs[i]))
                    errs.append(rel_err(f64(h.state(s, i, 0), idx), o.ms[i]))
                    if optimizer in ("adam", "adamw"):
                        errs.append(rel_err(f64(h.state(s, i, 1), idx), o.vs[i]))
                worst = max(worst, max(errs))
                assert max(errs) <= TOL, (optimizer, t, s, max(errs))
    h.close()
    return worst


@pytest.mark.parametrize("optimizer", ["sgd", "adam", "adamw", "asgd"])
def test_c2_full_size_100_steps_accumulated(optimizer):
    """The north-star gate at the bench's full size: C2 (25 M params, K=4, N=4), 100 steps, sampled."""
    cfg = synth.CONFIGS["C2"]
    _run_trajectory(cfg.n_pipelines, cfg.stage_sizes, 100, optimizer)


def test_c4_stage_100_steps_accumulated():
    """One C4-sized stage (44.4 M params) co-located with N = 8 (the 1-GPU point of the C4 curve), 100 steps."""
    cfg = synth.CONFIGS["C4"]
    _run_trajectory(8, cfg.stage_sizes[:1], 100, "sgd", k=50_000)


@pytest.mark.parametrize("variant", ["auto", "regloop", "laneshfl", "bulkpipe"])
def test_c2_full_size_sampled(variant):
    cfg = synth.CONFIGS["C2"]
    _run_sampled(cfg.n_pipelines, cfg.stage_sizes, 3, variant)


@pytest.mark.parametrize("optimizer", ["adam", "adamw"])
def test_c2_full_size_sampled_adam(optimizer):
    cfg = synth.CONFIGS["C2"]
    _run_sampled(cfg.n_pipelines, cfg.stage_sizes, 3, "auto", optimizer=optimizer)


def test_c2_full_size_per_stage_launches():
    cfg = synth.CONFIGS["C2"]
    _run_sampled(cfg.n_pipelines, cfg.stage_sizes, 2, "auto", many=False)


@pytest.mark.parametrize("n,p", [(1, (1 << 31) + 5), (2, (1 << 30) + 3)])
def test_beyond_int32_elements(n, p):
    free, _ = torch.cuda.mem_get_info()
    need = (3 * n + 1) * 4 * p * 1.2
    if free < need:
        pytest.skip(f"needs {need / 1e9:.0f} GB")
    _run_sampled(n, [p], 1, "auto", k=100_000)
    torch.cuda.empty_cache()


def _run_spread_sampled(n, sizes, steps, exchange, optimizer="sgd", k=200_000):
    """Spread layout at full stage sizes, in bench.py's launch configuration (ea_step per stage in the global
    order K-1..0, ea_sync per step): world 1 over NCCL, or N virtual ranks on this GPU with the fused P2P
    kernel.  Sampled elements of every rank's replica, optimizer state and center against the oracle."""
    from paper_conf_ppopp_chen0qz23_b200.binding import get_unique_id
    from paper_conf_ppopp_chen0qz23_b200.parallel import replica_of, stage_order
    dev = torch.device("cuda:0")
    lr = synth.LR if optimizer == "sgd" else 1e-3
    hp = hyper(n, "combined", lr=lr, wd=0.0 if optimizer == "sgd" else 1e-2)
    kw = dict(alpha=hp.alpha, beta=hp.beta, rho=hp.rho, lr=hp.lr, momentum=hp.momentum,
              weight_decay=hp.weight_decay, layout="spread", world=n, optimizer=optimizer, exchange=exchange)
    if n == 1:
        hs = [ElasticAveraging(sizes, 1, rank=0, nccl_id=get_unique_id() if exchange == "nccl" else None, **kw)]
    else:
        hs = [ElasticAveraging(sizes, n, rank=r, **kw) for r in range(n)]
        ElasticAveraging.p2p_connect(hs)
    streams = [torch.cuda.Stream() for _ in range(n)]
    gen = torch.Generator(device=dev)
    gen.manual_seed(11)
    rng = np.random.default_rng(1)
    state = []
    for s, p in enumerate(sizes):
        reps, c, grads = synth.device_state(n, p, dev, seed=100 + s)
        cap = hs[0].center_capacity(s)
        centers = []
        for r in range(n):
            cc = torch.zeros(cap, device=dev)
            cc[:p] = c
            centers.append(cc)
        del c
        # rank r hosts replica replica_of(r, s, n): keep the replicas indexed by rank
        xs = [reps[replica_of(r, s, n)] for r in range(n)]
        gs = [grads[replica_of(r, s, n)] for r in range(n)]
        state.append((xs, gs, centers, _sample_idx(p, k, rng).to(dev)))
    order = stage_order(len(sizes))
    f64 = lambda t, idx: t[idx].double().cpu().numpy()
    for t in range(steps):
        before = []
        for s, (xs, gs, centers, idx) in enumerate(state):
            for g in gs:
                g.normal_(0.0, synth.GRAD_STD, generator=gen)
            vs = [f64(hs[r].state(s, 0, 1), idx) for r in range(n)] if optimizer != "sgd" else None
            before.append(([f64(x, idx) for x in xs], [f64(hs[r].momentum(s, 0), idx) for r in range(n)],
                           f64(centers[0], idx), [f64(g, idx) for g in gs], vs))
        torch.cuda.synchronize()
        for s in order:
            xs, gs, centers, _ = state[s]
            for r in range(n):
                hs[r].step(s, [xs[r]], [gs[r]], centers[r], stream=streams[r])
        for r in range(n):
            hs[r].sync(streams[r])
        torch.cuda.synchronize()
        for s, (xs, gs, centers, idx) in enumerate(state):
            bx, bm, bc, bg, bv = before[s]
            if optimizer == "sgd":
                ox, om, oc = ea_step(bx, bm, bc, bg, hp)
            else:
                ox, om, ov, oc = ea_step_adam(bx, bm, bv, bc, bg, hp, t + 1, decoupled=optimizer == "adamw")
            for r in range(n):
                assert rel_err(f64(centers[r], idx), oc) <= TOL, (s, t, r)
                assert rel_err(f64(xs[r], idx), ox[r]) <= TOL, (s, t, r)
                assert rel_err(f64(hs[r].momentum(s, 0), idx), om[r]) <= TOL, (s, t, r)
                if optimizer != "sgd":
                    assert rel_err(f64(hs[r].state(s, 0, 1), idx), ov[r]) <= TOL, (s, t, r)
    for h in hs:
        h.close()


@pytest.mark.parametrize("optimizer", ["sgd", "adamw"])
def test_c4_stages_spread_nccl_world1_sampled(optimizer):
    """Two C4-sized stages (44,375,000 elements each) through the NCCL spread path at world 1."""
    cfg = synth.CONFIGS["C4"]
    _run_spread_sampled(1, cfg.stage_sizes[:2], 2, "nccl", optimizer)


def test_c4_stage_p2p_8_virtual_ranks_sampled():
    """One C4-sized stage, 8 virtual ranks, the fused P2P exchange (the bench's N=8 kernel at full size)."""
    cfg = synth.CONFIGS["C4"]
    _run_spread_sampled(8, cfg.stage_sizes[:1], 2, "p2p")
