"""Randomised parity sweep (fixed seeds, so it is reproducible): random N,
stage counts and sizes (tiny, ragged, multi-tile), hyper-parameters across
their valid ranges, optimizer, kernel variant and call form (ea_step per
stage / ea_step_many / ea_step_many_host), a few steps each, against the
float64 oracle with the c13 gate."""
import numpy as np
import pytest
import torch

from paper_conf_ppopp_chen0qz23_b200 import synth
from paper_conf_ppopp_chen0qz23_b200.binding import ElasticAveraging
from tests._parity import TOL, OracleStage, f32, rel_err, to_np
from oracle.ea_oracle import Hyper

pytestmark = pytest.mark.gpu


def _case(seed):
    rng = np.random.default_rng(seed)
    n = int(rng.choice([1, 2, 3, 4, 5, 6, 7, 8, 9, 12, 16]))
    k = int(rng.integers(1, 11))
    sizes = [int(rng.choice([1, 3, 4, 17, 255, 4096, 70_001, int(rng.integers(1, 300_000))])) for _ in range(k)]
    opt = str(rng.choice(["sgd", "sgd", "adam", "adamw"]))
    nesterov = bool(rng.integers(0, 2)) and opt == "sgd"
    momentum = float(rng.uniform(0.0, 0.99)) if opt == "sgd" else 0.0
    if nesterov and momentum == 0.0:
        momentum = 0.5
    hp = dict(alpha=float(rng.uniform(0, 1)), beta=float(rng.uniform(0, 2)), rho=float(rng.uniform(0, 1.5)),
              lr=float(rng.uniform(1e-3, 0.1)) if opt == "sgd" else float(rng.uniform(1e-4, 3e-3)),
              momentum=momentum, weight_decay=float(rng.choice([0.0, 1e-4, 1e-2])), nesterov=nesterov,
              betas=(float(rng.uniform(0.8, 0.95)), float(rng.uniform(0.99, 0.9999))), eps=1e-8)
    variant = str(rng.choice(["auto", "auto", "regloop", "laneshfl", "bulkpipe"]))
    form = str(rng.choice(["step", "many", "host"]))
    return n, sizes, opt, hp, variant, form


@pytest.mark.parametrize("seed", range(120))
def test_random_configuration(seed):
    n, sizes, opt, hp, variant, form = _case(seed)
    dev = torch.device("cuda:0")
    h = ElasticAveraging(sizes, n, alpha=hp["alpha"], beta=hp["beta"], rho=hp["rho"], lr=hp["lr"],
                         momentum=hp["momentum"], weight_decay=hp["weight_decay"], nesterov=hp["nesterov"],
                         kernel_variant=variant, optimizer=opt, betas=hp["betas"], eps=hp["eps"])
    ohp = Hyper(alpha=f32(hp["alpha"]), beta=f32(hp["beta"]), rho=f32(hp["rho"]), lr=f32(hp["lr"]),
                momentum=f32(hp["momentum"]), weight_decay=f32(hp["weight_decay"]), nesterov=hp["nesterov"],
                beta1=hp["betas"][0], beta2=hp["betas"][1], eps=f32(hp["eps"]))
    oracle, gstreams, xs, cs, outs = [], [], [], [], []
    for s, p in enumerate(sizes):
        reps, c = synth.host_state(n, p, seed=1000 * seed + s)
        oracle.append(OracleStage(reps, c, opt))
        gstreams.append(synth.GradStream(n, p, seed=1000 * seed + 500 + s))
        xs.append([torch.from_numpy(x).to(dev) for x in reps])
        cs.append(torch.from_numpy(c).to(dev))
        outs.append(torch.empty(p, dtype=torch.float32).pin_memory())
    order = list(reversed(range(len(sizes))))
    for t in range(3):
        gh = {}
        for s in range(len(sizes)):
            g = gstreams[s].next()
            oracle[s].step(g, ohp)
            gh[s] = [torch.from_numpy(a) for a in g]
        if form == "step":
            for s in order:
                h.step(s, xs[s], [a.to(dev) for a in gh[s]], cs[s])
        elif form == "many":
            h.step_many(order, [xs[s] for s in order], [[a.to(dev) for a in gh[s]] for s in order],
                        [cs[s] for s in order])
        else:
            h.step_many_host(order, [xs[s] for s in order], [[a.pin_memory() for a in gh[s]] for s in order],
                             [cs[s] for s in order], [outs[s] for s in order])
        torch.cuda.synchronize()
    for s, p in enumerate(sizes):
        o = oracle[s]
        assert rel_err(to_np(cs[s]), o.c) <= TOL, (seed, s)
        for i in range(n):
            assert rel_err(to_np(xs[s][i]), o.xs[i]) <= TOL, (seed, s, i)
            assert rel_err(to_np(h.state(s, i, 0)), o.ms[i]) <= TOL, (seed, s, i)
            if opt != "sgd":
                assert rel_err(to_np(h.state(s, i, 1)), o.vs[i]) <= TOL, (seed, s, i)
        if form == "host":
            assert torch.equal(outs[s], cs[s].cpu())
    h.close()
