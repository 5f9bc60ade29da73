"""Stale center in the spread layout at world 1 (real NCCL), the stale center's
checkpoint slot and CUDA-graph guard, and checkpoint/resume of the peer-memory
exchange (ea_set_step must not disturb the exchange's epoch).
Every result is compared with the float64 oracle (c13 <= 1e-5)."""
import numpy as np
import pytest
import torch

from paper_conf_ppopp_chen0qz23_b200 import synth
from paper_conf_ppopp_chen0qz23_b200.binding import SLOT_CENTER_PREV, EAError, ElasticAveraging, get_unique_id
from paper_conf_ppopp_chen0qz23_b200.parallel import replica_of
from tests._parity import TOL, OracleStage, asgd_kw, hyper, rel_err, to_np

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda:0")


@pytest.mark.parametrize("optimizer", ["sgd", "adamw", "asgd"])
def test_stale_spread_world1_real_nccl(optimizer):
    """Row f4 in EA_SPREAD through the real NCCL (world 1) from a non-default stream, 60 steps."""
    sizes = [100_003, 5, 4096]
    lr = 1e-3 if optimizer == "adamw" else synth.LR
    hp = hyper(1, "combined", lr=lr, wd=0.0 if optimizer == "sgd" else 1e-2)
    h = ElasticAveraging(sizes, 1, alpha=hp.alpha, beta=hp.beta, rho=hp.rho, lr=hp.lr, momentum=hp.momentum,
                         weight_decay=hp.weight_decay, layout="spread", rank=0, world=1, nccl_id=get_unique_id(),
                         optimizer=optimizer, staleness=1, **asgd_kw(hp))
    stream = torch.cuda.Stream()
    oracle, gstreams, xs, cs = [], [], [], []
    for s, p in enumerate(sizes):
        reps, c = synth.host_state(1, p, seed=synth.WEIGHT_SEED + s)
        oracle.append(OracleStage(reps, c, optimizer, staleness=1))
        gstreams.append(synth.GradStream(1, p, seed=synth.GRAD_SEED + s))
        cc = torch.zeros(h.center_capacity(s), device=DEV)
        cc[:p] = torch.from_numpy(c)
        cs.append(cc)
        xs.append(torch.from_numpy(reps[0]).to(DEV))
    torch.cuda.synchronize()
    for t in range(60):
        for s in reversed(range(len(sizes))):
            g = gstreams[s].next()
            gd = torch.from_numpy(g[0]).to(DEV)
            torch.cuda.synchronize()
            h.step(s, [xs[s]], [gd], cs[s], stream=stream)
            gd.record_stream(stream)     # allocated on the default stream, read on `stream` (see test_gpu_p2p._run)
            oracle[s].step(g, hp)
        stream.synchronize()
    h.sync(stream)
    stream.synchronize()
    for s, p in enumerate(sizes):
        o = oracle[s]
        assert rel_err(to_np(xs[s]), o.xs[0]) <= TOL
        assert rel_err(to_np(cs[s][:p]), o.c) <= TOL
        assert rel_err(to_np(h.state(s, 0, 0)), o.ms[0]) <= TOL
        assert rel_err(to_np(h.state(s, 0, SLOT_CENTER_PREV)), o.c_prev) <= TOL   # x~_{t-1} after the run
        assert torch.all(cs[s][p:] == 0)
    h.close()


def test_stale_first_step_refused_under_graph_capture_and_prev_slot_resume():
    """The x~_{-1} := x~_0 initialisation is not captured (it would replay every step, i.e. staleness 0):
    the first step of a stale stage inside a capture is EA_ESTATE; once x~_{-1} is set through the
    EA_SLOT_CENTER_PREV slot, capture works, and graph replays follow the stale oracle -- which also makes
    the slot a checkpoint of x~_{t-1}: a resumed handle equals the uninterrupted run."""
    n, p = 3, 60_001
    hp = hyper(n, "combined")
    reps, c = synth.host_state(n, p)
    o = OracleStage(reps, c, staleness=1)
    gs = synth.GradStream(n, p)
    xs = [torch.from_numpy(x).to(DEV) for x in reps]
    cc = torch.from_numpy(c).to(DEV)
    gb = [torch.zeros(p, device=DEV) for _ in range(n)]
    kw = dict(alpha=hp.alpha, beta=hp.beta, rho=hp.rho, lr=hp.lr, momentum=hp.momentum, staleness=1)
    h = ElasticAveraging([p], n, **kw)
    side = torch.cuda.Stream()
    side.wait_stream(torch.cuda.current_stream())
    graph = torch.cuda.CUDAGraph()
    with pytest.raises(EAError, match="EA_ESTATE"):
        with torch.cuda.stream(side):
            with torch.cuda.graph(graph, stream=side):
                h.step(0, xs, gb, cc, stream=side)
    torch.cuda.synchronize()
    # eager steps, then checkpoint (x, x~, momentum, x~_{t-1}) and resume in a fresh handle under a graph
    for t in range(4):
        g = gs.next()
        for i in range(n):
            gb[i].copy_(torch.from_numpy(g[i]))
        h.step(0, xs, gb, cc)
        o.step(g, hp)
    torch.cuda.synchronize()
    saved_m = [h.state(0, i, 0).clone() for i in range(n)]
    saved_prev = h.state(0, 0, SLOT_CENTER_PREV).clone()
    assert rel_err(to_np(saved_prev), o.c_prev) <= TOL
    h.close()
    h2 = ElasticAveraging([p], n, **kw)
    for i in range(n):
        h2.set_state(0, i, saved_m[i])
    h2.set_state(0, 0, saved_prev, slot=SLOT_CENTER_PREV)
    torch.cuda.synchronize()
    graph = torch.cuda.CUDAGraph()
    side.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(side):
        with torch.cuda.graph(graph, stream=side):
            h2.step(0, xs, gb, cc, stream=side)
    torch.cuda.synchronize()
    for t in range(5):
        g = gs.next()
        for i in range(n):
            gb[i].copy_(torch.from_numpy(g[i]))
        o.step(g, hp)
        graph.replay()
    torch.cuda.synchronize()
    assert rel_err(to_np(cc), o.c) <= TOL
    assert rel_err(to_np(h2.state(0, 0, SLOT_CENTER_PREV)), o.c_prev) <= TOL
    for i in range(n):
        assert rel_err(to_np(xs[i]), o.xs[i]) <= TOL
        assert rel_err(to_np(h2.state(0, i, 0)), o.ms[i]) <= TOL
    with pytest.raises(EAError):
        ElasticAveraging([p], n).state(0, 0, SLOT_CENTER_PREV)      # no stale center without staleness 1
    h2.close()


def test_stale_rejected_with_p2p_exchange():
    with pytest.raises(EAError, match="EA_EINVAL"):
        ElasticAveraging([1000], 2, layout="spread", rank=0, world=2, exchange="p2p", staleness=1)


@pytest.mark.parametrize("optimizer", ["sgd", "adam"])
def test_p2p_checkpoint_resume_with_set_step(optimizer):
    """EA_XCHG_P2P, 2 virtual ranks: run 4 steps, checkpoint (replicas, centers, optimizer state, step count),
    resume 4 more steps in FRESH handles with ea_set_step(t).  The exchange keeps its own epoch, so the resumed
    handles neither wait for arrivals that never come nor consume stale inboxes; the result equals the oracle's
    uninterrupted 8 steps.  Also: set_step on a live handle between steps leaves the exchange intact."""
    n, sizes = 2, [70_003, 19]
    lr = 1e-3 if optimizer == "adam" else synth.LR
    hp = hyper(n, "combined", lr=lr, wd=0.0 if optimizer == "sgd" else 1e-2)
    kw = dict(alpha=hp.alpha, beta=hp.beta, rho=hp.rho, lr=hp.lr, momentum=hp.momentum,
              weight_decay=hp.weight_decay, layout="spread", world=n, exchange="p2p", optimizer=optimizer)

    def make():
        hs = [ElasticAveraging(sizes, n, rank=r, **kw) for r in range(n)]
        ElasticAveraging.p2p_connect(hs)
        return hs

    oracle, gstreams, xs, cs = [], [], [], []
    hs = make()
    for s, p in enumerate(sizes):
        reps, c = synth.host_state(n, p, seed=synth.WEIGHT_SEED + s)
        oracle.append(OracleStage(reps, c, optimizer))
        gstreams.append(synth.GradStream(n, p, seed=synth.GRAD_SEED + s))
        per = []
        for r in range(n):
            cc = torch.zeros(hs[0].center_capacity(s), device=DEV)
            cc[:p] = torch.from_numpy(c)
            per.append(cc)
        cs.append(per)
        xs.append([torch.from_numpy(reps[replica_of(r, s, n)]).to(DEV) for r in range(n)])
    streams = [torch.cuda.Stream() for _ in range(n)]

    def run(handles, steps, poke_step=False):
        for t in range(steps):
            grads = {}
            for s in reversed(range(len(sizes))):
                g = gstreams[s].next()
                oracle[s].step(g, hp)
                grads[s] = [torch.from_numpy(g[replica_of(r, s, n)]).to(DEV) for r in range(n)]
            torch.cuda.synchronize()
            for s in reversed(range(len(sizes))):
                for r in range(n):
                    handles[r].step(s, [xs[s][r]], [grads[s][r]], cs[s][r], stream=streams[r])
            for r in range(n):
                handles[r].sync(streams[r])
            torch.cuda.synchronize()
            if poke_step:
                for r in range(n):
                    for s in range(len(sizes)):
                        handles[r].set_step(s, handles[r].get_step(s))   # a no-op for the optimizer

    run(hs, 4, poke_step=True)
    slots = 2 if optimizer == "adam" else 1
    saved = [[[hs[r].state(s, 0, k).clone() for k in range(slots)] for s in range(len(sizes))] for r in range(n)]
    steps = [[hs[r].get_step(s) for s in range(len(sizes))] for r in range(n)]
    assert all(v == 4 for row in steps for v in row)
    for h in hs:
        h.close()
    hs = make()
    for r in range(n):
        for s in range(len(sizes)):
            for k in range(slots):
                hs[r].set_state(s, 0, saved[r][s][k], slot=k)
            hs[r].set_step(s, steps[r][s])
    run(hs, 4)
    for s, p in enumerate(sizes):
        o = oracle[s]
        for r in range(n):
            i = replica_of(r, s, n)
            assert rel_err(to_np(xs[s][r]), o.xs[i]) <= TOL, (s, r)
            assert rel_err(to_np(cs[s][r][:p]), o.c) <= TOL, (s, r)
            assert rel_err(to_np(hs[r].state(s, 0, 0)), o.ms[i]) <= TOL, (s, r)
    for h in hs:
        h.close()
