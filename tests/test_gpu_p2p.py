"""Fused peer-memory spread exchange (EA_XCHG_P2P; rows a4-a7 in one kernel).

N ranks as N handles on ONE GPU (connected in-process with ea_p2p_connect,
each driving its own stream, sharing the device's SMs): the same kernel code
as on N GPUs, with the peer pointers pointing at the other handles' exchange
buffers.  Compared with the float64 oracle at N (the oracle is layout-
agnostic), c13 <= 1e-5, after every rank's steps; plus the timeout path.
"""
import os
import subprocess
import sys

import pytest
import torch

from paper_conf_ppopp_chen0qz23_b200 import synth
from paper_conf_ppopp_chen0qz23_b200.binding import EAError, ElasticAveraging
from paper_conf_ppopp_chen0qz23_b200.parallel import replica_of
from tests._parity import TOL, OracleStage, asgd_kw, hyper, rel_err, to_np

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(n, sizes, steps, mode, optimizer="sgd", stage_order=None):
    lr = synth.LR if optimizer in ("sgd", "asgd") else 1e-3
    hp = hyper(n, mode, lr=lr, wd=0.0 if optimizer == "sgd" else 1e-2)
    dev = torch.device("cuda:0")
    hs = [ElasticAveraging(sizes, n, alpha=hp.alpha, beta=hp.beta, rho=hp.rho, lr=hp.lr, momentum=hp.momentum,
                           weight_decay=hp.weight_decay, layout="spread", rank=r, world=n, optimizer=optimizer,
                           exchange="p2p", **asgd_kw(hp)) for r in range(n)]
    if n > 1:
        ElasticAveraging.p2p_connect(hs)
    streams = [torch.cuda.Stream() for _ in range(n)]
    oracle, gstreams, xs, centers = [], [], [], []
    for s, p in enumerate(sizes):
        reps, c = synth.host_state(n, p, seed=synth.WEIGHT_SEED + s)
        oracle.append(OracleStage(reps, c, optimizer))
        gstreams.append(synth.GradStream(n, p, seed=synth.GRAD_SEED + s))
        cap = hs[0].center_capacity(s)
        cs = []
        for r in range(n):
            cc = torch.zeros(cap, device=dev)
            cc[:p] = torch.from_numpy(c)
            cs.append(cc)
        centers.append(cs)
        xs.append([torch.from_numpy(reps[replica_of(r, s, n)]).to(dev) for r in range(n)])
    order = stage_order or list(reversed(range(len(sizes))))
    torch.cuda.synchronize()
    for t in range(steps):
        grads = {}
        for s in order:
            g = gstreams[s].next()
            grads[s] = [torch.from_numpy(g[replica_of(r, s, n)]).to(dev) for r in range(n)]
            oracle[s].step(g, hp)
        torch.cuda.synchronize()
        for s in order:                  # every rank issues its stages in the same global order
            for r in range(n):
                hs[r].step(s, [xs[s][r]], [grads[s][r]], centers[s][r], stream=streams[r])
                # the gradient was allocated on the default stream and is read on streams[r]: without this the
                # caching allocator may hand its block to the next step's gradient, whose copy (default stream)
                # then overwrites it while this step's push still reads it (seen under compute-sanitizer racecheck,
                # which slows the kernels enough to expose it: profiles/r02_sanitizers.md)
                grads[s][r].record_stream(streams[r])
    for r in range(n):
        hs[r].sync(streams[r])
    torch.cuda.synchronize()
    for s, p in enumerate(sizes):
        o = oracle[s]
        for r in range(n):
            i = replica_of(r, s, n)
            assert rel_err(to_np(xs[s][r]), o.xs[i]) <= TOL, (s, r)
            assert rel_err(to_np(hs[r].momentum(s, 0)), o.ms[i]) <= TOL, (s, r)
            assert rel_err(to_np(centers[s][r][:p]), o.c) <= TOL, (s, r)
            assert torch.all(centers[s][r][p:] == 0)
    for h in hs:
        h.close()


@pytest.mark.parametrize("n", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("mode", synth.MODES)
def test_p2p_exchange_matches_oracle(n, mode):
    _run(n, [200_003, 64, 1_000_000], 10, mode)


@pytest.mark.parametrize("n,optimizer", [(2, "adam"), (4, "adamw"), (3, "asgd")])
def test_p2p_exchange_adam(n, optimizer):
    _run(n, [300_001, 17], 12, "combined", optimizer)


@pytest.mark.parametrize("n,mode", [(2, m) for m in synth.MODES] + [(4, m) for m in synth.MODES] + [(8, "combined")])
def test_p2p_exchange_c1_100_steps(n, mode):
    """The north-star gate in the spread layout: C1 sizes + the 1,000,003 tail stage, 100 steps, N = 2/4/8."""
    _run(n, [1_000_000, 1_000_003], 100, mode)


_TIMEOUT_SCRIPT = r'''
import os, sys, torch
sys.path.insert(0, sys.argv[1])
os.environ["AVGPIPE_EA_P2P_TIMEOUT_MS"] = "1500"
from paper_conf_ppopp_chen0qz23_b200.binding import ElasticAveraging, EAError
hs = [ElasticAveraging([100_000], 2, layout="spread", rank=r, world=2, exchange="p2p") for r in range(2)]
ElasticAveraging.p2p_connect(hs)
x = torch.zeros(100_000, device="cuda:0"); c = torch.zeros(hs[0].center_capacity(0), device="cuda:0")
hs[0].step(0, [x], [x], c)          # rank 1 never steps: rank 0 must time out, not hang
torch.cuda.synchronize()
try:
    hs[0].sync()
    print("NO ERROR")
except EAError as e:
    print("TIMEOUT REPORTED", e)
'''


def test_p2p_missing_rank_times_out_instead_of_hanging():
    out = subprocess.run([sys.executable, "-c", _TIMEOUT_SCRIPT, ROOT], capture_output=True, text=True, timeout=120)
    assert "TIMEOUT REPORTED" in out.stdout, out.stdout + out.stderr


def _ipc_worker(rank, world, port, q):
    """One rank in its own process on cuda:0: IPC handles through gloo, then
    the fused exchange against the other process (time-sliced on one GPU)."""
    import numpy as np  # noqa: F401
    import torch.distributed as dist
    os.environ["AVGPIPE_EA_P2P_TIMEOUT_MS"] = "60000"
    try:
        dist.init_process_group("gloo", init_method=port, rank=rank, world_size=world)
        from paper_conf_ppopp_chen0qz23_b200.parallel import connect_p2p
        n, sizes, steps = world, [100_003, 70], 5
        hp = hyper(n, "combined")
        dev = torch.device("cuda:0")
        h = ElasticAveraging(sizes, n, alpha=hp.alpha, beta=hp.beta, rho=hp.rho, lr=hp.lr, momentum=hp.momentum,
                             layout="spread", rank=rank, world=n, exchange="p2p")
        connect_p2p(h)
        oracle, gstreams, xs, cs = [], [], [], []
        for s, p in enumerate(sizes):
            reps, c = synth.host_state(n, p, seed=synth.WEIGHT_SEED + s)
            oracle.append(OracleStage(reps, c))
            gstreams.append(synth.GradStream(n, p, seed=synth.GRAD_SEED + s))
            cc = torch.zeros(h.center_capacity(s), device=dev)
            cc[:p] = torch.from_numpy(c)
            cs.append(cc)
            xs.append(torch.from_numpy(reps[replica_of(rank, s, n)]).to(dev))
        for t in range(steps):
            for s in reversed(range(len(sizes))):
                g = gstreams[s].next()
                oracle[s].step(g, hp)
                h.step(s, [xs[s]], [torch.from_numpy(g[replica_of(rank, s, n)]).to(dev)], cs[s])
        h.sync()
        torch.cuda.synchronize()
        for s, p in enumerate(sizes):
            i = replica_of(rank, s, n)
            assert rel_err(to_np(xs[s]), oracle[s].xs[i]) <= TOL
            assert rel_err(to_np(cs[s][:p]), oracle[s].c) <= TOL
        h.close()
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover
        q.put((rank, repr(e)))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


def test_p2p_exchange_across_processes_via_cuda_ipc():
    """The multi-process path (cudaIpcGetMemHandle -> all-gather -> cudaIpcOpenMemHandle,
    system-scope release/acquire across processes) with 2 processes on one GPU."""
    import tempfile
    import torch.multiprocessing as mp
    port = "file://" + os.path.join(tempfile.mkdtemp(prefix="gloo_"), "store")   # no TCP port race
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_ipc_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in range(2))
    for p in procs:
        p.join(timeout=120)
    assert all(v == "ok" for v in res.values()), res
