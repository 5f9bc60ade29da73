#!/usr/bin/env python
"""Reproduces, without compute-sanitizer, the peer-memory mismatch round 2 first saw only under racecheck: the test
harness built each step's gradients on the default stream and handed them to the library on another stream
without record_stream, so the caching allocator could give a gradient's block to the next step's gradient while
the (slow) push kernel still read it.  Here the library's stream is slowed by a sleep kernel instead of the
sanitizer: without record_stream the result differs from the oracle, with it the result matches.

    python scripts/probes/p2p_alloc_race_probe.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))


def run(record):
    import torch
    from paper_conf_ppopp_chen0qz23_b200 import synth
    from paper_conf_ppopp_chen0qz23_b200.binding import ElasticAveraging
    from tests._parity import TOL, OracleStage, hyper, rel_err, to_np
    n, sizes, steps = 1, [70_003, 17], 4
    hp = hyper(n, "combined")
    dev = torch.device("cuda:0")
    h = ElasticAveraging(sizes, n, alpha=hp.alpha, beta=hp.beta, rho=hp.rho, lr=hp.lr, momentum=hp.momentum,
                         layout="spread", rank=0, world=1, exchange="p2p")
    stream = torch.cuda.Stream()
    oracle, gstreams, xs, cs = [], [], [], []
    for s, p in enumerate(sizes):
        reps, c = synth.host_state(n, p, seed=synth.WEIGHT_SEED + s)
        oracle.append(OracleStage(reps, c))
        gstreams.append(synth.GradStream(n, p, seed=synth.GRAD_SEED + s))
        cc = torch.zeros(h.center_capacity(s), device=dev)
        cc[:p] = torch.from_numpy(c)
        cs.append(cc)
        xs.append(torch.from_numpy(reps[0]).to(dev))
    torch.cuda.synchronize()
    for t in range(steps):
        grads = {}
        for s in reversed(range(len(sizes))):
            g = gstreams[s].next()
            grads[s] = torch.from_numpy(g[0]).to(dev)       # default stream
            oracle[s].step(g, hp)
        torch.cuda.synchronize()
        for s in reversed(range(len(sizes))):
            with torch.cuda.stream(stream):
                torch.cuda._sleep(20_000_000)               # the library's stream runs ~10 ms late
            h.step(s, [xs[s]], [grads[s]], cs[s], stream=stream)
            if record:
                grads[s].record_stream(stream)
    h.sync(stream)
    torch.cuda.synchronize()
    errs = []
    for s, p in enumerate(sizes):
        errs.append(rel_err(to_np(xs[s]), oracle[s].xs[0]))
        errs.append(rel_err(to_np(cs[s][:p]), oracle[s].c))
    h.close()
    return max(errs), TOL


if __name__ == "__main__":
    for record in (False, True):
        e, tol = run(record)
        print(f"record_stream={record}: worst c13 {e:.3e} ({'PASS' if e <= tol else 'FAIL'} at {tol})", flush=True)
