"""Spread-layout host logic at world_size 2 (and 4) over gloo on CPU.

The kernels cannot run here; the local / shard phases are injected from the
oracle so that what is tested is the product's orchestration
(paper_conf_ppopp_chen0qz23_b200.parallel): placement, padding, shard
bounds, collective calls and stage order.  The composition must equal the
co-located oracle step (the oracle is layout-agnostic).
"""
import os
import tempfile

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle.ea_oracle import Hyper, ea_step, local_update
from paper_conf_ppopp_chen0qz23_b200 import parallel, synth


def _free_port():
    """A fresh file:// rendezvous (no TCP port to race for between tests)."""
    d = tempfile.mkdtemp(prefix="gloo_")
    return "file://" + os.path.join(d, "store")


def test_placement_is_a_latin_square():
    for n in (1, 2, 3, 4, 8):
        for k in (1, 2, 4, 8):
            for s in range(k):
                reps = [parallel.replica_of(r, s, n) for r in range(n)]
                assert sorted(reps) == list(range(n))         # N distinct ranks per stage
                for r in range(n):
                    assert parallel.rank_of(parallel.replica_of(r, s, n), s, n) == r


def test_padding_and_shards():
    for n in (1, 2, 3, 8):
        for p in (1, 31, 32, 1000, 44_375_000):
            pad = parallel.padded_size(p, n)
            assert pad >= p and pad % (32 * n) == 0 and pad - p < 32 * n
            bounds = [parallel.shard_bounds(pad, n, r) for r in range(n)]
            assert bounds[0][0] == 0 and bounds[-1][1] == pad
            assert all(b[1] == c[0] for b, c in zip(bounds, bounds[1:]))
            assert all((hi - lo) % 32 == 0 for lo, hi in bounds)    # 128-byte aligned shards
    assert parallel.stage_order(4) == [3, 2, 1, 0]


def _worker(rank, world, port, q):
    dist.init_process_group("gloo", init_method=port, rank=rank, world_size=world)
    try:
        n = world
        a, b, r = synth.mode_coeffs("combined", n)
        hp = Hyper(alpha=a, beta=b, rho=r, lr=0.05, momentum=0.9)
        sizes = [1001, 70]
        # unique-id bootstrap (fake 128-byte id; NCCL needs a GPU)
        uid = parallel.broadcast_unique_id(make_id=lambda: bytes(range(128)))
        assert uid == bytes(range(128))
        mom = {}

        def local_fn(stage, x, g, center, contrib):
            p = x.numel()
            xv, gv, cv = x.double().numpy(), g.double().numpy(), center[:p].double().numpy()
            m = mom.get(stage, np.zeros(p))
            delta, m_new = local_update(xv, m, gv, hp)
            mom[stage] = m_new
            contrib.zero_()
            contrib[:p] = torch.from_numpy(hp.rho * delta + hp.beta * (xv - cv))
            x.copy_(torch.from_numpy((1 - hp.alpha) * xv + hp.alpha * cv + delta))

        def apply_fn(stage, shard, reduced):
            shard.add_(reduced / n)

        drv = parallel.CollectiveSpread(local_fn=local_fn, apply_fn=apply_fn)
        states, centers, oracle = {}, {}, {}
        for s, p in enumerate(sizes):
            reps, c = synth.host_state(n, p, seed=7 + s)
            reps = [x.astype(np.float64) for x in reps]
            c = c.astype(np.float64)
            oracle[s] = (reps, [np.zeros(p)] * n, c)
            states[s] = torch.from_numpy(reps[parallel.replica_of(rank, s, n)].copy())
            cc = torch.zeros(parallel.padded_size(p, n), dtype=torch.float64)
            cc[:p] = torch.from_numpy(c)
            centers[s] = cc
        rng = np.random.default_rng(3)
        for t in range(6):
            for s in parallel.stage_order(len(sizes)):
                p = sizes[s]
                g = [rng.normal(0, 1e-2, p) for _ in range(n)]
                drv.step(s, states[s], torch.from_numpy(g[parallel.replica_of(rank, s, n)]), centers[s])
                oracle[s] = ea_step(*oracle[s], g, hp)
        for s, p in enumerate(sizes):
            xs, _, c = oracle[s]
            np.testing.assert_allclose(states[s].numpy(), xs[parallel.replica_of(rank, s, n)], rtol=1e-12,
                                       atol=1e-15)
            np.testing.assert_allclose(centers[s][:p].numpy(), c, rtol=1e-12, atol=1e-15)
            assert torch.all(centers[s][p:] == 0)
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
def test_collective_spread_matches_colocated_oracle(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    results = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert all(v == "ok" for v in results.values()), results
