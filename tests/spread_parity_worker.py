"""Multi-rank parity of the spread layout under torchrun (north-star gate:
"spread at N = 2, 4 and 8 under torchrun", C1 sizes + the 1,000,003 tail
stage, 100 steps): one process per GPU, each rank hosts replica
(rank - s) mod N of every stage, drives the real exchange (NCCL reduce-scatter
-> shard update -> all-gather, or the fused P2P kernel) and compares its
replica, optimizer state and center with the float64 oracle after the run
(c13 metric); the max error over ranks is printed by rank 0 as one JSON line.

    torchrun --nproc-per-node N tests/spread_parity_worker.py --exchange nccl|p2p

AVGPIPE_BENCH_SHARED_GPU=1 (tests on a one-GPU box) puts every rank on cuda:0
with a gloo control group and the P2P exchange over CUDA IPC (NCCL refuses two
ranks on one device).
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--exchange", choices=("nccl", "p2p"), default="nccl")
    ap.add_argument("--optimizer", choices=("sgd", "adam", "adamw", "asgd"), default="sgd")
    ap.add_argument("--mode", default="combined")
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--sizes", default="1000000,1000003")
    args = ap.parse_args()

    import torch
    import torch.distributed as dist

    from paper_conf_ppopp_chen0qz23_b200 import parallel, synth
    from paper_conf_ppopp_chen0qz23_b200.binding import ElasticAveraging
    from tests._parity import OracleStage, asgd_kw, hyper, rel_err, to_np

    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    shared = os.environ.get("AVGPIPE_BENCH_SHARED_GPU") == "1"
    if shared:
        local = 0
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if shared:
        if args.exchange != "p2p" and world > 1:
            raise SystemExit("shared-GPU mode needs --exchange p2p")
        dist.init_process_group("gloo")
        uid = None
    else:
        dist.init_process_group("nccl", device_id=dev)
        uid = parallel.broadcast_unique_id()
    n = world
    sizes = [int(v) for v in args.sizes.split(",")]
    opt = args.optimizer
    lr = synth.LR if opt in ("sgd", "asgd") else 1e-3
    hp = hyper(n, args.mode, lr=lr, wd=0.0 if opt == "sgd" else 1e-2)
    h = ElasticAveraging(sizes, n, alpha=hp.alpha, beta=hp.beta, rho=hp.rho, lr=hp.lr, momentum=hp.momentum,
                         weight_decay=hp.weight_decay, layout="spread", rank=rank, world=world, device=local,
                         nccl_id=uid, optimizer=opt, exchange=args.exchange, **asgd_kw(hp))
    if shared and world > 1:
        parallel.connect_p2p(h)
    oracle, gstreams, xs, cs = [], [], [], []
    for s, p in enumerate(sizes):
        reps, c = synth.host_state(n, p, seed=synth.WEIGHT_SEED + s)       # every rank draws the same state
        oracle.append(OracleStage(reps, c, opt))
        gstreams.append(synth.GradStream(n, p, seed=synth.GRAD_SEED + s))
        cc = torch.zeros(h.center_capacity(s), device=dev)
        cc[:p] = torch.from_numpy(c)
        cs.append(cc)
        xs.append(torch.from_numpy(reps[parallel.replica_of(rank, s, n)]).to(dev))
    order = parallel.stage_order(len(sizes))
    for _ in range(args.steps):
        for s in order:
            g = gstreams[s].next()
            oracle[s].step(g, hp)
            gd = torch.from_numpy(g[parallel.replica_of(rank, s, n)]).to(dev)
            h.step(s, [xs[s]], [gd], cs[s])
        h.sync()
    torch.cuda.synchronize()
    worst = 0.0
    for s, p in enumerate(sizes):
        o, i = oracle[s], parallel.replica_of(rank, s, n)
        errs = [rel_err(to_np(xs[s]), o.xs[i]), rel_err(to_np(h.state(s, 0, 0)), o.ms[i]),
                rel_err(to_np(cs[s][:p]), o.c)]
        if opt in ("adam", "adamw"):
            errs.append(rel_err(to_np(h.state(s, 0, 1)), o.vs[i]))
        if not bool(torch.all(cs[s][p:] == 0)):
            errs.append(float("inf"))                                     # padding must stay zero
        worst = max(worst, max(errs))
    t = torch.tensor([worst], dtype=torch.float64, device=dev if not shared else "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    h.close()
    if rank == 0:
        print(json.dumps({"world": world, "exchange": args.exchange, "optimizer": opt, "mode": args.mode,
                          "steps": args.steps, "sizes": sizes, "max_rel_err": float(t.item())}), flush=True)
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
