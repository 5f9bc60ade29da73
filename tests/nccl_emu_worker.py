"""N spread ranks of the NCCL exchange on ONE GPU, through the library's own
ea_step (local kernel -> ncclReduceScatter -> spread_apply -> in-place
ncclAllGather on the side stream), with NCCL replaced by the in-process
emulation tests/nccl_emu/libnccl_emu.so (LD_PRELOAD; the parent test sets it).

Rank r is a host thread driving its own handle (rank r of world N, every
handle on cuda:0) and its own stream; the emulated collectives rendezvous the
threads exactly as NCCL rendezvouses processes.  After the run every rank's
replica, optimizer state and center are compared with the float64 oracle
(c13 metric), and every collective's arguments (from NCCL_EMU_LOG) are checked
against parallel.shard_bounds: reduce-scatter count = P_pad/N into a buffer of
that size, all-gather in place (recvbuff = the caller's center, sendbuff =
center + rank * P_pad/N).  Prints one JSON line.

    LD_PRELOAD=tests/nccl_emu/libnccl_emu.so NCCL_EMU_LOG=/tmp/log \
        python tests/nccl_emu_worker.py --world 4 [--optimizer sgd] [--staleness 0]
"""
import argparse
import json
import os
import sys
import threading

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--world", type=int, required=True)
    ap.add_argument("--optimizer", choices=("sgd", "adam", "adamw", "asgd"), default="sgd")
    ap.add_argument("--mode", default="combined")
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--sizes", default="1000000,1000003")
    ap.add_argument("--staleness", type=int, default=0)
    args = ap.parse_args()

    import numpy as np
    import torch

    from paper_conf_ppopp_chen0qz23_b200 import parallel, synth
    from paper_conf_ppopp_chen0qz23_b200.binding import ElasticAveraging, get_unique_id
    from tests._parity import OracleStage, asgd_kw, hyper, rel_err, to_np

    n = args.world
    sizes = [int(v) for v in args.sizes.split(",")]
    opt = args.optimizer
    lr = synth.LR if opt in ("sgd", "asgd") else 1e-3
    hp = hyper(n, args.mode, lr=lr, wd=0.0 if opt == "sgd" else 1e-2)
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    uid = get_unique_id()                      # the emulation's id (LD_PRELOAD)
    order = parallel.stage_order(len(sizes))

    oracle, gstreams = [], []
    init = []
    for s, p in enumerate(sizes):
        reps, c = synth.host_state(n, p, seed=synth.WEIGHT_SEED + s)
        oracle.append(OracleStage(reps, c, opt, staleness=args.staleness))
        gstreams.append(synth.GradStream(n, p, seed=synth.GRAD_SEED + s))
        init.append((reps, c))

    handles = [None] * n
    xs = [[None] * len(sizes) for _ in range(n)]
    cs = [[None] * len(sizes) for _ in range(n)]
    errors = []
    start = threading.Barrier(n + 1)
    done = threading.Barrier(n + 1)
    grads = {}

    def rank_main(r):
        try:
            torch.cuda.set_device(dev)
            h = ElasticAveraging(sizes, n, alpha=hp.alpha, beta=hp.beta, rho=hp.rho, lr=hp.lr,
                                 momentum=hp.momentum, weight_decay=hp.weight_decay, layout="spread", rank=r,
                                 world=n, device=0, nccl_id=uid, optimizer=opt, staleness=args.staleness,
                                 **asgd_kw(hp))
            handles[r] = h
            for s, p in enumerate(sizes):
                reps, c = init[s]
                cc = torch.zeros(h.center_capacity(s), device=dev)
                cc[:p] = torch.from_numpy(c)
                cs[r][s] = cc
                xs[r][s] = torch.from_numpy(reps[parallel.replica_of(r, s, n)]).to(dev)
            torch.cuda.synchronize()
            stream = torch.cuda.Stream(device=dev)
            for _ in range(args.steps):
                start.wait()
                for s in order:
                    h.step(s, [xs[r][s]], [grads[s][r]], cs[r][s], stream=stream)
                stream.synchronize()            # the local kernels are done with this step's gradients
                done.wait()
            h.sync(stream)
            stream.synchronize()
        except Exception as e:  # pragma: no cover
            errors.append((r, repr(e)))
            start.abort()
            done.abort()

    threads = [threading.Thread(target=rank_main, args=(r,)) for r in range(n)]
    for t in threads:
        t.start()
    try:
        for _ in range(args.steps):
            for s in order:
                g = gstreams[s].next()
                oracle[s].step(g, hp)
                grads[s] = [torch.from_numpy(g[parallel.replica_of(r, s, n)]).to(dev) for r in range(n)]
            torch.cuda.synchronize()
            start.wait()
            done.wait()
    except threading.BrokenBarrierError:
        pass
    for t in threads:
        t.join()
    if errors:
        print(json.dumps({"world": n, "error": errors}))
        return
    torch.cuda.synchronize()

    worst = {"x": 0.0, "state": 0.0, "center": 0.0}
    pad_ok = True
    for r in range(n):
        h = handles[r]
        for s, p in enumerate(sizes):
            i = parallel.replica_of(r, s, n)
            o = oracle[s]
            worst["x"] = max(worst["x"], rel_err(to_np(xs[r][s]), o.xs[i]))
            worst["state"] = max(worst["state"], rel_err(to_np(h.state(s, 0, 0)), o.ms[i]))
            worst["center"] = max(worst["center"], rel_err(to_np(cs[r][s][:p]), o.c))
            pad_ok = pad_ok and bool(torch.all(cs[r][s][p:] == 0))

    # every collective's arguments, in issue order per rank
    checks = {"rs": 0, "ag": 0, "bad": []}
    log = os.environ.get("NCCL_EMU_LOG")
    if log and os.path.exists(log):
        per_rank = {r: [] for r in range(n)}
        for line in open(log):
            op, rank, world, send, recv, count, dtype = line.split()
            if op in ("RS", "AG") and int(world) == n:
                per_rank[int(rank)].append((op, int(send, 16), int(recv, 16), int(count)))
        chunks = 1 if args.staleness else int(os.environ.get("AVGPIPE_EA_SPREAD_CHUNKS", "1") or 1)

        def pieces(p_pad):
            """The library's cut of a stage into pieces of whole 32N-float blocks (ea_api.cu spread_step)."""
            q = 32 * n
            L = (-(-p_pad // chunks) + q - 1) // q * q
            return [(off, min(L, p_pad - off)) for off in range(0, p_pad, L)]

        for r in range(n):
            h = handles[r]
            seq = per_rank[r]
            want = [(kind, s, off, ln) for _ in range(args.steps) for s in order
                    for off, ln in pieces(h.center_capacity(s)) for kind in ("RS", "AG")]
            if len(seq) != len(want):
                checks["bad"].append(f"rank {r}: {len(seq)} calls, expected {len(want)}")
                continue
            for (op, send, recv, count), (kind, s, off, ln) in zip(seq, want):
                p_pad = h.center_capacity(s)
                if chunks == 1:
                    lo, hi = parallel.shard_bounds(p_pad, n, r)
                    ok = op == kind and count == hi - lo == h.shard_elems(s)
                else:     # piece [off, off + ln): rank r owns its block r
                    lo, hi = off + r * (ln // n), off + (r + 1) * (ln // n)
                    ok = op == kind and count == ln // n
                center = cs[r][s].data_ptr()
                if kind == "AG":
                    ok = ok and recv == center + 4 * off and send == center + 4 * lo     # in place, own block
                    checks["ag"] += 1
                else:
                    ok = ok and recv != center and send != center          # library scratch
                    checks["rs"] += 1
                if not ok:
                    checks["bad"].append(f"rank {r} stage {s} {op}: send {send:#x} recv {recv:#x} count {count}")
                    break
    for h in handles:
        h.close()
    print(json.dumps({"world": n, "optimizer": opt, "staleness": args.staleness, "steps": args.steps,
                      "chunks": int(os.environ.get("AVGPIPE_EA_SPREAD_CHUNKS", "1") or 1),
                      "max_err": max(worst.values()), "worst": worst, "padding_zero": pad_ok,
                      "collectives": checks}))


if __name__ == "__main__":
    main()
