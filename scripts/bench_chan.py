#!/usr/bin/env python
"""Activation channel (ea_chan_*) between two processes: one-way bandwidth for large messages and ping-pong
latency for small ones, timed with CUDA events on the device (two processes sharing cuda:0 here; the same calls
map NVLink peers on a multi-GPU node).

    python scripts/bench_chan.py
"""
import json
import os
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def worker(rank, port, q):
    os.environ["CUDA_MODULE_LOADING"] = "EAGER"
    import torch
    import torch.distributed as dist
    from paper_conf_ppopp_chen0qz23_b200.binding import Channel
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", init_method=port, rank=rank, world_size=2)
    out = []
    s = torch.cuda.Stream()
    # one-way bandwidth: rank 0 sends `reps` messages of `nbytes`, rank 1 times their arrival
    for nbytes in (1 << 20, 16 << 20, 64 << 20):
        reps, slots = 20, 4
        ch = Channel("send" if rank == 0 else "recv", nbytes, slots)
        hs = [None, None]
        dist.all_gather_object(hs, ch.export())
        ch.connect(hs[1 - rank])
        buf = torch.empty(nbytes // 4, device="cuda")
        torch.cuda.synchronize()
        dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            if rank == 1:
                ch.recv(buf, stream=s)           # first message: start the clock when it has arrived
                e0.record(s)
                for _ in range(reps):
                    ch.recv(buf, stream=s)
                e1.record(s)
            else:
                for _ in range(reps + 1):
                    ch.send(buf, stream=s)
        s.synchronize()
        if rank == 1:
            ms = e0.elapsed_time(e1)
            out.append({"what": "one-way bandwidth", "bytes": nbytes, "messages": reps, "ms": ms,
                        "gbs": nbytes * reps / (ms * 1e-3) / 1e9})
        dist.barrier()
        ch.close()
    # ping-pong latency: 4 KB each way, rank 0 times round trips
    nbytes, reps = 4096, 200
    fwd = Channel("send" if rank == 0 else "recv", nbytes, 2)
    bwd = Channel("recv" if rank == 0 else "send", nbytes, 2)
    hs = [None, None]
    dist.all_gather_object(hs, (fwd.export(), bwd.export()))
    fwd.connect(hs[1 - rank][0])
    bwd.connect(hs[1 - rank][1])
    buf = torch.zeros(nbytes // 4, device="cuda")
    torch.cuda.synchronize()
    dist.barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        if rank == 0:
            e0.record(s)
            for _ in range(reps):
                fwd.send(buf, stream=s)
                bwd.recv(buf, stream=s)
            e1.record(s)
        else:
            for _ in range(reps):
                fwd.recv(buf, stream=s)
                bwd.send(buf, stream=s)
    s.synchronize()
    if rank == 0:
        out.append({"what": "ping-pong round trip", "bytes": nbytes, "round_trips": reps,
                    "us_per_round_trip": e0.elapsed_time(e1) * 1e3 / reps})
    dist.barrier()
    fwd.close()
    bwd.close()
    dist.destroy_process_group()
    q.put((rank, out))


def main():
    import torch.multiprocessing as mp
    port = "file://" + os.path.join(tempfile.mkdtemp(prefix="gloo_"), "store")
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=worker, args=(r, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in range(2))
    for p in procs:
        p.join(timeout=60)
    for r in (0, 1):
        for d in res[r]:
            d["note"] = "two processes sharing one B200 (CUDA IPC of the same device)"
            print(json.dumps(d))


if __name__ == "__main__":
    main()
