#!/usr/bin/env python
"""Live pipeline runtime (row f2) end to end: K = 2 stages as 2 processes sharing cuda:0, N = 2 parallel
pipelines run concurrently, M micro-batches in Algorithm 1's order, one fused elastic-averaging step per stage and
iteration on its own stream.  Iteration time (host wall clock between synchronised iterations, median) with the
activations over gloo (host-staged) vs the library's activation channels (transport "ipc").

    python scripts/bench_pipeline.py [--hidden 2048] [--tokens 2048] [--layers 4] [--m 8] [--iters 6]
"""
import argparse
import json
import os
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
K, N = 2, 2


def worker(rank, port, q, transport, a):
    if transport == "ipc":
        os.environ["CUDA_MODULE_LOADING"] = "EAGER"
    import torch
    import torch.distributed as dist
    from paper_conf_ppopp_chen0qz23_b200.binding import ElasticAveraging
    from paper_conf_ppopp_chen0qz23_b200.pipeline import PipelineStage
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    dist.init_process_group("gloo", init_method=port, rank=rank, world_size=K)
    torch.manual_seed(1)
    mods = []
    for _ in range(N):
        layers = []
        for _ in range(a.layers):
            layers += [torch.nn.Linear(a.hidden, a.hidden), torch.nn.GELU()]
        mods.append(torch.nn.Sequential(*layers).to(dev))
    flats = []
    for m in mods:
        params = list(m.parameters())
        n = sum(p.numel() for p in params)
        flat, gflat = torch.empty(n, device=dev), torch.zeros(n, device=dev)
        off = 0
        for p in params:
            k = p.numel()
            flat[off:off + k].copy_(p.data.reshape(-1))
            p.data = flat[off:off + k].view_as(p)
            p.grad = gflat[off:off + k].view_as(p)
            off += k
        flats.append((flat, gflat))
    P = flats[0][0].numel()
    center = flats[0][0].clone()
    ea = ElasticAveraging([P], N, beta=1.0, rho=1.0, lr=1e-3, momentum=0.9, device=0)
    act = (a.tokens, a.hidden)
    st = PipelineStage(mods, rank, K, a.m, ea=ea, ea_stage=0, center=center, flat_params=[f for f, _ in flats],
                       flat_grads=[g for _, g in flats], concurrent=True, transport=transport,
                       act_bytes=a.tokens * a.hidden * 4, device=dev)
    g = torch.Generator(device="cuda").manual_seed(5)
    xs = [[torch.randn(act, device=dev, generator=g) for _ in range(a.m)] for _ in range(N)]
    ys = [[torch.randn(act, device=dev, generator=g) for _ in range(a.m)] for _ in range(N)]
    times = []
    for it in range(a.iters):
        dist.barrier()
        t0 = time.perf_counter()
        st.run_iteration(inputs=xs if rank == 0 else None, targets=ys if rank == K - 1 else None,
                         loss_fn=torch.nn.functional.mse_loss, act_shape=act, act_dtype=torch.float32, device=dev,
                         zero_grads=True, sync=True)
        dist.barrier()
        times.append(time.perf_counter() - t0)
    st.close()
    ea.close()
    dist.destroy_process_group()
    q.put((rank, times))


def main():
    import torch.multiprocessing as mp
    ap = argparse.ArgumentParser()
    ap.add_argument("--hidden", type=int, default=2048)
    ap.add_argument("--tokens", type=int, default=2048)
    ap.add_argument("--layers", type=int, default=4)
    ap.add_argument("--m", type=int, default=8)
    ap.add_argument("--iters", type=int, default=6)
    a = ap.parse_args()
    for transport in ("dist", "ipc"):
        port = "file://" + os.path.join(tempfile.mkdtemp(prefix="gloo_"), "store")
        ctx = mp.get_context("spawn")
        q = ctx.Queue()
        procs = [ctx.Process(target=worker, args=(r, port, q, transport, a)) for r in range(K)]
        for p in procs:
            p.start()
        res = dict(q.get(timeout=900) for _ in range(K))
        for p in procs:
            p.join(timeout=60)
        t = sorted(res[0][2:])          # drop 2 warm-up iterations
        med = t[len(t) // 2]
        print(json.dumps({"what": "pipeline iteration", "transport": "gloo (host-staged)" if transport == "dist"
                          else "ipc (ea_chan: copy engine + stream memory ops)", "K": K, "N": N, "M": a.m,
                          "hidden": a.hidden, "tokens_per_microbatch": a.tokens, "layers_per_stage": a.layers,
                          "activation_bytes": a.tokens * a.hidden * 4, "median_s": med, "all_s": res[0],
                          "note": "2 stage processes time-sharing one B200"}), flush=True)


if __name__ == "__main__":
    main()
