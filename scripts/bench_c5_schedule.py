#!/usr/bin/env python
"""C5 harness (rows a8 + a9): the elastic-averaging step
of the spread layout overlapped with a synthetic advance-forward iteration.

Every rank hosts one replica of each of the K stages (replica i of stage s on
rank (i+s) mod N, the north-star spread layout) and runs, per iteration, the
micro-batch ops of its K stages in the order `ea_schedule(K, M, k, a_k)` gives
(Alg. 1; a_k = min(M, K-k+e), reading c15), interleaved op by op across the
hosted stages.  F = forward GEMMs of 6 GPT-2-XL layers (hidden 1600, QKV,
proj, 4h MLP), B = their dgrad + wgrad GEMMs, bf16 on tensor cores (cuBLAS:
the compute is a stand-in, not the product).  Right after a stage's last B
the stage's EA step is issued through the public API (`ea_step`: local kernel
on the compute stream, reduce-scatter -> owner update -> all-gather on the
library's side stream); `ea_sync` only at the end of the iteration.

Reports, as CUDA-event time per iteration (max over ranks):
  t_compute  the schedule alone,
  t_ea       the EA steps alone (all K stages + ea_sync),
  t_overlap  schedule with the EA steps issued after each stage's last B,
  exposed    t_overlap - t_compute  (vs t_ea if run serially).

    python scripts/bench_c5_schedule.py [--tokens 1024] [--micro 8] [--extra 1]
    torchrun --nproc-per-node 8 scripts/bench_c5_schedule.py        (N = 8, C5)
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C5")
    ap.add_argument("--tokens", type=int, default=1024, help="tokens per micro-batch")
    ap.add_argument("--micro", type=int, default=8, help="M micro-batches per iteration (Fig. 7 scale)")
    ap.add_argument("--extra", type=int, default=1, help="extra advance e: a_k = min(M, K-k+e)")
    ap.add_argument("--layers", type=int, default=6)
    ap.add_argument("--iters", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=2)
    a = ap.parse_args()

    import torch
    import torch.distributed as dist
    from paper_conf_ppopp_chen0qz23_b200 import parallel, synth
    from paper_conf_ppopp_chen0qz23_b200.binding import ElasticAveraging, schedule

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ.setdefault("MASTER_PORT", "29541")
    os.environ.setdefault("RANK", str(rank))
    os.environ.setdefault("WORLD_SIZE", str(world))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist.init_process_group("nccl", device_id=dev)
    cfg = synth.CONFIGS[a.config]
    sizes = cfg.stage_sizes
    K, M, n = len(sizes), a.micro, world
    al, be, rh = synth.mode_coeffs("combined", n)
    h = ElasticAveraging(sizes, n, alpha=al, beta=be, rho=rh, lr=synth.LR, momentum=synth.MOMENTUM,
                         layout="spread", rank=rank, world=world, device=local,
                         nccl_id=parallel.broadcast_unique_id())
    state = []
    for s, p in enumerate(sizes):
        reps, c0, grads = synth.device_state(1, p, dev, seed=1000 * s)
        cc = torch.zeros(h.center_capacity(s), device=dev)
        cc[:p] = c0
        state.append((reps, grads, cc))

    # synthetic stage compute: GPT-2-XL layer shapes, bf16
    hd = 1600
    shapes = [(hd, 3 * hd), (hd, hd), (hd, 4 * hd), (4 * hd, hd)]
    ws = [[torch.randn(i, o, device=dev, dtype=torch.bfloat16) * 0.02 for (i, o) in shapes]
          for _ in range(a.layers)]
    acts = {i: torch.randn(a.tokens, i, device=dev, dtype=torch.bfloat16) for (i, _) in shapes}
    gout = {o: torch.randn(a.tokens, o, device=dev, dtype=torch.bfloat16) for (_, o) in shapes}

    def fwd():
        for layer in ws:
            for (i, o), w in zip(shapes, layer):
                torch.matmul(acts[i], w)

    def bwd():
        for layer in ws:
            for (i, o), w in zip(shapes, layer):
                torch.matmul(gout[o], w.t())
                torch.matmul(acts[i].t(), gout[o])

    flops_mb = sum(2 * a.tokens * i * o for (i, o) in shapes) * a.layers   # one forward of one stage

    # the K stages this rank hosts: stage s of pipeline (rank - s) mod N; pipeline position k = s (0-based)
    advances = [min(M, K - 1 - s + a.extra) for s in range(K)]
    ops = [schedule(K, M, s, advances[s]) for s in range(K)]
    last_b = [max(j for j, (kind, _) in enumerate(ops[s]) if kind == "B") for s in range(K)]
    order = parallel.stage_order(K)
    stream = torch.cuda.current_stream(dev)

    def iteration(with_ea: bool, with_compute: bool = True):
        if with_compute:
            for j in range(2 * M):                    # op j of every hosted stage in turn
                for s in order:
                    kind, _ = ops[s][j]
                    fwd() if kind == "F" else bwd()
                    if with_ea and j == last_b[s]:    # the stage's last backward is done
                        reps, grads, cc = state[s]
                        h.step(s, reps, grads, cc, stream=stream)
        elif with_ea:
            for s in order:
                reps, grads, cc = state[s]
                h.step(s, reps, grads, cc, stream=stream)
        if with_ea:
            h.sync(stream)

    def timed(fn):
        for _ in range(a.warmup):
            fn()
        torch.cuda.synchronize()
        dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(a.iters):
            fn()
        e1.record(stream)
        torch.cuda.synchronize()
        t = torch.tensor([e0.elapsed_time(e1) / a.iters], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    t_comp = timed(lambda: iteration(False))
    t_ea = timed(lambda: iteration(True, with_compute=False))
    t_ovl = timed(lambda: iteration(True))
    out = {"what": "C5 harness: spread-layout EA steps issued after each stage's last backward in ea_schedule order",
           "workload": cfg.name, "n_gpus": world, "n_pipelines": n, "stages": K, "micro_batches": M,
           "advances": advances, "tokens_per_micro_batch": a.tokens, "layers_per_stage": a.layers,
           "t_compute_ms": t_comp, "t_ea_ms": t_ea, "t_overlap_ms": t_ovl, "exposed_ea_ms": t_ovl - t_comp,
           "exposed_fraction_of_ea": (t_ovl - t_comp) / t_ea,
           "compute_tflops": 3 * flops_mb * K * M / (t_comp * 1e-3) / 1e12,
           "ea_local_hbm_bytes": sum(28 * p for p in sizes)}
    if rank == 0:
        print(json.dumps(out), flush=True)
    h.close()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
