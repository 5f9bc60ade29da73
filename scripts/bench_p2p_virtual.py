#!/usr/bin/env python
"""Single-GPU proxy measurement of the fused peer-memory spread step
(EA_XCHG_P2P, rows a4-a7): N ranks run as N handles on ONE B200, each on
its own stream, connected in-process, so every "peer" access is a local HBM
access.  It measures the fused kernel's on-device efficiency (the HBM side
of the exchange); it does not measure NVLink.

Bytes per rank per element (fp32, SGD): phase A reads x, g, m, x~ and writes
x, m and the pushed contribution (28 B); phase B (the 1/N owned chunks) reads
N contributions + x~ and writes x~ and the outbox (4 + 12/N B); phase C reads
the owners' outboxes and writes x~ for the other (N-1)/N chunks (8 (N-1)/N B):
40 + 4/N B.  On N GPUs the same kernel would move (N-1)/N * 4 B per element
out and in over NVLink per GPU.
"""
import argparse
import json
import os
import sys

os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")   # 2N streams of N virtual ranks (ea.h)

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C4")
    ap.add_argument("--n", type=int, default=None)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--exchange", default="p2p", choices=("p2p",))
    a = ap.parse_args()

    import torch
    from paper_conf_ppopp_chen0qz23_b200 import synth
    from paper_conf_ppopp_chen0qz23_b200.binding import ElasticAveraging

    cfg = synth.CONFIGS[a.config]
    n = a.n or cfg.n_pipelines
    sizes = cfg.stage_sizes
    dev = torch.device("cuda:0")
    al, be, rh = synth.mode_coeffs("combined", n)
    hs = [ElasticAveraging(sizes, n, alpha=al, beta=be, rho=rh, lr=synth.LR, momentum=synth.MOMENTUM,
                           layout="spread", rank=r, world=n, exchange="p2p") for r in range(n)]
    if n > 1:
        ElasticAveraging.p2p_connect(hs)
    streams = [torch.cuda.Stream() for _ in range(n)]
    state = []
    for s, p in enumerate(sizes):
        reps, c0, grads = synth.device_state(1, p, dev, seed=1000 * s)
        per_rank = []
        for r in range(n):
            cc = torch.zeros(hs[0].center_capacity(s), device=dev)
            cc[:p] = c0
            per_rank.append(([reps[0].clone()], [grads[0]], cc))
        state.append(per_rank)
    order = list(reversed(range(len(sizes))))

    def step():
        for s in order:
            for r in range(n):
                x, g, c = state[s][r]
                hs[r].step(s, x, g, c, stream=streams[r])

    for _ in range(a.warmup):
        step()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for st in streams:
        st.wait_event(e0)
    for _ in range(a.steps):
        step()
    for st in streams:
        ev = torch.cuda.Event()
        ev.record(st)
        torch.cuda.current_stream().wait_event(ev)
    e1.record()
    torch.cuda.synchronize()
    for r in range(n):
        hs[r].sync(streams[r])
    ms = e0.elapsed_time(e1) / a.steps
    P = sum(sizes)
    bytes_step = n * P * (40 + 4 / n)
    peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
    gbs = bytes_step / (ms * 1e-3) / 1e9
    print(json.dumps({"what": "fused peer-memory spread step, N virtual ranks on one GPU (HBM proxy, no NVLink)",
                      "workload": cfg.name, "n_ranks": n, "params": P, "ms_per_step": ms,
                      "replica_params_per_s": n * P / (ms * 1e-3), "hbm_bytes_per_step": bytes_step,
                      "achieved_gbs": gbs, "peak_gbs": peak, "frac": gbs / peak,
                      "nvlink_bytes_per_gpu_if_spread": 2 * (n - 1) / n * 4 * P}), flush=True)
    for h in hs:
        h.close()


if __name__ == "__main__":
    main()
