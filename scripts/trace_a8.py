#!/usr/bin/env python
"""Row a8 evidence on one B200: does the elastic-averaging exchange stay off the
critical path?  ("in an asynchronous manner ... to prevent the
inter-process communication blocking the pipeline".)

One iteration of a synthetic pipeline stage set on this GPU, spread layout:
    for s = K-1 .. 0:  backward GEMMs of stage s  ->  ea_step(s)
    for s = 0 .. K-1:  forward GEMMs of stage s (the next iteration's forward)
    ea_sync
ea_step(s) puts the local kernel (x_i, optimizer state, contribution) on the
compute stream and the exchange (NCCL reduce-scatter -> shard update ->
all-gather, or the peer-memory p2p_exchange kernel) on the library's side
stream; the compute stream never waits for the exchange.  The stage compute
is GPT-2-medium-shaped bf16 GEMMs (cuBLAS: a stand-in for the model, not the
product).  At world 1 the exchange's collectives are local copies, so this
measures scheduling -- whether the side-stream work runs concurrently with the
compute stream's kernels -- not NVLink.

Reported (CUDA events, median of --iters):
  t_compute      the GEMMs alone
  t_ea           the K ea_steps + ea_sync alone
  t_overlap      both, interleaved as above
  exposed        t_overlap - t_compute
  local_sum      sum of the local kernels' durations (from the trace): the part of
                 the EA step that is on the compute stream by design
and, from a torch.profiler (CUPTI) trace of one iteration -- the image has no
nsys -- every kernel's stream, start and duration: the fraction of side-stream
kernel time that ran while a compute-stream kernel was running.

    python scripts/trace_a8.py --exchange nccl|p2p [--staleness 1] [--config C4] [--out trace.json]
"""
import argparse
import json
import os
import statistics
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def overlap_stats(kernels, main_stream):
    """kernels: [(stream, name, t0, t1)] in us.  Fraction of side-stream busy time covered by main-stream busy."""
    def merge(iv):
        iv = sorted(iv)
        out = []
        for a, b in iv:
            if out and a <= out[-1][1]:
                out[-1][1] = max(out[-1][1], b)
            else:
                out.append([a, b])
        return out

    main = merge([(t0, t1) for s, _, t0, t1 in kernels if s == main_stream])
    side = merge([(t0, t1) for s, _, t0, t1 in kernels if s != main_stream])
    side_total = sum(b - a for a, b in side)
    cov = 0.0
    j = 0
    for a, b in side:
        for c, d in main:
            lo, hi = max(a, c), min(b, d)
            if hi > lo:
                cov += hi - lo
    return {"side_busy_us": side_total, "side_covered_by_compute_us": cov,
            "side_overlap_fraction": cov / side_total if side_total else None,
            "main_busy_us": sum(b - a for a, b in main)}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C4")
    ap.add_argument("--exchange", choices=("nccl", "p2p"), default="nccl")
    ap.add_argument("--staleness", type=int, default=0)
    ap.add_argument("--tokens", type=int, default=8192, help="tokens of one stage backward (GEMM M dimension)")
    ap.add_argument("--layers", type=int, default=3, help="transformer layers per stage (GPT-2-medium: 24/8)")
    ap.add_argument("--iters", type=int, default=7)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--out", default=None, help="write the per-kernel timeline of the traced iteration (JSON)")
    a = ap.parse_args()

    import torch
    from paper_conf_ppopp_chen0qz23_b200 import synth
    from paper_conf_ppopp_chen0qz23_b200.binding import ElasticAveraging, get_unique_id

    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    cfg = synth.CONFIGS[a.config]
    sizes = cfg.stage_sizes
    K = len(sizes)
    al, be, rh = synth.mode_coeffs("combined", 1)
    h = ElasticAveraging(sizes, 1, alpha=al, beta=be, rho=rh, lr=synth.LR, momentum=synth.MOMENTUM,
                         layout="spread", rank=0, world=1, device=0,
                         nccl_id=get_unique_id() if a.exchange == "nccl" else None, exchange=a.exchange,
                         staleness=a.staleness)
    state = []
    for s, p in enumerate(sizes):
        reps, c0, grads = synth.device_state(1, p, dev, seed=1000 * s)
        cc = torch.zeros(h.center_capacity(s), device=dev)
        cc[:p] = c0
        state.append((reps, grads, cc))

    hd = 1024  # GPT-2 medium
    shapes = [(hd, 3 * hd), (hd, hd), (hd, 4 * hd), (4 * hd, hd)]
    ws = [[torch.randn(i, o, device=dev, dtype=torch.bfloat16) * 0.02 for (i, o) in shapes]
          for _ in range(a.layers)]
    acts = {i: torch.randn(a.tokens, i, device=dev, dtype=torch.bfloat16) for (i, _) in shapes}
    gout = {o: torch.randn(a.tokens, o, device=dev, dtype=torch.bfloat16) for (_, o) in shapes}
    stream = torch.cuda.current_stream(dev)

    def fwd():
        for layer in ws:
            for (i, o), w in zip(shapes, layer):
                torch.matmul(acts[i], w)

    def bwd():
        for layer in ws:
            for (i, o), w in zip(shapes, layer):
                torch.matmul(gout[o], w.t())
                torch.matmul(acts[i].t(), gout[o])

    def iteration(with_ea=True, with_compute=True):
        for s in reversed(range(K)):
            if with_compute:
                bwd()
            if with_ea:
                reps, grads, cc = state[s]
                h.step(s, reps, grads, cc, stream=stream)
        if with_compute:
            for s in range(K):
                fwd()
        if with_ea:
            h.sync(stream)

    def timed(fn):
        for _ in range(a.warmup):
            fn()
        torch.cuda.synchronize()
        ts = []
        for _ in range(a.iters):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            fn()
            e1.record(stream)
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        return statistics.median(ts)

    t_comp = timed(lambda: iteration(False, True))
    t_ea = timed(lambda: iteration(True, False))
    t_ovl = timed(lambda: iteration(True, True))

    # one traced iteration of the overlapped case
    from torch.profiler import ProfilerActivity, profile
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        iteration(True, True)
        torch.cuda.synchronize()
    path = os.path.join(tempfile.mkdtemp(), "trace.json")
    prof.export_chrome_trace(path)
    ev = json.load(open(path))["traceEvents"]
    kernels = []
    for e in ev:
        if e.get("cat") in ("kernel", "gpu_memcpy", "gpu_memset") and "dur" in e:
            kernels.append((e["args"].get("stream"), e["name"], float(e["ts"]), float(e["ts"]) + float(e["dur"])))
    kernels.sort(key=lambda k: k[2])
    main_stream = max(set(k[0] for k in kernels), key=lambda s: sum(k[3] - k[2] for k in kernels if k[0] == s))
    local_names = ("spread_bulkpipe", "spread_local", "p2p_push")
    local_sum = sum(k[3] - k[2] for k in kernels if any(n in k[1] for n in local_names)) / 1e3
    side = [k for k in kernels if k[0] != main_stream]
    st = overlap_stats(kernels, main_stream)
    t00 = kernels[0][2] if kernels else 0.0
    out = {"what": "row a8 on one B200: EA exchange on the side stream vs the compute stream (spread layout, "
                   "world 1)", "workload": cfg.name, "stages": K, "stage_params": sizes[0],
           "exchange": a.exchange, "staleness": a.staleness, "tokens": a.tokens, "layers_per_stage": a.layers,
           "t_compute_ms": t_comp, "t_ea_ms": t_ea, "t_overlap_ms": t_ovl, "exposed_ms": t_ovl - t_comp,
           "local_kernels_sum_ms": local_sum, "exposed_minus_local_ms": t_ovl - t_comp - local_sum,
           "trace": {"kernels": len(kernels), "main_stream": main_stream,
                     "side_streams": sorted(set(str(k[0]) for k in side)),
                     "side_kernel_names": sorted(set(k[1][:60] for k in side)), **st},
           "knobs": {k: v for k, v in os.environ.items() if k.startswith("AVGPIPE_EA_")}}
    print(json.dumps(out), flush=True)
    if a.out:
        tl = [{"stream": k[0], "name": k[1][:80], "start_us": round(k[2] - t00, 2), "dur_us": round(k[3] - k[2], 2)}
              for k in kernels]
        json.dump({"summary": out, "timeline": tl}, open(a.out, "w"), indent=0)
    h.close()


if __name__ == "__main__":
    main()
