#!/usr/bin/env python
"""Row a8 on one GPU: how much of the elastic-averaging step hides under
backward compute when it runs on a side stream.

Synthetic backward: GPT-2-XL-shaped bf16 GEMMs (hidden 1600, 4h MLP, 6 layers
per stage; dgrad + wgrad of each layer, SURVEY §8(d) C5 recipe) for a
micro-batch of `--tokens` tokens, on the compute stream.  The EA step: the
co-located fused kernel over `--stages` stages of `--params` each, N
replicas, on a side stream gated by an event (what ea_step does in the
spread layout, and what a caller does co-located).

Reports t_bwd (GEMMs alone), t_ea (EA alone), t_serial (EA after the GEMMs on
one stream) and t_overlap (EA on the side stream launched when the
backward starts); exposed EA time = t_overlap - t_bwd.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=2)
    ap.add_argument("--stages", type=int, default=1)
    ap.add_argument("--params", type=int, default=187_500_000)   # one GPT-2-XL stage (1.5B / 8)
    ap.add_argument("--tokens", type=int, default=8192)
    ap.add_argument("--layers", type=int, default=6)
    ap.add_argument("--micro", type=int, default=4, help="backward micro-batches covered by one EA step")
    ap.add_argument("--reps", type=int, default=20)
    a = ap.parse_args()

    import torch
    from paper_conf_ppopp_chen0qz23_b200 import synth
    from paper_conf_ppopp_chen0qz23_b200.binding import ElasticAveraging

    dev = torch.device("cuda:0")
    h_ = 1600
    # per layer: (in, out) of QKV, proj, fc1, fc2
    shapes = [(h_, 3 * h_), (h_, h_), (h_, 4 * h_), (4 * h_, h_)]
    ws = [[torch.randn(i, o, device=dev, dtype=torch.bfloat16) * 0.02 for (i, o) in shapes] for _ in range(a.layers)]
    acts = {i: torch.randn(a.tokens, i, device=dev, dtype=torch.bfloat16) for (i, _) in shapes}
    grads_out = {o: torch.randn(a.tokens, o, device=dev, dtype=torch.bfloat16) for (_, o) in shapes}

    def backward_mb():
        for layer in ws:
            for (i, o), w in zip(shapes, layer):
                torch.matmul(grads_out[o], w.t())          # dgrad: [T,o] x [o,i]
                torch.matmul(acts[i].t(), grads_out[o])    # wgrad: [i,T] x [T,o]

    flops = a.micro * a.layers * sum(2 * 2 * a.tokens * i * o for (i, o) in shapes)

    sizes = [a.params] * a.stages
    al, be, rh = synth.mode_coeffs("combined", a.n)
    h = ElasticAveraging(sizes, a.n, alpha=al, beta=be, rho=rh, lr=synth.LR, momentum=synth.MOMENTUM)
    state = []
    for s, p in enumerate(sizes):
        reps, c, g = synth.device_state(a.n, p, dev, seed=s)
        state.append((reps, g, c))
    order = list(reversed(range(a.stages)))
    comp = torch.cuda.Stream(priority=-1)     # backward: high priority
    side = torch.cuda.Stream(priority=0)      # EA: low priority (fills SM slots the GEMMs leave)
    torch.cuda.set_stream(comp)

    def ea(stream):
        h.step_many(order, [state[s][0] for s in order], [state[s][1] for s in order], [state[s][2] for s in order],
                    stream=stream)

    def timed(fn):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(comp)
        for _ in range(a.reps):
            fn()
        e1.record(comp)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1) / a.reps

    def bwd_only():
        for _ in range(a.micro):
            backward_mb()

    def ea_only():
        ea(comp)

    def serial():
        bwd_only()
        ea(comp)

    def overlap():
        ev = torch.cuda.Event()
        ev.record(comp)
        side.wait_event(ev)
        ea(side)                      # EA of the stage whose backward just finished ...
        bwd_only()                    # ... under the backward of the remaining stages
        done = torch.cuda.Event()
        done.record(side)
        comp.wait_event(done)

    t_bwd, t_ea, t_ser, t_ovl = timed(bwd_only), timed(ea_only), timed(serial), timed(overlap)
    ea_bytes = sum((20 * a.n + 8) * p for p in sizes)
    out = {"what": "a8 stream overlap (1 GPU, co-located EA step on a side stream vs bf16 GEMM backward)",
           "grid_knob": os.environ.get("AVGPIPE_EA_GRID", "0"),
           "n": a.n, "stages": a.stages, "params_per_stage": a.params, "tokens": a.tokens, "layers": a.layers,
           "micro_batches": a.micro, "t_bwd_ms": t_bwd, "t_ea_ms": t_ea, "t_serial_ms": t_ser, "t_overlap_ms": t_ovl,
           "exposed_ea_ms": t_ovl - t_bwd, "hidden_fraction": 1 - (t_ovl - t_bwd) / t_ea,
           "bwd_tflops_alone": flops / (t_bwd * 1e-3) / 1e12, "ea_gbs_alone": ea_bytes / (t_ea * 1e-3) / 1e9}
    print(json.dumps(out), flush=True)
    h.close()


if __name__ == "__main__":
    main()
