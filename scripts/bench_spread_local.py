#!/usr/bin/env python
"""Spread-layout local kernel alone (rows a1-a4 for the one replica a GPU holds):
CUDA-event time of ea_spread_local on C3/C4/C5 stage sizes, and its HBM
fraction at the algorithmic 28 B (SGD) / 36 B (Adam) per element.

    python scripts/bench_spread_local.py [--optimizer sgd|adam] [--reps 200]

AVGPIPE_EA_SPREAD_KERNEL=reg selects the register kernel instead of the
bulk-copy pipeline (measurement knob)."""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    import torch
    from paper_conf_ppopp_chen0qz23_b200.binding import ElasticAveraging
    from paper_conf_ppopp_chen0qz23_b200 import synth
    import bench

    ap = argparse.ArgumentParser()
    ap.add_argument("--optimizer", default="sgd")
    ap.add_argument("--reps", type=int, default=200)
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    peak, _ = bench.measured_peaks()
    for key, n in (("C3N2", 2), ("C4", 8), ("C5", 8)):
        p = synth.CONFIGS[key].stage_sizes[0]
        h = ElasticAveraging([p], n, alpha=1.0 / n, beta=1.0, rho=1.0, lr=1e-3, momentum=0.9, layout="spread",
                             rank=0, world=n, optimizer=args.optimizer)
        cap = h.center_capacity(0)
        x = torch.randn(p, device=dev) * 0.02
        g = torch.randn(p, device=dev) * 0.01
        c = torch.zeros(cap, device=dev)
        c[:p] = x
        r = torch.empty(cap, device=dev)
        for _ in range(5):
            h.spread_local(0, x, g, c, r)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(args.reps):
            h.spread_local(0, x, g, c, r)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / args.reps
        nbytes = bench.bytes_spread_local(p, args.optimizer)
        gbs = nbytes / (ms * 1e-3) / 1e9
        print(json.dumps({"what": "spread local kernel", "kernel": os.environ.get("AVGPIPE_EA_SPREAD_KERNEL", "bulk"),
                          "optimizer": args.optimizer, "workload": key, "stage_params": p, "ms": ms,
                          "bytes": nbytes, "gbs": gbs, "peak": peak, "frac": gbs / peak}))
        h.close()
        del x, g, c, r
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
