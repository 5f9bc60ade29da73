#!/usr/bin/env python
"""Turn scripts/trace_a8.py outputs (gpurun_out/trace_*.json) into profiles/<out>.md: one table row per run and,
for the first run, an excerpt of the kernel timeline of one stage (which stream ran what, when).

    python scripts/summarize_a8.py OUT.md gpurun_out/trace_nccl_s0.json [...]
"""
import json
import sys


def main():
    out, paths = sys.argv[1], sys.argv[2:]
    runs = [json.load(open(p)) for p in paths]
    lines = ["# Row a8 on one B200: the exchange on the side stream vs the compute stream", "",
             "`scripts/trace_a8.py` (spread layout, world 1, C4 stage sizes: K = 8 stages of 44.4 M params, "
             "GPT-2-medium-shaped bf16 GEMMs as the stage compute).  One iteration = backward of stage 7 → "
             "`ea_step(7)` → … → backward of stage 0 → `ea_step(0)` → forward of stages 0..7 → `ea_sync`.  Times are "
             "CUDA events (median of 7 iterations); the overlap columns come from a CUPTI trace "
             "(`torch.profiler`, the image has no nsys) of one iteration: side-stream kernel time covered by "
             "compute-stream kernels.", "",
             "| exchange | staleness | knobs | t_compute ms | t_ea ms | t_overlap ms | exposed ms | local kernels ms | "
             "exposed / t_ea | side-stream busy ms | covered by compute |",
             "|---|---|---|---:|---:|---:|---:|---:|---:|---:|---:|"]
    for r in runs:
        s = r["summary"] if "summary" in r else r
        t = s["trace"]
        knobs = ", ".join(f"{k}={v}" for k, v in s.get("knobs", {}).items()) or "default"
        lines.append(f"| {s['exchange']} | {s['staleness']} | {knobs} | {s['t_compute_ms']:.2f} | {s['t_ea_ms']:.2f} | "
                     f"{s['t_overlap_ms']:.2f} | {s['exposed_ms']:.2f} | {s['local_kernels_sum_ms']:.2f} | "
                     f"{s['exposed_ms'] / s['t_ea_ms']:.2f} | {t['side_busy_us'] / 1e3:.2f} | "
                     f"{(t['side_overlap_fraction'] or 0) * 100:.0f}% |")
    first = next((r for r in runs if "timeline" in r), None)
    if first:
        tl = first["timeline"]
        main_stream = first["summary"]["trace"]["main_stream"]
        # one stage's window: from the first local kernel to the next one
        idx = [i for i, k in enumerate(tl) if "spread_bulkpipe" in k["name"] or "p2p_push" in k["name"]]
        if len(idx) >= 2:
            a, b = idx[0], idx[1]
            t0 = tl[a]["start_us"]
            lines += ["", f"Timeline excerpt ({first['summary']['exchange']}, staleness "
                      f"{first['summary']['staleness']}): stage 7's local kernel up to stage 6's, every kernel on "
                      f"every stream (compute stream = {main_stream}).", "",
                      "| stream | start us | dur us | kernel |", "|---|---:|---:|---|"]
            end = tl[b]["start_us"] + tl[b]["dur_us"]
            for k in tl:
                if t0 - 1 <= k["start_us"] <= end:
                    tag = "compute" if k["stream"] == main_stream else "side"
                    lines.append(f"| {k['stream']} ({tag}) | {k['start_us'] - t0:.1f} | {k['dur_us']:.1f} | "
                                 f"`{k['name'][:70]}` |")
    open(out, "w").write("\n".join(lines) + "\n")


if __name__ == "__main__":
    main()
