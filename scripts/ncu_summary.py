#!/usr/bin/env python
"""Summarise ncu captures for profiles/ (run here, on the CPU box).

    python scripts/ncu_summary.py OUT.md [--launches launches.csv] [--full name=rep.ncu-rep ...]
"""
import argparse
import csv
import io
import subprocess
from collections import defaultdict

FULL_METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
    "lts__t_bytes.sum", "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
    "launch__occupancy_limit_registers", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__inst_executed.sum",
    "launch__shared_mem_per_block_static", "sm__cycles_elapsed.avg.per_second",
    "dram__cycles_elapsed.avg.per_second",
]


def launches(path):
    rows = [r for r in csv.reader(open(path)) if len(r) > 5]
    hdr = rows[0]
    ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
    agg = defaultdict(lambda: [0, 0.0])
    for r in rows[1:]:
        try:
            v = float(r[vi].replace(",", ""))
        except ValueError:
            continue
        name = r[ki]
        name = name.split("(")[0][:90]
        agg[name][0] += 1
        agg[name][1] += v
    tot = sum(v[1] for v in agg.values())
    out = ["| launches | total us | share | kernel |", "|---:|---:|---:|---|"]
    for k, (c, v) in sorted(agg.items(), key=lambda x: -x[1][1]):
        out.append(f"| {c} | {v / 1e3:.1f} | {100 * v / tot:.1f}% | `{k}` |")
    return "\n".join(out)


def full(rep):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    out = []
    for r in rows[2:]:
        name = r[hdr.index("Kernel Name")].split("(")[0]
        out.append(f"* `{name}`")
        for m in FULL_METRICS:
            if m in hdr:
                i = hdr.index(m)
                out.append(f"  * {m} = {r[i]} {units[i]}")
    return "\n".join(out)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("out")
    ap.add_argument("--title", default="ncu summary")
    ap.add_argument("--launches")
    ap.add_argument("--full", nargs="*", default=[])
    ap.add_argument("--note", default="")
    a = ap.parse_args()
    parts = [f"# {a.title}", "", a.note, ""]
    if a.launches:
        parts += ["## Launch list (`--metrics gpu__time_duration.sum --clock-control none`; cold, serialised)", "",
                  launches(a.launches), ""]
    for spec in a.full:
        name, rep = spec.split("=", 1)
        parts += [f"## `--set full` capture: {name}", "", full(rep), ""]
    open(a.out, "w").write("\n".join(parts))


if __name__ == "__main__":
    main()
