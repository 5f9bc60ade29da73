#!/bin/bash
# Round-2 session z: closing evidence -- the default bench line as the driver runs it, ncu full captures of the Adam
# N = 7 default (warp-specialised, U = 3) and the stale Adam N = 8 default.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 600 python bench.py > gpurun_out/bench_default.jsonl 2> gpurun_out/bench_default.err
python scripts/show_bench.py gpurun_out/bench_default.jsonl
timeout 900 ncu --set full --clock-control none -k regex:colocated -s 3 -c 1 -o gpurun_out/adam7 -f \
    python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --optimizer adam --n 7 > gpurun_out/ncu_adam7.log 2>&1
timeout 900 ncu --set full --clock-control none -k regex:colocated -s 3 -c 1 -o gpurun_out/stale_adam8 -f \
    python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --optimizer adam --n 8 --staleness 1 > gpurun_out/ncu_stale_adam8.log 2>&1
python scripts/ncu_summary.py gpurun_out/ncu_closing.md --full adam7=gpurun_out/adam7.ncu-rep stale_adam8=gpurun_out/stale_adam8.ncu-rep > /dev/null 2>&1
rm -f gpurun_out/*.ncu-rep
cat gpurun_out/ncu_closing.md
echo session done
