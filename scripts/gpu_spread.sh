#!/bin/bash
# Spread-layout local kernel: bulk pipeline vs register kernel; spread parity tests; world-1 spread bench
# (with its e2e line); ncu full capture of the default co-located kernel.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
: > gpurun_out/spread_local.jsonl
for opt in sgd adam; do
  timeout 300 python scripts/bench_spread_local.py --optimizer $opt >> gpurun_out/spread_local.jsonl 2>> gpurun_out/spread.err
  AVGPIPE_EA_SPREAD_KERNEL=reg timeout 300 python scripts/bench_spread_local.py --optimizer $opt >> gpurun_out/spread_local.jsonl 2>> gpurun_out/spread.err
done
timeout 1200 python -m pytest tests -m gpu -q -k "spread or p2p or fuzz" > gpurun_out/pytest_spread.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_spread.log
: > gpurun_out/bench_spread.json
for cfg in C3N2 C4; do
  timeout 300 python bench.py --layout spread --config $cfg --steps 100 >> gpurun_out/bench_spread.json 2>> gpurun_out/spread.err
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:colocated -s 5 -c 1 -o gpurun_out/prof_default2 -f \
    python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_default2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spread -s 5 -c 1 -o gpurun_out/prof_spread -f \
    python scripts/bench_spread_local.py --reps 10 > gpurun_out/ncu_full_spread.log 2>&1
echo done
