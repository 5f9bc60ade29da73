#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -m paper_conf_ppopp_chen0qz23_b200.build > /dev/null 2>&1
timeout 900 compute-sanitizer --tool racecheck --error-exitcode 9 python scripts/quick_check.py bulkpipe > gpurun_out/san_racecheck_bulkpipe.log 2>&1; echo "rc=$?" >> gpurun_out/san_racecheck_bulkpipe.log
: > gpurun_out/overlap.json
for g in 0 -1 16 32 64; do
  for cfg in "" "--n 4 --stages 4 --params 6250000 --micro 1 --tokens 4096"; do
    AVGPIPE_EA_GRID=$g timeout 300 python scripts/bench_overlap.py $cfg >> gpurun_out/overlap.json 2>> gpurun_out/overlap.err
  done
done
for g in -1 16 32 64; do
  AVGPIPE_EA_GRID=$g timeout 300 python bench.py --no-e2e --no-cpu-baseline --steps 300 | sed "s/^{/{\"grid\": \"$g\", /" >> gpurun_out/grid_bench.json 2>> gpurun_out/overlap.err
done
echo done
