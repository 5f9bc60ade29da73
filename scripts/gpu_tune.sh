#!/bin/bash
# Tuning sweep + sanitizers + overlap harness (one GPU).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -m paper_conf_ppopp_chen0qz23_b200.build > /dev/null 2>&1
timeout 300 python scripts/quick_check.py laneshfl > gpurun_out/quick_laneshfl.log 2>&1; echo "rc=$?" >> gpurun_out/quick_laneshfl.log
: > gpurun_out/tune.json
for t in 0 23 24 81; do
  AVGPIPE_EA_LANE_TUNE=$t timeout 300 python bench.py --no-e2e --no-cpu-baseline | sed "s/^{/{\"tune\": \"$t\", /" >> gpurun_out/tune.json 2>> gpurun_out/tune.err
done
timeout 300 python bench.py --variant bulkpipe --no-e2e --no-cpu-baseline | sed 's/^{/{"tune": "bulk", /' >> gpurun_out/tune.json 2>> gpurun_out/tune.err
for v in laneshfl bulkpipe regloop; do
  timeout 900 compute-sanitizer --tool memcheck --error-exitcode 9 python scripts/quick_check.py $v > gpurun_out/san_memcheck_$v.log 2>&1; echo "rc=$?" >> gpurun_out/san_memcheck_$v.log
done
for v in laneshfl bulkpipe; do
  timeout 900 compute-sanitizer --tool racecheck --error-exitcode 9 python scripts/quick_check.py $v > gpurun_out/san_racecheck_$v.log 2>&1; echo "rc=$?" >> gpurun_out/san_racecheck_$v.log
  timeout 900 compute-sanitizer --tool synccheck --error-exitcode 9 python scripts/quick_check.py $v > gpurun_out/san_synccheck_$v.log 2>&1; echo "rc=$?" >> gpurun_out/san_synccheck_$v.log
done
: > gpurun_out/overlap.json
timeout 300 python scripts/bench_overlap.py >> gpurun_out/overlap.json 2>> gpurun_out/overlap.err
timeout 300 python scripts/bench_overlap.py --n 4 --stages 4 --params 6250000 --micro 1 --tokens 4096 >> gpurun_out/overlap.json 2>> gpurun_out/overlap.err
timeout 300 python scripts/bench_overlap.py --n 8 --params 44375000 --micro 2 >> gpurun_out/overlap.json 2>> gpurun_out/overlap.err
echo done
