#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -m paper_conf_ppopp_chen0qz23_b200.build > /dev/null 2>&1
timeout 300 python scripts/quick_check.py bulkpipe > gpurun_out/quick_bulk.log 2>&1
timeout 900 compute-sanitizer --tool racecheck --error-exitcode 9 python scripts/quick_check.py bulkpipe > gpurun_out/san_racecheck_bulkpipe.log 2>&1; echo "rc=$?" >> gpurun_out/san_racecheck_bulkpipe.log
: > gpurun_out/nsweep2.json
for n in 1 5 6 8; do
  for v in auto bulkpipe; do
    timeout 300 python bench.py --config C2 --n $n --variant $v --no-e2e --no-cpu-baseline --steps 200 | sed "s/^{/{\"sweep\": \"n=$n $v\", /" >> gpurun_out/nsweep2.json 2>> gpurun_out/nsweep.err
  done
done
for n in 6 8; do
  timeout 300 python bench.py --config C2 --n $n --optimizer adam --no-e2e --no-cpu-baseline --steps 200 | sed "s/^{/{\"sweep\": \"adam n=$n auto\", /" >> gpurun_out/nsweep2.json 2>> gpurun_out/nsweep.err
done
timeout 600 python bench.py --config C4 --no-e2e --no-cpu-baseline --steps 100 | sed "s/^{/{\"sweep\": \"C4 auto\", /" >> gpurun_out/nsweep2.json 2>> gpurun_out/nsweep.err
timeout 600 python bench.py --config C4 --optimizer adam --no-e2e --no-cpu-baseline --steps 100 | sed "s/^{/{\"sweep\": \"C4 adam auto\", /" >> gpurun_out/nsweep2.json 2>> gpurun_out/nsweep.err
timeout 1200 python -m pytest tests -q -m gpu -k "replica_counts or step_many or adam" > gpurun_out/pytest_gpu.log 2>&1; echo rc=$? >> gpurun_out/pytest_gpu.log
echo done
