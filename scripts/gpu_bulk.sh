#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -m paper_conf_ppopp_chen0qz23_b200.build > /dev/null 2>&1
: > gpurun_out/bulk.json
for n in 1 2 3; do
  for t in 512; do
    AVGPIPE_EA_BULK_TILE=$t timeout 300 python bench.py --config C2 --n $n --variant bulkpipe --no-e2e --no-cpu-baseline --steps 200 | sed "s/^{/{\"sweep\": \"n=$n tile=$t\", /" >> gpurun_out/bulk.json 2>> gpurun_out/bulk.err
  done
done
for n in 2 3 4; do
  timeout 300 python bench.py --config C2 --n $n --variant laneshfl --no-e2e --no-cpu-baseline --steps 200 | sed "s/^{/{\"sweep\": \"n=$n lane\", /" >> gpurun_out/bulk.json 2>> gpurun_out/bulk.err
  AVGPIPE_EA_BULK_TILE=128 timeout 300 python bench.py --config C2 --n $n --variant bulkpipe --no-e2e --no-cpu-baseline --steps 200 | sed "s/^{/{\"sweep\": \"n=$n tile=128\", /" >> gpurun_out/bulk.json 2>> gpurun_out/bulk.err
done
echo done
