#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -m paper_conf_ppopp_chen0qz23_b200.build > /dev/null 2>&1
timeout 300 python scripts/quick_check.py bulkpipe > gpurun_out/quick_bulk.log 2>&1
: > gpurun_out/bulk.json
for n in 1 2 3 4 5 6 7 8; do
  for t in 0 64 128 256; do
    AVGPIPE_EA_BULK_TILE=$t timeout 300 python bench.py --config C2 --n $n --variant bulkpipe --no-e2e --no-cpu-baseline --steps 200 | sed "s/^{/{\"sweep\": \"n=$n tile=$t\", /" >> gpurun_out/bulk.json 2>> gpurun_out/bulk.err
  done
done
echo done
