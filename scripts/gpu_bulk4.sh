#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -m paper_conf_ppopp_chen0qz23_b200.build > /dev/null 2>&1
timeout 300 python scripts/quick_check.py bulkpipe > gpurun_out/quick_bulk.log 2>&1
: > gpurun_out/bulk4.json
for t in 96 128 160 192 256; do
  AVGPIPE_EA_BULK_TILE=$t timeout 300 python bench.py --config C2 --variant bulkpipe --no-e2e --no-cpu-baseline --steps 400 | sed "s/^{/{\"sweep\": \"n=4 tile=$t\", /" >> gpurun_out/bulk4.json 2>> gpurun_out/bulk.err
done
for n in 1 5 6 7 8; do
  timeout 300 python bench.py --config C2 --n $n --no-e2e --no-cpu-baseline --steps 200 | sed "s/^{/{\"sweep\": \"n=$n auto\", /" >> gpurun_out/bulk4.json 2>> gpurun_out/bulk.err
done
timeout 300 python bench.py --config C2 --no-e2e --no-cpu-baseline --steps 400 | sed "s/^{/{\"sweep\": \"n=4 auto\", /" >> gpurun_out/bulk4.json 2>> gpurun_out/bulk.err
echo done
