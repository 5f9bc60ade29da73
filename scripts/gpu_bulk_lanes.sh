#!/bin/bash
# Bulk-copy pipeline with the copies issued from all producer lanes: parity + tile sweep per N.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
timeout 900 python -m pytest tests -m gpu -q -k "bulk or spread_decomposition or fullsize" > gpurun_out/pytest_bulk.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_bulk.log
: > gpurun_out/bulk_lanes.jsonl
for opt in sgd adam; do
  for n in 1 2 3 4 5 6 7 8; do
    for t in 64 128 256; do
      AVGPIPE_EA_BULK_TILE=$t timeout 200 python bench.py --optimizer $opt --n $n --variant bulkpipe --no-e2e --no-cpu-baseline --steps 500 | sed "s/^{/{\"tile\": \"$t\", /" >> gpurun_out/bulk_lanes.jsonl 2>> gpurun_out/bulk_lanes.err
    done
  done
done
for opt in sgd adam; do
  timeout 300 python scripts/bench_spread_local.py --optimizer $opt >> gpurun_out/bulk_lanes_spread.jsonl 2>> gpurun_out/bulk_lanes.err
done
echo done
