#!/bin/bash
# Replica-loop kernel with the software-pipelined replica loop: parity + N sweep; bench JSON GPU test.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
timeout 1200 python -m pytest tests -m gpu -q -k "stale or maximum or replica_counts or adam_replica or gpu_bench or fuzz" > gpurun_out/pytest_wide.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_wide.log
: > gpurun_out/wide.jsonl
for opt in sgd adam; do for n in 7 8 12 16 32; do
  AVGPIPE_EA_FORCE_WIDE=1 timeout 200 python bench.py --optimizer $opt --n $n --no-e2e --no-cpu-baseline --steps 300 | sed "s/^{/{\"forced_wide\": 1, /" >> gpurun_out/wide.jsonl 2>> gpurun_out/wide.err
done; done
timeout 200 python bench.py --staleness 1 --no-e2e --no-cpu-baseline --steps 300 >> gpurun_out/wide.jsonl 2>> gpurun_out/wide.err
timeout 200 python bench.py --config C4 --optimizer adam --no-e2e --no-cpu-baseline --steps 100 >> gpurun_out/wide.jsonl 2>> gpurun_out/wide.err
echo done
