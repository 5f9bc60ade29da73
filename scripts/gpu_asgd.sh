#!/bin/bash
# Row f1 ASGD: GPU parity (every kernel path) and bench lines.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
timeout 1500 python -m pytest tests -m gpu -q -k "asgd or graph or host_pipelined or p2p_exchange_adam" > gpurun_out/pytest_asgd.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_asgd.log
: > gpurun_out/bench_asgd.jsonl
timeout 300 python bench.py --optimizer asgd --no-e2e --no-cpu-baseline >> gpurun_out/bench_asgd.jsonl 2>> gpurun_out/bench_asgd.err
timeout 300 python bench.py --no-e2e --no-cpu-baseline >> gpurun_out/bench_asgd.jsonl 2>> gpurun_out/bench_asgd.err
for n in 1 8 12; do
  timeout 300 python bench.py --optimizer asgd --n $n --no-e2e --no-cpu-baseline --steps 300 >> gpurun_out/bench_asgd.jsonl 2>> gpurun_out/bench_asgd.err
done
timeout 300 python bench.py --optimizer asgd --layout spread --config C4 --no-e2e --no-cpu-baseline --steps 50 >> gpurun_out/bench_asgd.jsonl 2>> gpurun_out/bench_asgd.err
echo done
