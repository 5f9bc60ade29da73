#!/bin/bash
# Row f4 on the lane kernel (2 <= N <= 4): stale-center GPU parity, then bench lines of the stale lane kernel vs the
# replica loop (AVGPIPE_EA_FORCE_WIDE=1) for SGD / ASGD / Adam at C2, and the ncu launch list of the stale line.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/stale_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/stale_smoke.log
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "stale" > gpurun_out/stale_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/stale_pytest.log
: > gpurun_out/stale_bench.jsonl
for opt in sgd asgd adam; do
  timeout 300 python bench.py --staleness 1 --optimizer $opt --no-e2e --no-cpu-baseline >> gpurun_out/stale_bench.jsonl 2>> gpurun_out/stale_bench.err
  AVGPIPE_EA_FORCE_WIDE=1 timeout 300 python bench.py --staleness 1 --optimizer $opt --no-e2e --no-cpu-baseline | sed 's/^{/{"knob": "FORCE_WIDE", /' >> gpurun_out/stale_bench.jsonl 2>> gpurun_out/stale_bench.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"colocated" -c 40 --csv --log-file gpurun_out/stale_launches.csv \
    python bench.py --staleness 1 --optimizer asgd --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/stale_ncu.log 2>&1
echo done
