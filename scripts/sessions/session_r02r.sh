#!/bin/bash
# Round-2 session r: the spread local step on the warp-per-replica kernel (AVGPIPE_EA_SPREAD_KERNEL=warp) -- parity,
# then the local kernel alone on C3/C4/C5 stage sizes against the bulk-copy pipeline, twice.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "spread_local_kernel_variants" --timeout 600 > gpurun_out/pytest_sw.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_sw.log; tail -2 gpurun_out/pytest_sw.log
: > gpurun_out/spread_local.jsonl
for rep in 1 2; do
  for opt in sgd adam asgd; do
    for k in bulk warp; do
      AVGPIPE_EA_SPREAD_KERNEL=$k timeout 300 python scripts/bench_spread_local.py --optimizer $opt >> gpurun_out/spread_local.jsonl 2>> gpurun_out/spread_local.err
    done
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/spread_local.jsonl'):
    if l.startswith('{'):
        d = json.loads(l); print(f"spread local {d['kernel']:5s} {d['optimizer']:5s} {d['workload']:5s} frac {d['frac']:.3f} ms {d['ms']:.4f}")
PY
echo session done
