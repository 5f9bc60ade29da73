#!/bin/bash
# Round-2 session i: the cp.async ring kernel with the stale center and as the spread local step -- parity, then
# same-box measurements against the current defaults (stale sweep per optimizer and N; spread local kernel alone
# on C3/C4/C5 stage sizes).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -k "warp_ring_stale or spread_local_kernel_variants" \
  > gpurun_out/pytest_ring2.log 2>&1
echo "ring2 pytest rc=$?" >> gpurun_out/pytest_ring2.log; tail -2 gpurun_out/pytest_ring2.log
: > gpurun_out/spread_local.jsonl
for opt in sgd adam; do
  for k in bulk ring; do
    AVGPIPE_EA_SPREAD_KERNEL=$k timeout 300 python scripts/bench_spread_local.py --optimizer $opt >> gpurun_out/spread_local.jsonl 2>> gpurun_out/spread_local.err
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/spread_local.jsonl'):
    if l.startswith('{'):
        d = json.loads(l); print(f"spread local {d['kernel']:5s} {d['optimizer']:5s} {d['workload']:5s} frac {d['frac']:.3f} ms {d['ms']:.4f}")
PY
: > gpurun_out/sweep_stale.jsonl
run() {
  local envs="$1"; shift
  env $envs timeout 300 python bench.py --steps 400 --warmup 10 --no-e2e --no-cpu-baseline "$@" 2>> gpurun_out/sweep_stale.err \
    | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['knob']='$envs'; d['args']='$*'; print(json.dumps(d))" >> gpurun_out/sweep_stale.jsonl
}
for opt in sgd adam asgd; do
  for n in 1 2 3 4 5 6 7 8; do
    run "X=0" --optimizer $opt --n $n --staleness 1
    run "X=0" --optimizer $opt --n $n --staleness 1 --variant warpring
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/sweep_stale.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:55s} {r['kernel']:34s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f} {d['clocks']['reasons']}")
PY
echo session done
