#!/bin/bash
# Round-2 session o: the warp-specialised warp-per-replica kernel (variant 6) -- parity, then a same-box sweep
# against the defaults (every optimizer, N <= 8, U = 2 / 4; the stale center).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "warp_specialised" --timeout 600 > gpurun_out/pytest_ws.log 2>&1
echo "ws pytest rc=$?" >> gpurun_out/pytest_ws.log; tail -3 gpurun_out/pytest_ws.log
if ! grep -q "ws pytest rc=0" gpurun_out/pytest_ws.log; then echo "parity failed; no sweep"; exit 0; fi
: > gpurun_out/sweep_ws.jsonl
run() {
  local envs="$1"; shift
  env $envs timeout 300 python bench.py --steps 400 --warmup 10 --no-e2e --no-cpu-baseline "$@" 2>> gpurun_out/sweep_ws.err \
    | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['knob']='$envs'; d['args']='$*'; print(json.dumps(d))" >> gpurun_out/sweep_ws.jsonl
}
for opt in adam sgd asgd; do
  for n in 1 2 3 4 5 6 7 8; do
    run "X=0" --optimizer $opt --n $n
    run "X=0" --optimizer $opt --n $n --variant warpspec
    run "AVGPIPE_EA_WARPSPEC_U=2" --optimizer $opt --n $n --variant warpspec
  done
done
for opt in adam sgd; do
  for n in 1 3 4 6 8; do
    run "X=0" --optimizer $opt --n $n --staleness 1
    run "X=0" --optimizer $opt --n $n --staleness 1 --variant warpspec
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/sweep_ws.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:55s} {d['knob']:24s} {r['kernel']:32s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f} {d['clocks']['reasons']}")
PY
echo session done
