#!/bin/bash
# Round-2 session l: the software-pipelined warp-per-replica kernel (AVGPIPE_EA_WARPREP_PF=1) -- parity under the
# knobs, then a same-box sweep against the defaults (every optimizer, N <= 8; Adam with U = 2 and 4; stale).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -k "warp_per_replica_knobs" > gpurun_out/pytest_pf.log 2>&1
echo "pf pytest rc=$?" >> gpurun_out/pytest_pf.log; tail -2 gpurun_out/pytest_pf.log
: > gpurun_out/sweep_pf.jsonl
run() {
  local envs="$1"; shift
  env $envs timeout 300 python bench.py --steps 400 --warmup 10 --no-e2e --no-cpu-baseline "$@" 2>> gpurun_out/sweep_pf.err \
    | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['knob']='$envs'; d['args']='$*'; print(json.dumps(d))" >> gpurun_out/sweep_pf.jsonl
}
for n in 1 2 3 4 5 6 7 8; do
  run "X=0" --optimizer adam --n $n
  run "AVGPIPE_EA_WARPREP_PF=1" --optimizer adam --n $n --variant warprep
  run "AVGPIPE_EA_WARPREP_PF=1 AVGPIPE_EA_WARPREP_U=2" --optimizer adam --n $n --variant warprep
done
for n in 1 3 4 6 8; do
  run "X=0" --n $n
  run "AVGPIPE_EA_WARPREP_PF=1" --n $n
  run "X=0" --optimizer asgd --n $n
  run "AVGPIPE_EA_WARPREP_PF=1" --optimizer asgd --n $n
done
for n in 2 5; do
  run "X=0" --n $n --staleness 1
  run "AVGPIPE_EA_WARPREP_PF=1" --n $n --staleness 1
done
python - <<'PY'
import json
for l in open('gpurun_out/sweep_pf.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:50s} {d['knob']:48s} {r['kernel']:30s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f} {d['clocks']['reasons']}")
PY
echo session done
