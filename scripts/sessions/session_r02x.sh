#!/bin/bash
# Round-2 session x: the stale center with Adam on the warp-specialised kernel at U = 3 (N = 5..8) against the
# stale defaults (replica loop), after parity of that geometry.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
code="import tests.test_gpu_parity as t
for opt in ('adam', 'adamw'):
    for n in (1, 3, 5, 6, 8):
        t._run_colocated(n, [100_003, 7, 4096], 20, 'combined', variants=('warpspec',), many=True, optimizer=opt, lr=1e-3, staleness=1)
print('stale u3 parity ok')"
AVGPIPE_EA_WARPSPEC_U=3 timeout 900 python -c "$code" > gpurun_out/stale_u3_parity.log 2>&1; tail -1 gpurun_out/stale_u3_parity.log
: > gpurun_out/stale_u3.jsonl
run() {
  local envs="$1"; shift
  env $envs timeout 300 python bench.py --steps 500 --warmup 10 --no-e2e --no-cpu-baseline "$@" 2>> gpurun_out/stale_u3.err \
    | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['knob']='$envs'; d['args']='$*'; print(json.dumps(d))" >> gpurun_out/stale_u3.jsonl
}
for n in 1 5 6 7 8; do
  run "X=0" --optimizer adam --n $n --staleness 1
  run "AVGPIPE_EA_WARPSPEC_U=3" --optimizer adam --n $n --staleness 1 --variant warpspec
  run "AVGPIPE_EA_WARPSPEC_U=2" --optimizer adam --n $n --staleness 1 --variant warpspec
done
python - <<'PY'
import json
for l in open('gpurun_out/stale_u3.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:50s} {d['knob']:24s} {r['kernel']:32s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f}")
PY
echo session done
