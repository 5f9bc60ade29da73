#!/bin/bash
# Round-2 session v: the warp-specialised kernel with U = 3 for Adam (ncu, session u: at U = 2 N = 6 / 7 keep only
# 12 / 14 replica warps per SM -- the register file is per SM sub-partition -- so fewer bytes are in flight than at
# N = 8); parity of the geometries, then Adam N = 5..8 against the defaults.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -k "warp_specialised_u2" --timeout 1400 > gpurun_out/pytest_u3.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_u3.log; tail -2 gpurun_out/pytest_u3.log
: > gpurun_out/u3.jsonl
run() {
  local envs="$1"; shift
  env $envs timeout 300 python bench.py --steps 500 --warmup 10 --no-e2e --no-cpu-baseline "$@" 2>> gpurun_out/u3.err \
    | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['knob']='$envs'; d['args']='$*'; print(json.dumps(d))" >> gpurun_out/u3.jsonl
}
for n in 5 6 7 8; do
  run "X=0" --optimizer adam --n $n
  run "AVGPIPE_EA_WARPSPEC_U=3" --optimizer adam --n $n --variant warpspec
  run "AVGPIPE_EA_WARPSPEC_U=2" --optimizer adam --n $n --variant warpspec
done
python - <<'PY'
import json
for l in open('gpurun_out/u3.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:45s} {d['knob']:24s} {r['kernel']:30s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f} {d['clocks']['reasons']}")
PY
echo session done
