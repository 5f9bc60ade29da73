#!/bin/bash
# Round-2 session: compute-sanitizer over the round-2 kernels, the parity-margin log with unrounded (float64)
# hyper-parameters in the oracle, the push kernel's chunk size, the split kernel's grid.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
bash scripts/sessions/gpu_sanitize.sh
AVGPIPE_PARITY_F64_HYPER=1 AVGPIPE_PARITY_LOG=gpurun_out/parity_margins_f64hyper.jsonl timeout 1800 \
  python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -m gpu -k "adam or c1_100 or accumulated" > gpurun_out/pytest_f64hyper.log 2>&1
tail -3 gpurun_out/pytest_f64hyper.log
AVGPIPE_PARITY_LOG=gpurun_out/parity_margins_f32hyper.jsonl timeout 1800 \
  python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -m gpu -k "adam or c1_100 or accumulated" > gpurun_out/pytest_f32hyper.log 2>&1
tail -3 gpurun_out/pytest_f32hyper.log
: > gpurun_out/sweep.jsonl
run() {
  local envs="$1"; shift
  env $envs timeout 300 python bench.py --steps 200 --warmup 10 --no-e2e --no-cpu-baseline "$@" 2>> gpurun_out/sweep.err \
    | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['knob']='$envs'; d['args']='$*'; print(json.dumps(d))" >> gpurun_out/sweep.jsonl
}
for c in 8192 16384 32768; do run "AVGPIPE_EA_P2P_CHUNK=$c" --layout spread --config C4 --exchange p2p --steps 50; done
for n in 5 6 7 8; do run "AVGPIPE_EA_GRID=296" --n $n --variant split; run "AVGPIPE_EA_GRID=296" --n $n --variant split --optimizer adam; done
python - <<'PY'
import json
for l in open('gpurun_out/sweep.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:55s} {d['knob']:26s} {r['kernel']:24s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f} step_hbm {d.get('step_hbm',{}).get('frac',0):.3f}")
PY
for c in 8192 32768; do AVGPIPE_EA_P2P_CHUNK=$c python scripts/bench_p2p_virtual.py --config C4 --steps 10 | tail -1; done
echo session done
