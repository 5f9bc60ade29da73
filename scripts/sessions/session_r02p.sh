#!/bin/bash
# Round-2 session p: the session-o defaults (warp-specialised kernel for Adam N = 8, SGD/ASGD N = 5, stale Adam N = 3)
# -- bench lines against the previous choices on one box, an ncu capture of the Adam N = 8 kernel, the whole GPU suite.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
: > gpurun_out/defaults.jsonl
run() {
  local envs="$1"; shift
  env $envs timeout 300 python bench.py --steps 500 --warmup 10 --no-e2e --no-cpu-baseline "$@" 2>> gpurun_out/defaults.err \
    | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['knob']='$envs'; d['args']='$*'; print(json.dumps(d))" >> gpurun_out/defaults.jsonl
}
run "X=0"
run "X=0" --optimizer adam --n 8
run "AVGPIPE_EA_FORCE_WIDE=1" --optimizer adam --n 8
run "X=0" --optimizer adamw --n 8
run "X=0" --n 5
run "X=0" --n 5 --variant warprep
run "X=0" --optimizer asgd --n 5
run "X=0" --optimizer asgd --n 5 --variant warprep
run "X=0" --optimizer adam --n 3 --staleness 1
run "X=0" --optimizer adam --n 3 --staleness 1 --variant laneshfl
run "X=0" --optimizer adam --n 7
python - <<'PY'
import json
for l in open('gpurun_out/defaults.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:55s} {d['knob']:24s} {r['kernel']:32s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f} {d['clocks']['reasons']}")
PY
timeout 900 ncu --set full --clock-control none --import-source on -k regex:colocated -s 3 -c 1 -o gpurun_out/prof_adam8 -f \
    python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --optimizer adam --n 8 > gpurun_out/ncu_adam8.log 2>&1
python scripts/ncu_summary.py gpurun_out/ncu_adam8.md --full adam8=gpurun_out/prof_adam8.ncu-rep > /dev/null 2>&1
rm -f gpurun_out/*.ncu-rep
cat gpurun_out/ncu_adam8.md | head -24
timeout 3000 python -m pytest tests -m gpu -q -rs -p no:cacheprovider --timeout 900 > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log; tail -5 gpurun_out/pytest_gpu.log
echo session done
