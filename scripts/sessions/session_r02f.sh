#!/bin/bash
# Round-2 session: warp-per-replica defaults (N = 1..8 SGD / ASGD, stale), parity of the stale variant.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
timeout 1800 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "warp_per_replica" > gpurun_out/pytest_warprep.log 2>&1; tail -2 gpurun_out/pytest_warprep.log
: > gpurun_out/sweep.jsonl
run() {
  local envs="$1"; shift
  env $envs timeout 300 python bench.py --steps 500 --warmup 10 --no-e2e --no-cpu-baseline "$@" 2>> gpurun_out/sweep.err \
    | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['knob']='$envs'; d['args']='$*'; print(json.dumps(d))" >> gpurun_out/sweep.jsonl
}
for n in 1 2 3; do for opt in sgd asgd; do run "X=0" --optimizer $opt --n $n; run "X=0" --optimizer $opt --n $n --variant warprep; done; done
run "X=0"; run "X=0" --variant warprep; run "X=0"; run "X=0" --variant warprep
for n in 1 2 3 4 5 6 7 8; do for opt in sgd asgd; do run "X=0" --staleness 1 --optimizer $opt --n $n; run "X=0" --staleness 1 --optimizer $opt --n $n --variant warprep; done; done
for n in 2 4; do run "X=0" --staleness 1 --optimizer adam --n $n; run "X=0" --staleness 1 --optimizer adam --n $n --variant warprep; done
python - <<'PY'
import json
for l in open('gpurun_out/sweep.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:50s} {r['kernel']:32s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f} {d['clocks']['reasons']}")
PY
echo session done
