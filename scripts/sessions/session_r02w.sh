#!/bin/bash
# Round-2 session w: the Adam N = 6..8 defaults on the warp-specialised kernel (U = 3 / 3 / 2) -- bench lines, smoke,
# the default C2 line, the whole GPU suite.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
: > gpurun_out/adam678.jsonl
for a in "" "--optimizer adam --n 6" "--optimizer adam --n 7" "--optimizer adam --n 8" "--optimizer adamw --n 7" "--optimizer adam"; do
  timeout 300 python bench.py --steps 500 --warmup 10 --no-e2e --no-cpu-baseline $a 2>> gpurun_out/adam678.err \
    | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['args']='$a'; print(json.dumps(d))" >> gpurun_out/adam678.jsonl
done
python - <<'PY'
import json
for l in open('gpurun_out/adam678.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:30s} {r['kernel']:30s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f} {d['clocks']['reasons']}")
PY
timeout 3000 python -m pytest tests -m gpu -q -rs -p no:cacheprovider --timeout 900 > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log; tail -5 gpurun_out/pytest_gpu.log
echo session done
