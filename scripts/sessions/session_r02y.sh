#!/bin/bash
# Round-2 session y: the stale-center Adam defaults on the warp-specialised kernel (N = 1, 3, 5-8) -- smoke, bench
# lines, the default C2 line, the whole GPU suite.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
: > gpurun_out/stale_defaults.jsonl
for a in "" "--optimizer adam --n 1 --staleness 1" "--optimizer adam --n 5 --staleness 1" "--optimizer adam --n 6 --staleness 1" \
         "--optimizer adam --n 7 --staleness 1" "--optimizer adam --n 8 --staleness 1" "--staleness 1"; do
  timeout 300 python bench.py --steps 500 --warmup 10 --no-e2e --no-cpu-baseline $a 2>> gpurun_out/stale_defaults.err \
    | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['args']='$a'; print(json.dumps(d))" >> gpurun_out/stale_defaults.jsonl
done
python - <<'PY'
import json
for l in open('gpurun_out/stale_defaults.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:40s} {r['kernel']:32s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f} launches {d.get('gpu_launches')}")
PY
timeout 3000 python -m pytest tests -m gpu -q -rs -p no:cacheprovider --timeout 900 > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log; tail -5 gpurun_out/pytest_gpu.log
echo session done
