#!/bin/bash
# Round-2 session s: N = 1 on the warp-per-replica kernel applying x~ += r directly (no contribution tile, no barrier)
# -- parity, then N = 1 bench lines (SGD, ASGD, Adam on warprep vs the lane kernel).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "warp_per_replica or library_default" --timeout 600 > gpurun_out/pytest_n1.log 2>&1
echo "rc=$?" >> gpurun_out/pytest_n1.log; tail -2 gpurun_out/pytest_n1.log
: > gpurun_out/n1.jsonl
for rep in 1 2; do
  for a in "--n 1" "--optimizer asgd --n 1" "--optimizer adam --n 1" "--optimizer adam --n 1 --variant warprep" "--n 4"; do
    timeout 300 python bench.py --steps 500 --warmup 10 --no-e2e --no-cpu-baseline $a 2>> gpurun_out/n1.err \
      | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['args']='$a'; print(json.dumps(d))" >> gpurun_out/n1.jsonl
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/n1.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:45s} {r['kernel']:30s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f} {d['clocks']['reasons']}")
PY
echo session done
