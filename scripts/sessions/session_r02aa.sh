#!/bin/bash
# Round-2 session aa: the stale center with SGD / ASGD at N = 6..8 on the warp-per-replica and warp-specialised
# kernels against the replica loop (measurement only).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
: > gpurun_out/stale_sgd678.jsonl
for opt in asgd sgd; do
  for n in 6 7 8; do
    for v in auto warprep warpspec; do
      timeout 300 python bench.py --steps 500 --warmup 10 --no-e2e --no-cpu-baseline --optimizer $opt --n $n --staleness 1 --variant $v 2>> gpurun_out/stale_sgd678.err \
        | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['args']='$opt $n $v'; print(json.dumps(d))" >> gpurun_out/stale_sgd678.jsonl
    done
  done
done
python - <<'PY'
import json
for l in open('gpurun_out/stale_sgd678.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:20s} {r['kernel']:32s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f}")
PY
echo session done
