#!/bin/bash
# Round-2 session k: activation-channel + pipeline tests (per-test timeouts), eager-loading init cost, the stale
# center with Adam on the warp-per-replica kernel (U = 4) against the stale defaults.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
( time CUDA_MODULE_LOADING=EAGER python -c "import torch; torch.zeros(1).cuda(); torch.cuda.synchronize()" ) > gpurun_out/eager_init.log 2>&1
( time python -c "import torch; torch.zeros(1).cuda(); torch.cuda.synchronize()" ) >> gpurun_out/eager_init.log 2>&1
grep real gpurun_out/eager_init.log
timeout 1200 python -m pytest tests/test_gpu_chan.py tests/test_gpu_pipeline.py -v -rs -p no:cacheprovider \
  --timeout 300 --timeout-method thread > gpurun_out/pytest_chan.log 2>&1
echo "chan pytest rc=$?" >> gpurun_out/pytest_chan.log; grep -E "PASSED|FAILED|SKIPPED|ERROR|Timeout|rc=|passed|failed" gpurun_out/pytest_chan.log | tail -20
: > gpurun_out/sweep_stale_adam.jsonl
run() {
  local envs="$1"; shift
  env $envs timeout 300 python bench.py --steps 400 --warmup 10 --no-e2e --no-cpu-baseline "$@" 2>> gpurun_out/sweep_stale_adam.err \
    | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['knob']='$envs'; d['args']='$*'; print(json.dumps(d))" >> gpurun_out/sweep_stale_adam.jsonl
}
for n in 1 2 3 4 5 6 7 8; do
  run "X=0" --optimizer adam --n $n --staleness 1
  run "X=0" --optimizer adam --n $n --staleness 1 --variant warprep
done
for n in 1 3 4; do
  run "X=0" --optimizer asgd --n $n --staleness 1 --variant warprep
  run "X=0" --optimizer sgd --n $n --staleness 1 --variant warprep
done
python - <<'PY'
import json
for l in open('gpurun_out/sweep_stale_adam.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:55s} {r['kernel']:34s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f} {d['clocks']['reasons']}")
PY
echo session done
