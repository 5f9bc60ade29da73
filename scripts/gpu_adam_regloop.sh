#!/bin/bash
# Adam/AdamW through the register-loop kernel: parity, then N = 1..8 against the per-N default.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "register_loop or adam" > gpurun_out/pytest_adam.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_adam.log
: > gpurun_out/adam_regloop.jsonl
for n in 1 2 3 4 5 6 7 8; do
  for v in auto regloop; do
    timeout 300 python bench.py --optimizer adam --n $n --variant $v --no-e2e --no-cpu-baseline >> gpurun_out/adam_regloop.jsonl 2>> gpurun_out/adam_regloop.err
  done
done
for cfg in C4; do
  for v in auto regloop; do
    timeout 300 python bench.py --optimizer adam --config $cfg --variant $v --no-e2e --no-cpu-baseline --steps 200 >> gpurun_out/adam_regloop.jsonl 2>> gpurun_out/adam_regloop.err
  done
done
timeout 300 python bench.py --n 8 --variant regloop --no-e2e --no-cpu-baseline >> gpurun_out/adam_regloop.jsonl 2>> gpurun_out/adam_regloop.err
echo done
