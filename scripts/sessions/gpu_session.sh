#!/bin/bash
# One gpurun session: build, a quick sanity check, then whatever the caller asks for.
#   TESTS="tests/test_gpu_state.py ..."   pytest targets (-m gpu), run under a timeout
#   BENCH="--optimizer adam|..."          extra bench.py lines (';'-separated argument lists)
#   CMDS="cmd1;cmd2"                      extra commands (each under timeout 900)
# Outputs under gpurun_out/ (scratch); the caller copies what is judged into profiles/.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?" >> gpurun_out/build.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
if ! grep -q "smoke ok" gpurun_out/smoke.log; then echo "smoke failed; stopping"; cat gpurun_out/smoke.log | tail -20; exit 3; fi
if [ -n "$TESTS" ]; then
  timeout ${TEST_TIMEOUT:-2400} python -m pytest $TESTS -m gpu -q -rf ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1
  echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
  tail -5 gpurun_out/pytest_gpu.log
fi
if [ -n "$BENCH" ]; then
  : > gpurun_out/bench.json
  IFS=';' read -ra LINES <<< "$BENCH"
  for b in "${LINES[@]}"; do
    timeout 600 python bench.py $b >> gpurun_out/bench.json 2>> gpurun_out/bench.err
  done
  python scripts/show_bench.py gpurun_out/bench.json 2>/dev/null | tail -20
fi
if [ -n "$CMDS" ]; then
  IFS=';' read -ra CS <<< "$CMDS"
  i=0
  for c in "${CS[@]}"; do
    i=$((i+1))
    timeout ${CMD_TIMEOUT:-900} bash -c "$c" > gpurun_out/cmd_$i.log 2>&1
    echo "cmd $i rc=$? : $c" >> gpurun_out/cmds.log
  done
  cat gpurun_out/cmds.log
fi
echo session done
