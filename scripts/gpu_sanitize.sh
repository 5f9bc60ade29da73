#!/bin/bash
# compute-sanitizer over the kernels changed in session 2 + the new GPU tests.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "stale or register_loop" > gpurun_out/pytest_stale.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_stale.log
for tool in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python scripts/sanitize_check.py > gpurun_out/san_$tool.log 2>&1
  echo "rc=$?" >> gpurun_out/san_$tool.log
done
echo done
