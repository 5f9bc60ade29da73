#!/bin/bash
# compute-sanitizer (memcheck, racecheck, synccheck) over scripts/sanitize_check.py.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
for tool in memcheck racecheck synccheck; do
  AVGPIPE_EA_P2P_TIMEOUT_MS=120000 timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python scripts/sanitize_check.py > gpurun_out/san_$tool.log 2>&1
  echo "rc=$?" >> gpurun_out/san_$tool.log
  tail -3 gpurun_out/san_$tool.log
done
echo done
