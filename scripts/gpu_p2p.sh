#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -m paper_conf_ppopp_chen0qz23_b200.build > /dev/null 2>&1
timeout 120 python scripts/quick_p2p.py > gpurun_out/quick_p2p.log 2>&1; echo "rc=$?" >> gpurun_out/quick_p2p.log
if ! grep -q "quick_p2p ok" gpurun_out/quick_p2p.log; then echo "p2p quick check failed"; exit 3; fi
timeout 1200 python -m pytest tests/test_gpu_p2p.py -q -m gpu > gpurun_out/pytest_p2p.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_p2p.log
timeout 600 compute-sanitizer --tool memcheck --error-exitcode 9 python scripts/quick_p2p.py > gpurun_out/san_memcheck_p2p.log 2>&1; echo "rc=$?" >> gpurun_out/san_memcheck_p2p.log
echo done
