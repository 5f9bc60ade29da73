#!/bin/bash
# Fused peer-memory exchange with unrolled phases: parity (virtual ranks + 2 processes), single-rank and
# virtual-rank efficiency.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
timeout 1200 python -m pytest tests -m gpu -q -k "p2p" > gpurun_out/pytest_p2p.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_p2p.log
: > gpurun_out/p2p_unroll.jsonl
for c in C4 C3N4 C3N2; do
  timeout 200 python scripts/bench_p2p_virtual.py --config $c --n 1 >> gpurun_out/p2p_unroll.jsonl 2>> gpurun_out/p2p.err
  timeout 200 python scripts/bench_p2p_virtual.py --config $c >> gpurun_out/p2p_unroll.jsonl 2>> gpurun_out/p2p.err
done
timeout 600 compute-sanitizer --tool memcheck python -m pytest tests/test_gpu_p2p.py -q -x -k "matches_oracle or adam" > gpurun_out/p2p_memcheck.log 2>&1; echo "rc=$?" >> gpurun_out/p2p_memcheck.log
echo done
