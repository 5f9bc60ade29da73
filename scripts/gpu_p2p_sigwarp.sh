#!/bin/bash
# Fused peer-memory exchange: dedicated signal warp (AVGPIPE_EA_P2P_SIGWARP=1) vs block barrier + thread 0.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
AVGPIPE_EA_P2P_SIGWARP=1 timeout 900 python -m pytest tests/test_gpu_p2p.py tests/test_gpu_multirank.py -q -x > gpurun_out/pytest_p2p_sigwarp.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_p2p_sigwarp.log
: > gpurun_out/p2p_sigwarp.jsonl
for rep in 1 2; do
for c in C4 C3N4 C3N2; do
  for sw in 0 1; do
    for f in 1 0; do
    for n in 1 0; do
      nn=""; [ $n = 1 ] && nn="--n 1"
      AVGPIPE_EA_P2P_FENCE=$f AVGPIPE_EA_P2P_SIGWARP=$sw timeout 200 python scripts/bench_p2p_virtual.py --config $c $nn \
        | sed "s/^{/{\"sigwarp\": $sw, \"fence\": $f, /" >> gpurun_out/p2p_sigwarp.jsonl 2>> gpurun_out/p2p_sigwarp.err
    done
    done
  done
done
done
echo done
