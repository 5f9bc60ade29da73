#!/bin/bash
# Fused peer-memory exchange: phase-A unroll (AVGPIPE_EA_P2P_UNROLL = 1, 2, 4) with per-instance occupancy;
# single rank and N virtual ranks; parity of the unrolled variants.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
for u in 2 4; do
  AVGPIPE_EA_P2P_UNROLL=$u timeout 900 python -m pytest tests/test_gpu_p2p.py -q -x -k "matches_oracle or adam" > gpurun_out/pytest_p2p_u$u.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_p2p_u$u.log
done
: > gpurun_out/p2p_unroll2.jsonl
for rep in 1 2; do
for c in C4 C3N4 C3N2; do
  for u in 1 2 4; do
    for n in 1 0; do
      nn=""; [ $n = 1 ] && nn="--n 1"
      AVGPIPE_EA_P2P_UNROLL=$u timeout 200 python scripts/bench_p2p_virtual.py --config $c $nn \
        | sed "s/^{/{\"unroll\": $u, /" >> gpurun_out/p2p_unroll2.jsonl 2>> gpurun_out/p2p_unroll2.err
    done
  done
done
done
echo done
