#!/bin/bash
# ncu --set full of the fused P2P kernel after the session-3 changes (one rank and 8 virtual ranks, C4 stage).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spread_p2p -s 10 -c 1 -o gpurun_out/prof_p2p_n1_s3 -f \
    python scripts/bench_p2p_virtual.py --config C4 --n 1 --steps 2 --warmup 2 > gpurun_out/ncu_p2p_n1_s3.log 2>&1
echo done
