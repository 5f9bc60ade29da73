#!/bin/bash
# ncu --set full of the fused peer-memory kernel, single rank (C4 stage sizes) and 8 virtual ranks.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spread_p2p -s 10 -c 1 -o gpurun_out/prof_p2p_n1 -f \
    python scripts/bench_p2p_virtual.py --config C4 --n 1 --steps 2 --warmup 2 > gpurun_out/ncu_p2p_n1.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spread_bulkpipe -s 10 -c 1 -o gpurun_out/prof_spread_bulk -f \
    python scripts/bench_spread_local.py --reps 12 > gpurun_out/ncu_spread_bulk.log 2>&1
echo done
