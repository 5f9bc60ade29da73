#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -m paper_conf_ppopp_chen0qz23_b200.build > /dev/null 2>&1
: > gpurun_out/sweep.json
for c in "--config C1" "--config C2" "--config C3N2" "--config C3N4" "--config C4" "--config C4 --optimizer adam"; do
  timeout 600 python bench.py $c --no-e2e --no-cpu-baseline --steps 200 | sed "s/^{/{\"sweep\": \"$c\", /" >> gpurun_out/sweep.json 2>> gpurun_out/sweep.err
done
for n in 1 2 3 4 5 6 7 8 12 16; do
  timeout 600 python bench.py --config C2 --n $n --no-e2e --no-cpu-baseline --steps 300 | sed "s/^{/{\"sweep\": \"C2 n=$n\", /" >> gpurun_out/sweep.json 2>> gpurun_out/sweep.err
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spread_p2p -s 20 -c 1 -o gpurun_out/prof_p2p -f \
    python scripts/bench_p2p_virtual.py --config C3N4 --steps 2 --warmup 6 > gpurun_out/ncu_p2p.log 2>&1
echo done
