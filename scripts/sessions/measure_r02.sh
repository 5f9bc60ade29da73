#!/bin/bash
# Round-2 measurement session on one B200: the bench line, the ncu launch list of the same command, one
# `ncu --set full` capture per judged kernel (default co-located kernel at C2; the spread layout's local kernels
# at a C4 stage), the row-a8 traces, and the oracle arm.  Outputs under gpurun_out/ (copied into profiles/ here).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv > gpurun_out/gpu.txt
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
timeout 900 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
timeout 600 python bench.py --layout spread --config C4 --exchange nccl --steps 50 --no-e2e --cpu-seconds 3 > gpurun_out/bench_spread_nccl_c4.json 2> gpurun_out/bench_spread_nccl.err
timeout 600 python bench.py --layout spread --config C4 --exchange p2p --steps 50 --no-e2e --no-cpu-baseline > gpurun_out/bench_spread_p2p_c4.json 2> gpurun_out/bench_spread_p2p.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:colocated -s 3 -c 1 -o gpurun_out/prof_default -f \
    python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_default.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spread_bulkpipe -s 8 -c 1 -o gpurun_out/prof_spread_local -f \
    python bench.py --layout spread --config C4 --exchange nccl --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_spread.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:p2p_push -s 8 -c 1 -o gpurun_out/prof_p2p_push -f \
    python bench.py --layout spread --config C4 --exchange p2p --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_p2p.log 2>&1
for x in "nccl 0" "p2p 0" "nccl 1"; do
  set -- $x
  timeout 600 python scripts/trace_a8.py --exchange $1 --staleness $2 --out gpurun_out/trace_$1_s$2.json > gpurun_out/trace_$1_s$2.log 2>&1
done
timeout 900 python scripts/bench_c5_schedule.py --tokens 1024 > gpurun_out/c5.json 2> gpurun_out/c5.err
echo measure done
