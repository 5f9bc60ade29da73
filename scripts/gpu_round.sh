#!/bin/bash
# One GPU session: build, smoke, gpu tests, bench (both variants), ncu launch list + full capture.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -q ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 300 python bench.py --variant regloop --no-e2e --no-cpu-baseline >> gpurun_out/bench.json 2>> gpurun_out/bench.err
timeout 300 python bench.py --variant laneshfl --no-e2e --no-cpu-baseline >> gpurun_out/bench.json 2>> gpurun_out/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:colocated -s 12 -c 2 -o gpurun_out/prof_regloop -f \
    python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --variant regloop > gpurun_out/ncu_full_regloop.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:colocated -s 12 -c 2 -o gpurun_out/prof_laneshfl -f \
    python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --variant laneshfl > gpurun_out/ncu_full_laneshfl.log 2>&1
echo done
