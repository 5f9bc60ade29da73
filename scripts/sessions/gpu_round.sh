#!/bin/bash
# One GPU session: build, smoke, gpu tests, bench lines, ncu launch list + full capture of the default kernel.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 180 python scripts/quick_check.py laneshfl > gpurun_out/quick.log 2>&1; echo "rc=$?" >> gpurun_out/quick.log
if ! grep -q "quick_check ok" gpurun_out/quick.log; then echo "quick check failed; stopping"; exit 3; fi
if [ -z "$SKIP_TESTS" ]; then
timeout 2400 python -m pytest tests -m gpu -q ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
fi
: > gpurun_out/bench.json
timeout 600 python bench.py >> gpurun_out/bench.json 2> gpurun_out/bench.err
for v in "--optimizer adam" "--optimizer adamw" "--variant regloop" "--variant bulkpipe" ${EXTRA_BENCH}; do
  timeout 300 python bench.py $v --no-e2e --no-cpu-baseline >> gpurun_out/bench.json 2>> gpurun_out/bench.err
done
for t in 22 23 31; do
  AVGPIPE_EA_LANE_TUNE=$t timeout 300 python bench.py --optimizer adam --no-e2e --no-cpu-baseline | sed "s/^{/{\"tune\": \"$t\", /" >> gpurun_out/bench_tune_adam.json 2>> gpurun_out/bench.err
done
timeout 300 python bench.py --impl reference --steps 200 --warmup 3 > gpurun_out/bench_reference.json 2>> gpurun_out/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"colocated|spread" -c 60 --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 50 --warmup 5 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:colocated -s 5 -c 1 -o gpurun_out/prof_default -f \
    python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_default.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:colocated -s 5 -c 1 -o gpurun_out/prof_adam -f \
    python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --optimizer adam > gpurun_out/ncu_full_adam.log 2>&1

# large-model points on one GPU (co-located)
timeout 900 python bench.py --config C5 --n 2 --no-e2e --no-cpu-baseline --steps 50 > gpurun_out/bench_c5n2.json 2>> gpurun_out/bench.err
echo done
