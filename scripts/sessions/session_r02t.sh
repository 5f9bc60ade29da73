#!/bin/bash
# Round-2 session t: verification of the committed state as the driver runs it -- build() from scratch, smoke(), the
# default bench line, the reference arm, Adam, a spread line, the ncu launch list + one full capture of the default
# kernel, then the whole -m gpu suite.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_default.jsonl 2> gpurun_out/bench_default.err
python scripts/show_bench.py gpurun_out/bench_default.jsonl
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_reference.jsonl 2> gpurun_out/bench_reference.err
tail -c 300 gpurun_out/bench_reference.jsonl
timeout 600 python bench.py --optimizer adam --no-cpu-baseline > gpurun_out/bench_adam.jsonl 2>> gpurun_out/bench_default.err
python scripts/show_bench.py gpurun_out/bench_adam.jsonl
timeout 600 python bench.py --layout spread --config C4 --no-cpu-baseline --steps 100 > gpurun_out/bench_spread_c4.jsonl 2>> gpurun_out/bench_default.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:colocated -s 3 -c 1 -o gpurun_out/prof_default -f \
    python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_default.log 2>&1
python scripts/ncu_summary.py gpurun_out/ncu_final.md --launches gpurun_out/launches.csv \
    --full default=gpurun_out/prof_default.ncu-rep > /dev/null 2>&1
rm -f gpurun_out/*.ncu-rep
head -30 gpurun_out/ncu_final.md
timeout 3000 python -m pytest tests -m gpu -q -rs -p no:cacheprovider --timeout 900 > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log; tail -5 gpurun_out/pytest_gpu.log
echo session done
