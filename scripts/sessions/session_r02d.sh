#!/bin/bash
# Round-2 closing session: the whole GPU suite, the bench line, the spread lines, ncu of the push kernel with the
# 32 K-float chunks, and the racecheck probe of the peer-memory path.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 4000 python -m pytest tests -m gpu -q -rf > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -4 gpurun_out/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
for a in "--layout spread --config C4 --exchange nccl --steps 50 --no-e2e --cpu-seconds 3" "--layout spread --config C4 --exchange p2p --steps 50 --no-e2e --no-cpu-baseline" "--layout spread --config C4 --exchange nccl --staleness 1 --steps 50 --no-e2e --no-cpu-baseline" "--staleness 1 --n 1 --no-e2e --no-cpu-baseline" "--optimizer adam --n 5 --no-e2e --no-cpu-baseline" "--optimizer asgd --n 5 --no-e2e --no-cpu-baseline"; do
  timeout 600 python bench.py $a >> gpurun_out/bench_more.json 2>> gpurun_out/bench_more.err
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:p2p_push -s 8 -c 1 -o gpurun_out/prof_p2p_push -f \
    python bench.py --layout spread --config C4 --exchange p2p --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_p2p.log 2>&1
for push in bulk plain; do
  AVGPIPE_EA_P2P_PUSH=$push AVGPIPE_EA_P2P_TIMEOUT_MS=120000 timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python scripts/probes/p2p_sanitize.py > gpurun_out/san_racecheck_p2p_$push.log 2>&1
  tail -3 gpurun_out/san_racecheck_p2p_$push.log
done
echo session done
