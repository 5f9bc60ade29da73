#!/bin/bash
# Round-2 session j: diagnose the activation-channel test stall (per-operation events + bounded polls; per-test
# timeouts with stack dumps), the allocator-race probe of the peer-memory test harness, Adam N = 5 default.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 120 python scripts/probes/chan_probe.py > gpurun_out/chan_probe.log 2>&1; echo "rc=$?" >> gpurun_out/chan_probe.log
cat gpurun_out/chan_probe.log
timeout 900 python -m pytest tests/test_gpu_chan.py tests/test_gpu_pipeline.py -v -rs -p no:cacheprovider \
  --timeout 120 --timeout-method thread > gpurun_out/pytest_chan.log 2>&1
echo "chan pytest rc=$?" >> gpurun_out/pytest_chan.log; grep -E "PASSED|FAILED|SKIPPED|Timeout|rc=" gpurun_out/pytest_chan.log | tail -20
timeout 300 python scripts/probes/p2p_alloc_race_probe.py > gpurun_out/alloc_race_probe.log 2>&1; echo "rc=$?" >> gpurun_out/alloc_race_probe.log
cat gpurun_out/alloc_race_probe.log | tail -4
for n in 5; do
  timeout 300 python bench.py --steps 400 --warmup 10 --no-e2e --no-cpu-baseline --optimizer adam --n $n >> gpurun_out/adam5.jsonl 2>> gpurun_out/adam5.err
done
python scripts/show_bench.py gpurun_out/adam5.jsonl
echo session done
