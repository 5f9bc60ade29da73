#!/bin/bash
# Round-2 session m: activation-channel bandwidth / latency and the live pipeline runtime over gloo vs the channels.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 600 python scripts/bench_chan.py > gpurun_out/bench_chan.jsonl 2> gpurun_out/bench_chan.err; echo "chan rc=$?"
cat gpurun_out/bench_chan.jsonl
timeout 1200 python scripts/bench_pipeline.py > gpurun_out/bench_pipeline.jsonl 2> gpurun_out/bench_pipeline.err; echo "pipeline rc=$?"
cat gpurun_out/bench_pipeline.jsonl
tail -5 gpurun_out/bench_pipeline.err
echo session done
