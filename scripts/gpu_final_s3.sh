#!/bin/bash
# Session-3 closing verification: the round script (build, smoke, all GPU tests, bench lines, ncu) plus the
# fused P2P kernel's proxy lines, memcheck of the P2P path, and ASGD / spread lines.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
bash scripts/gpu_round.sh
: > gpurun_out/final_extra.jsonl
for c in C4 C3N4 C3N2; do
  for n in 1 0; do
    nn=""; [ $n = 1 ] && nn="--n 1"
    timeout 200 python scripts/bench_p2p_virtual.py --config $c $nn >> gpurun_out/final_p2p.jsonl 2>> gpurun_out/final_extra.err
  done
done
timeout 300 python bench.py --optimizer asgd --no-cpu-baseline >> gpurun_out/final_extra.jsonl 2>> gpurun_out/final_extra.err
timeout 300 python bench.py --layout spread --config C4 --no-cpu-baseline --steps 50 >> gpurun_out/final_extra.jsonl 2>> gpurun_out/final_extra.err
timeout 300 python bench.py --layout spread --exchange p2p --config C4 --no-cpu-baseline --steps 50 >> gpurun_out/final_extra.jsonl 2>> gpurun_out/final_extra.err
timeout 600 compute-sanitizer --tool memcheck python -m pytest tests/test_gpu_p2p.py -q -x -k "matches_oracle or adam" > gpurun_out/final_p2p_memcheck.log 2>&1; echo "rc=$?" >> gpurun_out/final_p2p_memcheck.log
echo done
