#!/bin/bash
# Per-N library defaults (auto) for SGD and Adam, C2 sizes.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
: > gpurun_out/nauto.jsonl
for opt in sgd adam; do for n in 1 2 3 4 5 6 7 8 12; do
  timeout 200 python bench.py --optimizer $opt --n $n --no-e2e --no-cpu-baseline --steps 500 >> gpurun_out/nauto.jsonl 2>> gpurun_out/nauto.err
done; done
