#!/bin/bash
# Adam at N = 7, 8 (co-located): bulk-copy pipeline tile sweep against the replica-loop default.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
: > gpurun_out/adam8.jsonl
for n in 7 8; do
  timeout 300 python bench.py --optimizer adam --n $n --no-e2e --no-cpu-baseline | sed "s/^{/{\"tile\": \"auto\", /" >> gpurun_out/adam8.jsonl 2>> gpurun_out/adam8.err
  for t in 64 128; do
    AVGPIPE_EA_BULK_TILE=$t timeout 300 python bench.py --optimizer adam --n $n --variant bulkpipe --no-e2e --no-cpu-baseline | sed "s/^{/{\"tile\": \"$t\", /" >> gpurun_out/adam8.jsonl 2>> gpurun_out/adam8.err
  done
done
for t in 64 128; do
  AVGPIPE_EA_BULK_TILE=$t timeout 300 python bench.py --n 8 --variant bulkpipe --no-e2e --no-cpu-baseline | sed "s/^{/{\"tile\": \"$t\", /" >> gpurun_out/adam8.jsonl 2>> gpurun_out/adam8.err
done
timeout 300 python bench.py --n 8 --no-e2e --no-cpu-baseline | sed "s/^{/{\"tile\": \"auto\", /" >> gpurun_out/adam8.jsonl 2>> gpurun_out/adam8.err
timeout 600 python bench.py > gpurun_out/bench_default.json 2>> gpurun_out/adam8.err
echo done
