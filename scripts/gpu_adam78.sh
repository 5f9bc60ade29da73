#!/bin/bash
# Adam at N = 7, 8 through the bulk-copy pipeline with parallel copy issue (the earlier sweep predates it),
# against the replica-loop default; C4-sized Adam.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
: > gpurun_out/adam78.jsonl
for rep in 1 2; do
for n in 7 8; do
  for v in auto bulkpipe; do
    timeout 300 python bench.py --optimizer adam --n $n --variant $v --no-e2e --no-cpu-baseline --steps 300 | sed "s/^{/{\"sweep\": \"adam n=$n $v\", /" >> gpurun_out/adam78.jsonl 2>> gpurun_out/adam78.err
  done
  AVGPIPE_EA_BULK_TILE=64 timeout 300 python bench.py --optimizer adam --n $n --variant bulkpipe --no-e2e --no-cpu-baseline --steps 300 | sed "s/^{/{\"sweep\": \"adam n=$n bulkpipe tile64\", /" >> gpurun_out/adam78.jsonl 2>> gpurun_out/adam78.err
done
done
for v in auto bulkpipe; do
  timeout 600 python bench.py --config C4 --optimizer adam --variant $v --no-e2e --no-cpu-baseline --steps 50 | sed "s/^{/{\"sweep\": \"C4 adam $v\", /" >> gpurun_out/adam78.jsonl 2>> gpurun_out/adam78.err
done
echo done
