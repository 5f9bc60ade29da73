#!/bin/bash
# A/B on one box: bulk copies issued from one producer lane (AVGPIPE_EA_BULK_ISSUE=1) vs all 32 lanes.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
out=gpurun_out/issue_ab.jsonl; : > $out
B="--no-e2e --no-cpu-baseline --steps 500"
for n in 1 3 5 6 7; do for t in 128 256; do for k in 1 32; do
  AVGPIPE_EA_BULK_ISSUE=$k AVGPIPE_EA_BULK_TILE=$t timeout 200 python bench.py --n $n --variant bulkpipe $B | sed "s/^{/{\"tile\": \"$t\", \"issue\": $k, /" >> $out 2>> gpurun_out/issue_ab.err
done; done; done
for n in 3 4 5 6; do for k in 1 32; do
  AVGPIPE_EA_BULK_ISSUE=$k timeout 200 python bench.py --optimizer adam --n $n --variant bulkpipe $B | sed "s/^{/{\"tile\": \"auto\", \"issue\": $k, /" >> $out 2>> gpurun_out/issue_ab.err
done; done
for n in 2 3 5 6; do
  timeout 200 python bench.py --optimizer adam --n $n --variant regloop $B | sed "s/^{/{\"tile\": \"-\", \"issue\": 0, /" >> $out 2>> gpurun_out/issue_ab.err
done
: > gpurun_out/issue_ab_spread.jsonl
for k in 1 32; do for opt in sgd adam; do
  AVGPIPE_EA_BULK_ISSUE=$k timeout 300 python scripts/bench_spread_local.py --optimizer $opt | sed "s/^{/{\"issue\": $k, /" >> gpurun_out/issue_ab_spread.jsonl 2>> gpurun_out/issue_ab.err
done; done
echo done
