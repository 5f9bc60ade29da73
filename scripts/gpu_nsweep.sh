#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -m paper_conf_ppopp_chen0qz23_b200.build > /dev/null 2>&1
: > gpurun_out/nsweep.json
for n in 1 2 3 5 6 7 8; do
  for v in laneshfl regloop bulkpipe; do
    timeout 300 python bench.py --config C2 --n $n --variant $v --no-e2e --no-cpu-baseline --steps 200 | sed "s/^{/{\"sweep\": \"n=$n $v\", /" >> gpurun_out/nsweep.json 2>> gpurun_out/nsweep.err
  done
  AVGPIPE_EA_FORCE_WIDE=1 timeout 300 python bench.py --config C2 --n $n --no-e2e --no-cpu-baseline --steps 200 | sed "s/^{/{\"sweep\": \"n=$n wide\", /" >> gpurun_out/nsweep.json 2>> gpurun_out/nsweep.err
done
for n in 4 8; do
  AVGPIPE_EA_FORCE_WIDE=1 timeout 300 python bench.py --config C2 --n $n --optimizer adam --no-e2e --no-cpu-baseline --steps 200 | sed "s/^{/{\"sweep\": \"adam n=$n wide\", /" >> gpurun_out/nsweep.json 2>> gpurun_out/nsweep.err
  timeout 300 python bench.py --config C2 --n $n --optimizer adam --no-e2e --no-cpu-baseline --steps 200 | sed "s/^{/{\"sweep\": \"adam n=$n lane\", /" >> gpurun_out/nsweep.json 2>> gpurun_out/nsweep.err
done
echo done
