#!/bin/bash
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -m paper_conf_ppopp_chen0qz23_b200.build > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "adam" > gpurun_out/pytest_adam.log 2>&1; echo rc=$? >> gpurun_out/pytest_adam.log
: > gpurun_out/adam.json
for n in 1 2 3 4 5 6 8; do
  for v in laneshfl bulkpipe; do
    timeout 300 python bench.py --config C2 --n $n --optimizer adam --variant $v --no-e2e --no-cpu-baseline --steps 150 | sed "s/^{/{\"sweep\": \"adam n=$n $v\", /" >> gpurun_out/adam.json 2>> gpurun_out/adam.err
  done
  AVGPIPE_EA_BULK_TILE=128 timeout 300 python bench.py --config C2 --n $n --optimizer adam --variant bulkpipe --no-e2e --no-cpu-baseline --steps 150 | sed "s/^{/{\"sweep\": \"adam n=$n bulk128\", /" >> gpurun_out/adam.json 2>> gpurun_out/adam.err
  AVGPIPE_EA_FORCE_WIDE=1 timeout 300 python bench.py --config C2 --n $n --optimizer adam --no-e2e --no-cpu-baseline --steps 150 | sed "s/^{/{\"sweep\": \"adam n=$n wide\", /" >> gpurun_out/adam.json 2>> gpurun_out/adam.err
done
echo done
