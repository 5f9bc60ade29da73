#!/bin/bash
# Round-2 session q: after the channel-handle change (geometry + role in the exported handle) and the smoke()
# additions -- smoke, channel + pipeline tests, the Adam N = 8 bench line with its ncu traffic entry.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 900 python -m pytest tests/test_gpu_chan.py tests/test_gpu_pipeline.py -q -rs -p no:cacheprovider --timeout 300 \
  > gpurun_out/pytest_chan.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_chan.log; tail -3 gpurun_out/pytest_chan.log
timeout 300 python bench.py --optimizer adam --n 8 --no-e2e --no-cpu-baseline > gpurun_out/bench_adam8.jsonl 2>/dev/null
python -c "import json; d=json.loads(open('gpurun_out/bench_adam8.jsonl').read().strip().splitlines()[-1]); print(d['roofline'])"
echo session done
