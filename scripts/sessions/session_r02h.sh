#!/bin/bash
# Round-2 session h: the warp-per-replica cp.async ring kernel (variant 6) -- parity, then a same-box sweep against
# the library defaults for every optimizer and N <= 8, ring geometries for Adam; the peer-memory racecheck probe
# after the test-harness fix (gradients recorded on the stream that reads them).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
if [ -n "$REBUILD" ]; then
  python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
fi
timeout 900 python -m pytest tests/test_gpu_chan.py tests/test_gpu_pipeline.py -q -rs > gpurun_out/pytest_chan.log 2>&1
echo "chan pytest rc=$?" >> gpurun_out/pytest_chan.log; tail -4 gpurun_out/pytest_chan.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "warp_ring" -x > gpurun_out/pytest_ring.log 2>&1
echo "ring pytest rc=$?" >> gpurun_out/pytest_ring.log; tail -2 gpurun_out/pytest_ring.log
# ncu: launch list of the default bench command + one full capture of the C2 default kernel; summaries made here,
# the .ncu-rep files dropped (gpurun_out must stay under 64 MiB)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:colocated -s 3 -c 1 -o gpurun_out/prof_default -f \
    python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_default.log 2>&1
python scripts/ncu_summary.py gpurun_out/ncu_summary.md --launches gpurun_out/launches.csv \
    --full default=gpurun_out/prof_default.ncu-rep > gpurun_out/ncu_summary.log 2>&1
ncu -i gpurun_out/prof_default.ncu-rep --page raw --csv > gpurun_out/prof_default_raw.csv 2>/dev/null
rm -f gpurun_out/*.ncu-rep
: > gpurun_out/sweep_ring.jsonl
run() {
  local envs="$1"; shift
  env $envs timeout 300 python bench.py --steps 400 --warmup 10 --no-e2e --no-cpu-baseline "$@" 2>> gpurun_out/sweep_ring.err \
    | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['knob']='$envs'; d['args']='$*'; print(json.dumps(d))" >> gpurun_out/sweep_ring.jsonl
}
for opt in adam sgd asgd; do
  for n in 1 2 3 4 5 6 7 8; do
    run "X=0" --optimizer $opt --n $n
    run "X=0" --optimizer $opt --n $n --variant warpring
  done
done
for n in 1 2 3 4; do run "AVGPIPE_EA_WARPREP_U=4" --optimizer adam --n $n --variant warprep; done
for g in 16 18 24 23; do
  for n in 1 4 6 8; do run "AVGPIPE_EA_RING=$g" --optimizer adam --n $n --variant warpring; done
done
python - <<'PY'
import json
for l in open('gpurun_out/sweep_ring.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:50s} {d['knob']:18s} {r['kernel']:30s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f} {d['clocks']['reasons']}")
PY
AVGPIPE_EA_P2P_TIMEOUT_MS=120000 timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python scripts/probes/p2p_sanitize.py \
  > gpurun_out/san_racecheck_p2p.log 2>&1; echo "rc=$?" >> gpurun_out/san_racecheck_p2p.log
grep -E "ok|FAIL|hazard|ERROR SUMMARY|rc=" gpurun_out/san_racecheck_p2p.log | tail -12
echo session done
