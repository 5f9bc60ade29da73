#!/bin/bash
# Round-2 kernel sweep on one B200: bench.py lines (C2 sizes) for the configurations VERDICT r01 lists below 0.95
# of the HBM peak, default kernel vs the alternatives, same box.  Output: gpurun_out/sweep.jsonl (one line each,
# with "knob" and "args" added).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
: > gpurun_out/sweep.jsonl
run() {  # run "<env>" <bench args...>
  local envs="$1"; shift
  env $envs timeout 300 python bench.py --steps 300 --warmup 10 --no-e2e --no-cpu-baseline "$@" 2>> gpurun_out/sweep.err \
    | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['knob']='$envs'; d['args']='$*'; print(json.dumps(d))" >> gpurun_out/sweep.jsonl
}
for n in 1 5 6 7 8; do run "X=0" --staleness 1 --n $n; run "AVGPIPE_EA_FORCE_WIDE=1" --staleness 1 --n $n; done
run "X=0" --staleness 1 --n 6 --optimizer adam; run "AVGPIPE_EA_FORCE_WIDE=1" --staleness 1 --n 6 --optimizer adam
for v in auto bulkpipe laneshfl; do run "X=0" --optimizer asgd --n 8 --variant $v; done
run "X=0" --optimizer asgd --n 12; run "X=0" --n 12
for v in auto regloop bulkpipe; do run "X=0" --optimizer adam --n 7 --variant $v; run "X=0" --optimizer adam --n 8 --variant $v; done
for v in auto regloop laneshfl; do run "X=0" --n 1 --variant $v; done
run "X=0" --n 1 --optimizer adam; run "X=0" --n 1 --optimizer asgd
python scripts/bench_p2p_virtual.py --config C4 --steps 10 > gpurun_out/p2p_virtual.log 2>&1
python scripts/bench_p2p_virtual.py --config C3N4 --steps 10 >> gpurun_out/p2p_virtual.log 2>&1
python - <<'PY'
import json
for l in open('gpurun_out/sweep.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:45s} {d['knob']:26s} {r['kernel']:32s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f} clk {d['clocks']['sm_mhz']} {d['clocks']['reasons']}")
PY
grep -h '^{' gpurun_out/p2p_virtual.log
echo sweep done
