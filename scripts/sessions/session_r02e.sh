#!/bin/bash
# Round-2 session: the warp-per-replica variant vs the defaults (N = 2..8 and every optimizer), the spread
# local kernel's tile, parity of the new variant.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
timeout 1800 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "warp_per_replica" > gpurun_out/pytest_warprep.log 2>&1; tail -2 gpurun_out/pytest_warprep.log
: > gpurun_out/sweep.jsonl
run() {
  local envs="$1"; shift
  env $envs timeout 300 python bench.py --steps 300 --warmup 10 --no-e2e --no-cpu-baseline "$@" 2>> gpurun_out/sweep.err \
    | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['knob']='$envs'; d['args']='$*'; print(json.dumps(d))" >> gpurun_out/sweep.jsonl
}
for opt in sgd adam asgd; do for n in 2 4 5 6 7 8; do run "X=0" --optimizer $opt --n $n; run "X=0" --optimizer $opt --n $n --variant warprep; done; done
for t in 256 512; do run "AVGPIPE_EA_BULK_TILE=$t" --layout spread --config C4 --exchange nccl --steps 50; done
python - <<'PY'
import json
for l in open('gpurun_out/sweep.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:55s} {d['knob']:24s} {r['kernel']:28s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f} step_hbm {d.get('step_hbm',{}).get('frac',0):.3f} clk {d['clocks']['sm_mhz']} {d['clocks']['reasons']}")
PY
for t in 256 512; do
  AVGPIPE_EA_BULK_TILE=$t timeout 900 ncu --set full --clock-control none -k regex:spread_bulkpipe -s 8 -c 1 -o gpurun_out/prof_spread_tile$t -f \
    python bench.py --layout spread --config C4 --exchange nccl --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
done
echo session done
for push in bulk plain; do
  AVGPIPE_EA_P2P_PUSH=$push AVGPIPE_EA_P2P_TIMEOUT_MS=120000 timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python scripts/probes/p2p_sanitize.py > gpurun_out/san_racecheck_p2p_$push.log 2>&1
  grep -v "^=====" gpurun_out/san_racecheck_p2p_$push.log | tail -12
done
AVGPIPE_EA_P2P_TIMEOUT_MS=120000 timeout 900 compute-sanitizer --tool memcheck python scripts/probes/p2p_sanitize.py > gpurun_out/san_memcheck_p2p.log 2>&1
grep -v "^=====" gpurun_out/san_memcheck_p2p.log | tail -6
echo racecheck probe done
