#!/bin/bash
# Round-2 session: the split register-loop variant vs the defaults (N = 5..8, every optimizer), the push kernel
# with the producer-issued release, the row-a8 traces with the world-1 defaults, the C5 harness.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
: > gpurun_out/sweep.jsonl
run() {
  local envs="$1"; shift
  env $envs timeout 300 python bench.py --steps 300 --warmup 10 --no-e2e --no-cpu-baseline "$@" 2>> gpurun_out/sweep.err \
    | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['knob']='$envs'; d['args']='$*'; print(json.dumps(d))" >> gpurun_out/sweep.jsonl
}
for opt in sgd asgd adam; do for n in 5 6 7 8; do run "X=0" --optimizer $opt --n $n; run "X=0" --optimizer $opt --n $n --variant split; done; done
run "X=0" --layout spread --config C4 --exchange p2p --steps 50
run "X=0" --layout spread --config C4 --exchange nccl --steps 50
python - <<'PY'
import json
for l in open('gpurun_out/sweep.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:55s} {r['kernel']:32s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f} clk {d['clocks']['sm_mhz']} {d['clocks']['reasons']}")
PY
timeout 900 ncu --set full --clock-control none --import-source on -k regex:p2p_push -s 8 -c 1 -o gpurun_out/prof_p2p_push -f \
    python bench.py --layout spread --config C4 --exchange p2p --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_p2p.log 2>&1
for x in "nccl 0" "p2p 0" "nccl 1"; do
  set -- $x
  timeout 600 python scripts/trace_a8.py --exchange $1 --staleness $2 --out gpurun_out/trace_$1_s$2.json > gpurun_out/trace_$1_s$2.log 2>&1
done
AVGPIPE_EA_SIDE_PRIO=0 timeout 600 python scripts/trace_a8.py --exchange nccl --out gpurun_out/trace_nccl_s0_prio0.json > /dev/null 2>&1
AVGPIPE_EA_SIDE_CTAS=37 timeout 600 python scripts/trace_a8.py --exchange nccl --out gpurun_out/trace_nccl_s0_cap37.json > /dev/null 2>&1
timeout 900 python scripts/bench_c5_schedule.py --tokens 1024 > gpurun_out/c5.json 2> gpurun_out/c5.err
cat gpurun_out/c5.json
echo session done
