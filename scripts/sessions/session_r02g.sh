#!/bin/bash
# Round-2 session after the warp-per-replica defaults: bench line, ncu launch list + full capture of the new default
# kernel, Adam with U = 4 in the warp-per-replica kernel, then the whole GPU suite.
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 3; }
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
python scripts/show_bench.py gpurun_out/bench_default.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:colocated -s 3 -c 1 -o gpurun_out/prof_default -f \
    python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_full_default.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:colocated -s 3 -c 1 -o gpurun_out/prof_adam -f \
    python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --optimizer adam > gpurun_out/ncu_full_adam.log 2>&1
: > gpurun_out/sweep.jsonl
run() {
  local envs="$1"; shift
  env $envs timeout 300 python bench.py --steps 500 --warmup 10 --no-e2e --no-cpu-baseline "$@" 2>> gpurun_out/sweep.err \
    | python -c "import json,sys
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); d['knob']='$envs'; d['args']='$*'; print(json.dumps(d))" >> gpurun_out/sweep.jsonl
}
for n in 5 6 7 8; do run "AVGPIPE_EA_WARPREP_U=4" --optimizer adam --n $n --variant warprep; done
for n in 1 3 4 5 8; do run "X=0" --n $n; run "X=0" --optimizer asgd --n $n; done
run "X=0" --staleness 1 --n 2; run "X=0" --staleness 1 --n 5
python - <<'PY'
import json
for l in open('gpurun_out/sweep.jsonl'):
    d = json.loads(l); r = d['roofline']
    print(f"{d['args']:50s} {d['knob']:22s} {r['kernel']:30s} frac {r['frac']:.3f} ms {d['ms_per_step']:.4f} {d['clocks']['reasons']}")
PY
timeout 4000 python -m pytest tests -m gpu -q -rf > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -4 gpurun_out/pytest_gpu.log
echo session done
