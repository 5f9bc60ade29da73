"""The GPU suite cannot shrink silently (round 1 lost 184 GPU parity tests to an edit once): the number of
collected `-m gpu` tests, per file, may only grow past the floors recorded here.  Collection needs no GPU."""
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# floors per file (collected -m gpu tests), raised whenever tests are added
FLOORS = {
    "test_gpu_parity.py": 323,
    "test_gpu_p2p.py": 27,
    "test_gpu_nccl_emu.py": 17,
    "test_gpu_state.py": 7,
    "test_gpu_fullsize.py": 17,
    "test_gpu_bench.py": 5,
    "test_gpu_multirank.py": 5,
    "test_gpu_pipeline.py": 5,
    "test_gpu_chan.py": 9,
    "test_gpu_fuzz.py": 120,
}
TOTAL_FLOOR = 535


def test_gpu_suite_size():
    out = subprocess.run([sys.executable, "-m", "pytest", "--collect-only", "-q", "-m", "gpu", "tests"], cwd=ROOT,
                         capture_output=True, text=True, timeout=600).stdout
    ids = [ln for ln in out.splitlines() if "::" in ln]
    per = {}
    for i in ids:
        f = os.path.basename(i.split("::")[0])
        per[f] = per.get(f, 0) + 1
    short = {f: (per.get(f, 0), n) for f, n in FLOORS.items() if per.get(f, 0) < n}
    assert not short, f"GPU tests disappeared (collected, floor): {short}"
    m = re.search(r"(\d+)/\d+ tests collected", out)
    total = int(m.group(1)) if m else len(ids)
    assert total >= TOTAL_FLOOR, (total, TOTAL_FLOOR)
