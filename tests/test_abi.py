"""C-ABI library: loads, exports every symbol include/ea.h declares, validates
arguments before touching CUDA, and its host-only schedule generator (row a9)
matches the oracle bit-exactly.  No GPU needed."""
import ctypes
import os
import random
import re
import subprocess

import pytest

from oracle.schedule import advance_forward_schedule
from paper_conf_ppopp_chen0qz23_b200 import binding
from paper_conf_ppopp_chen0qz23_b200.build import build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "ea.h")


@pytest.fixture(scope="module")
def lib():
    build()
    return binding.load_library()


def header_functions():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(ea_[a-z0-9_]+)\s*\(", text)))


def test_header_lists_the_north_star_calls():
    fns = header_functions()
    for name in ("ea_init", "ea_step", "ea_sync", "ea_destroy", "ea_schedule", "ea_get_state", "ea_set_state",
                 "ea_center_capacity", "ea_get_unique_id", "ea_last_error"):
        assert name in fns


def test_every_header_symbol_exported(lib):
    out = subprocess.run(["nm", "-D", "--defined-only", binding.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (ea_\w+)", out))
    missing = [f for f in header_functions() if f not in exported]
    assert not missing, missing
    # and the binding types exactly those
    assert set(binding.SIGNATURES) == set(header_functions())
    # nothing else leaks (visibility=hidden)
    assert exported == set(header_functions())


def test_abi_version(lib):
    assert lib.ea_abi_version() == binding.ABI_VERSION


def test_config_struct_layout_matches_header(tmp_path):
    """ctypes' ea_config / ea_op layout == what the C compiler makes of include/ea.h (sizeof and the
    offset of every field)."""
    import shutil
    import subprocess
    if shutil.which("gcc") is None:
        pytest.skip("gcc not available")
    fields = [f for f, _ in binding.EAConfig._fields_]
    src = ['#include <stddef.h>', '#include <stdio.h>', '#include "ea.h"', "int main(void) {",
           '  printf("size %zu\\n", sizeof(ea_config));', '  printf("op %zu\\n", sizeof(ea_op));']
    src += [f'  printf("{f} %zu\\n", offsetof(ea_config, {f}));' for f in fields]
    src += ["  return 0;", "}"]
    (tmp_path / "layout.c").write_text("\n".join(src) + "\n")
    exe = tmp_path / "layout"
    subprocess.run(["gcc", "-std=c99", "-I", os.path.join(ROOT, "include"), str(tmp_path / "layout.c"), "-o",
                    str(exe)], check=True)
    got = dict(line.split() for line in subprocess.run([str(exe)], capture_output=True, text=True,
                                                       check=True).stdout.splitlines())
    assert int(got["size"]) == ctypes.sizeof(binding.EAConfig)
    assert int(got["op"]) == ctypes.sizeof(binding.EAOp)
    for f in fields:
        assert int(got[f]) == getattr(binding.EAConfig, f).offset, f


def _cfg(**kw):
    sp = (ctypes.c_int64 * 2)(1000, 1001)
    base = dict(n_pipelines=2, n_stages=2, stage_params=sp, alpha=0.5, beta=0.0, rho=1.0, lr=0.05, momentum=0.9,
                weight_decay=0.0, nesterov=0, layout=0, rank=0, world=1, device=0, kernel_variant=0, optimizer=0,
                beta1=0.9, beta2=0.999, eps=1e-8, exchange=0, staleness=0, asgd_lambd=1e-4, asgd_alpha=0.75,
                asgd_t0=1e6)
    base.update(kw)
    c = binding.EAConfig(**base)
    c._keep = sp
    return c


@pytest.mark.parametrize("kw,needle", [
    (dict(n_pipelines=0), "n_pipelines"),
    (dict(n_stages=0), "n_stages"),
    (dict(alpha=1.5), "alpha"),
    (dict(alpha=-0.1), "alpha"),
    (dict(momentum=1.0), "momentum"),
    (dict(weight_decay=-1.0), "weight_decay"),
    (dict(nesterov=2), "nesterov"),
    (dict(nesterov=1, momentum=0.0), "nesterov"),
    (dict(layout=7), "layout"),
    (dict(layout=1, world=3), "world"),
    (dict(layout=1, world=2, rank=2), "rank"),
    (dict(kernel_variant=9), "kernel_variant"),
    (dict(n_pipelines=65), "N must be"),
    (dict(lr=float("nan")), "finite"),
    (dict(optimizer=4), "optimizer"),
    (dict(optimizer=3, asgd_lambd=-1.0), "ASGD"),
    (dict(optimizer=3, asgd_t0=float("nan")), "ASGD"),
    (dict(optimizer=3, asgd_alpha=float("inf")), "ASGD"),
    (dict(exchange=5), "exchange"),
    (dict(staleness=2), "staleness"),
    (dict(staleness=1, layout=1, world=2, rank=0, exchange=1), "staleness 1"),   # stale spread needs NCCL
    (dict(layout=1, world=17, n_pipelines=17, rank=0, exchange=1), "world <="),
    (dict(optimizer=1, beta1=1.0), "betas"),
    (dict(optimizer=2, beta2=-0.5), "betas"),
    (dict(optimizer=1, eps=0.0), "eps"),
])
def test_init_rejects_bad_config(lib, kw, needle):
    h = ctypes.c_void_p(123)
    st = lib.ea_init(ctypes.byref(_cfg(**kw)), None, ctypes.byref(h))
    assert st == binding.EA_EINVAL
    assert h.value is None
    assert needle in binding.last_error(None)


def test_init_rejects_nonpositive_stage(lib):
    sp = (ctypes.c_int64 * 2)(1000, 0)
    c = _cfg(stage_params=sp)
    h = ctypes.c_void_p()
    assert lib.ea_init(ctypes.byref(c), None, ctypes.byref(h)) == binding.EA_EINVAL
    assert lib.ea_init(None, None, ctypes.byref(h)) == binding.EA_EINVAL
    assert lib.ea_init(ctypes.byref(c), None, None) == binding.EA_EINVAL


def test_null_handle_paths(lib):
    assert lib.ea_center_capacity(None, 0) == -1
    assert lib.ea_shard_elems(None, 0) == -1
    assert lib.ea_step(None, 0, None, None, None, None) == binding.EA_EINVAL
    assert lib.ea_sync(None, None) == binding.EA_EINVAL
    assert lib.ea_destroy(None) == binding.EA_OK
    assert lib.ea_set_hyper(None, None) == binding.EA_EINVAL
    assert lib.ea_get_step(None, 0, None) == binding.EA_EINVAL
    assert lib.ea_set_step(None, 0, 1) == binding.EA_EINVAL
    assert lib.ea_get_state(None, 0, 0, 0, None) == binding.EA_EINVAL
    assert isinstance(lib.ea_last_error(None), bytes)


@pytest.mark.skipif(__import__("torch").cuda.is_available(), reason="checks the no-GPU error path")
def test_valid_config_without_gpu_reports_cuda_error(lib):
    h = ctypes.c_void_p()
    st = lib.ea_init(ctypes.byref(_cfg()), None, ctypes.byref(h))
    assert st in (binding.EA_ECUDA, binding.EA_EINVAL)
    assert h.value is None


def test_channel_argument_checks_without_gpu(lib):
    """Activation channels (ea_chan_*): argument validation happens before any CUDA call, every call tolerates a
    NULL channel, and ea_chan_last_error(NULL) reports the last failed create."""
    out = ctypes.c_void_p()
    assert lib.ea_chan_create(0, 2, 1024, 4, ctypes.byref(out)) == binding.EA_EINVAL      # role
    assert b"role" in lib.ea_chan_last_error(None)
    assert lib.ea_chan_create(0, 0, 0, 4, ctypes.byref(out)) == binding.EA_EINVAL         # slot_bytes
    assert lib.ea_chan_create(0, 1, 1024, 0, ctypes.byref(out)) == binding.EA_EINVAL      # slots
    assert lib.ea_chan_create(0, 0, 1024, 4, None) == binding.EA_EINVAL                   # output
    assert out.value is None
    assert lib.ea_chan_send(None, None, 0, None) == binding.EA_EINVAL
    assert lib.ea_chan_recv(None, None, 0, None) == binding.EA_EINVAL
    assert lib.ea_chan_export(None, None) == binding.EA_EINVAL
    assert lib.ea_chan_connect(None, None) == binding.EA_EINVAL
    assert lib.ea_chan_pair(None, None) == binding.EA_EINVAL
    assert lib.ea_chan_count(None) == -1
    assert lib.ea_chan_destroy(None) == binding.EA_OK
    assert binding.CHAN_HANDLE_BYTES == 80 and binding.IPC_HANDLE_BYTES == 64


@pytest.mark.skipif(__import__("torch").cuda.is_available(), reason="checks the no-GPU error path")
def test_channel_create_without_gpu_reports_cuda_error(lib):
    out = ctypes.c_void_p()
    st = lib.ea_chan_create(0, 0, 1024, 4, ctypes.byref(out))
    assert st in (binding.EA_ECUDA, binding.EA_ENOMEM)
    assert out.value is None and lib.ea_chan_last_error(None)


# ----------------------------------------------------------------- schedule (a9)
def _oracle(K, M, stage, a):
    return advance_forward_schedule(K, M, stage + 1, a)


def test_schedule_bit_exact_exhaustive(lib):
    for K in range(1, 9):
        for M in range(0, 33):
            for stage in range(K):
                for a in range(-1, M + 2):
                    assert binding.schedule(K, M, stage, a) == _oracle(K, M, stage, a), (K, M, stage, a)


def test_schedule_bit_exact_sampled_large(lib):
    rnd = random.Random(0)
    for _ in range(3000):
        K = rnd.randint(1, 16)
        M = rnd.randint(0, 128)
        stage = rnd.randrange(K)
        a = rnd.randint(-2, M + 2)
        assert binding.schedule(K, M, stage, a) == _oracle(K, M, stage, a)


def test_schedule_rejects_bad_args(lib):
    out = (binding.EAOp * 16)()
    assert lib.ea_schedule(0, 4, 0, 1, out, 16) == -binding.EA_EINVAL
    assert lib.ea_schedule(2, -1, 0, 1, out, 16) == -binding.EA_EINVAL
    assert lib.ea_schedule(2, 4, 2, 1, out, 16) == -binding.EA_EINVAL
    assert lib.ea_schedule(2, 4, -1, 1, out, 16) == -binding.EA_EINVAL
    assert lib.ea_schedule(2, 9, 0, 1, out, 16) == -binding.EA_EINVAL      # cap < 2M
    assert lib.ea_schedule(2, 4, 0, 1, None, 8) == -binding.EA_EINVAL
    assert lib.ea_schedule(2, 0, 0, 1, None, 0) == 0


def test_advance_controller_native_equals_oracle(lib):
    """ea_advance_* (Alg. 1 lines 1, 9-10) bit-exact against oracle.schedule.AdvanceController."""
    from oracle.schedule import AdvanceController as OracleCtl
    rnd = random.Random(5)
    for _ in range(300):
        K, M = rnd.randint(1, 12), rnd.randint(0, 64)
        a, b = OracleCtl(K, M), binding.AdvanceController(K, M)
        assert a.advance_num == b.advance_num
        limit = rnd.uniform(5, 50)
        for _ in range(rnd.randint(1, 40)):
            t = rnd.choice([rnd.uniform(1, 10), a.last_time if a.last_time is not None else 3.0])
            peak, per = rnd.uniform(0, 50), rnd.uniform(0, 5)
            assert a.update(t, peak, per, limit) == b.update(t, peak, per, limit)
            assert [a.advance_for(k) for k in range(1, K + 1)] == [b.advance_for_stage(s) for s in range(K)]
