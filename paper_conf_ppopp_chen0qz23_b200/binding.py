"""Thin ctypes binding of ``include/ea.h`` (argument marshalling only).

Every step of the elastic-averaging path runs inside ``libavgpipe_ea.so``
(hand-written sm_100a kernels + NCCL).  This module converts torch tensors,
streams and Python scalars into the C ABI's pointers and sizes, raises on a
non-zero ``ea_status`` with the library's message, and never computes
anything itself.  There is no fallback: if the library is missing, every
entry point raises ``LibraryNotBuilt``.
"""
from __future__ import annotations

import ctypes
import os
from typing import List, Optional, Sequence, Tuple

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libavgpipe_ea.so")

EA_OK, EA_EINVAL, EA_ECUDA, EA_ENCCL, EA_ESTATE, EA_ENOMEM = range(6)
EA_COLOCATED, EA_SPREAD = 0, 1
STATUS_NAMES = {0: "EA_OK", 1: "EA_EINVAL", 2: "EA_ECUDA", 3: "EA_ENCCL", 4: "EA_ESTATE", 5: "EA_ENOMEM"}
LAYOUTS = {"colocated": EA_COLOCATED, "spread": EA_SPREAD}
VARIANTS = {"auto": 0, "regloop": 1, "laneshfl": 2, "bulkpipe": 3, "split": 4, "warprep": 5, "warpspec": 6}
OPTIMIZERS = {"sgd": 0, "adam": 1, "adamw": 2, "asgd": 3}
EXCHANGES = {"nccl": 0, "p2p": 1}
UNIQUE_ID_BYTES = 128
IPC_HANDLE_BYTES = 64   # == EA_IPC_HANDLE_BYTES (cudaIpcMemHandle_t)
CHAN_HANDLE_BYTES = 80  # == EA_CHAN_HANDLE_BYTES (IPC handle + slot_bytes, slots, role)
ABI_VERSION = 6
SLOT_CENTER_PREV = 2   # EA_SLOT_CENTER_PREV: the stale center x~_{t-1} (staleness 1)


class LibraryNotBuilt(RuntimeError):
    pass


class EAError(RuntimeError):
    def __init__(self, status: int, message: str):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {message}")
        self.status = status


class EAConfig(ctypes.Structure):
    _fields_ = [
        ("n_pipelines", ctypes.c_int32),
        ("n_stages", ctypes.c_int32),
        ("stage_params", ctypes.POINTER(ctypes.c_int64)),
        ("alpha", ctypes.c_float),
        ("beta", ctypes.c_float),
        ("rho", ctypes.c_float),
        ("lr", ctypes.c_float),
        ("momentum", ctypes.c_float),
        ("weight_decay", ctypes.c_float),
        ("nesterov", ctypes.c_int32),
        ("layout", ctypes.c_int32),
        ("rank", ctypes.c_int32),
        ("world", ctypes.c_int32),
        ("device", ctypes.c_int32),
        ("kernel_variant", ctypes.c_int32),
        ("optimizer", ctypes.c_int32),
        ("beta1", ctypes.c_double),
        ("beta2", ctypes.c_double),
        ("eps", ctypes.c_float),
        ("exchange", ctypes.c_int32),
        ("staleness", ctypes.c_int32),
        ("asgd_lambd", ctypes.c_double),
        ("asgd_alpha", ctypes.c_double),
        ("asgd_t0", ctypes.c_double),
    ]


class EAOp(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("micro_batch", ctypes.c_int32)]


class EAAdvanceCtl(ctypes.Structure):
    _fields_ = [("K", ctypes.c_int32), ("M", ctypes.c_int32), ("advance_num", ctypes.c_int32),
                ("has_last", ctypes.c_int32), ("last_time", ctypes.c_double)]


class AdvanceController:
    """Algorithm 1's run-time advance_num adjustment (ea_advance_*)."""

    def __init__(self, K: int, M: int):
        self.ctl = EAAdvanceCtl()
        _check(load_library().ea_advance_init(ctypes.byref(self.ctl), K, M))

    @property
    def advance_num(self) -> int:
        return self.ctl.advance_num

    def update(self, batch_time: float, peak_mem: float, mem_per_microbatch: float, mem_limit: float) -> int:
        r = load_library().ea_advance_update(ctypes.byref(self.ctl), batch_time, peak_mem, mem_per_microbatch,
                                             mem_limit)
        if r < 0:
            raise EAError(-r, "ea_advance_update rejected its arguments")
        return r

    def advance_for_stage(self, stage: int) -> int:
        r = load_library().ea_advance_for_stage(ctypes.byref(self.ctl), stage)
        if r < 0:
            raise EAError(-r, f"bad stage {stage}")
        return r


class EAProfile(ctypes.Structure):
    _fields_ = [("n_gpus", ctypes.c_int32), ("m", ctypes.c_int32), ("n", ctypes.c_int32),
                ("n_samples", ctypes.c_int32), ("dt", ctypes.c_double),
                ("phi", ctypes.POINTER(ctypes.c_double)), ("t_gpu", ctypes.POINTER(ctypes.c_double)),
                ("t_comm", ctypes.POINTER(ctypes.c_double)), ("f_mod", ctypes.POINTER(ctypes.c_double)),
                ("f_dat", ctypes.POINTER(ctypes.c_double))]


class EAGpuPrediction(ctypes.Structure):
    _fields_ = [(f, ctypes.c_double) for f in ("t_gpu", "t_com", "t_up", "t_down", "t_bub", "t_total", "mem")]


# name -> (restype, argtypes); mirrors include/ea.h one to one.
_VP = ctypes.c_void_p
_FPP = ctypes.POINTER(ctypes.c_void_p)
SIGNATURES = {
    "ea_abi_version": (ctypes.c_int32, []),
    "ea_get_unique_id": (ctypes.c_int, [ctypes.c_void_p]),
    "ea_init": (ctypes.c_int, [ctypes.POINTER(EAConfig), ctypes.c_void_p, ctypes.POINTER(_VP)]),
    "ea_center_capacity": (ctypes.c_int64, [_VP, ctypes.c_int32]),
    "ea_shard_elems": (ctypes.c_int64, [_VP, ctypes.c_int32]),
    "ea_step": (ctypes.c_int, [_VP, ctypes.c_int32, _FPP, _FPP, _VP, _VP]),
    "ea_step_many": (ctypes.c_int, [_VP, ctypes.c_int32, ctypes.POINTER(ctypes.c_int32), _FPP, _FPP, _FPP, _VP]),
    "ea_step_many_host": (ctypes.c_int, [_VP, ctypes.c_int32, ctypes.POINTER(ctypes.c_int32), _FPP, _FPP, _FPP,
                                         _FPP, _VP]),
    "ea_p2p_connect": (ctypes.c_int, [_VP, ctypes.POINTER(_VP), ctypes.c_int32]),
    "ea_p2p_export": (ctypes.c_int, [_VP, ctypes.c_void_p]),
    "ea_p2p_open": (ctypes.c_int, [_VP, ctypes.c_void_p, ctypes.c_int32]),
    "ea_sync": (ctypes.c_int, [_VP, _VP]),
    "ea_spread_local": (ctypes.c_int, [_VP, ctypes.c_int32, _VP, _VP, _VP, _VP, _VP]),
    "ea_spread_apply": (ctypes.c_int, [_VP, ctypes.c_int32, _VP, _VP, _VP]),
    "ea_get_state": (ctypes.c_int, [_VP, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, ctypes.POINTER(_VP)]),
    "ea_set_state": (ctypes.c_int, [_VP, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, _VP, _VP]),
    "ea_get_step": (ctypes.c_int, [_VP, ctypes.c_int32, ctypes.POINTER(ctypes.c_int64)]),
    "ea_set_step": (ctypes.c_int, [_VP, ctypes.c_int32, ctypes.c_int64]),
    "ea_set_hyper": (ctypes.c_int, [_VP, ctypes.POINTER(EAConfig)]),
    "ea_destroy": (ctypes.c_int, [_VP]),
    "ea_last_error": (ctypes.c_char_p, [_VP]),
    "ea_advance_init": (ctypes.c_int, [ctypes.POINTER(EAAdvanceCtl), ctypes.c_int32, ctypes.c_int32]),
    "ea_advance_update": (ctypes.c_int32, [ctypes.POINTER(EAAdvanceCtl), ctypes.c_double, ctypes.c_double,
                                           ctypes.c_double, ctypes.c_double]),
    "ea_advance_for_stage": (ctypes.c_int32, [ctypes.POINTER(EAAdvanceCtl), ctypes.c_int32]),
    "ea_predict": (ctypes.c_int, [ctypes.POINTER(EAProfile), ctypes.c_int32, ctypes.c_int32,
                                  ctypes.POINTER(EAGpuPrediction), ctypes.POINTER(ctypes.c_double),
                                  ctypes.POINTER(ctypes.c_double)]),
    "ea_tune": (ctypes.c_int, [ctypes.POINTER(EAProfile), ctypes.POINTER(ctypes.c_int32), ctypes.c_int32,
                               ctypes.POINTER(ctypes.c_int32), ctypes.c_int32, ctypes.c_double, ctypes.c_int32,
                               ctypes.POINTER(ctypes.c_int32), ctypes.POINTER(ctypes.c_int32),
                               ctypes.POINTER(ctypes.c_double)]),
    "ea_schedule": (ctypes.c_int32, [ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, ctypes.c_int32,
                                     ctypes.POINTER(EAOp), ctypes.c_int32]),
    "ea_chan_create": (ctypes.c_int, [ctypes.c_int32, ctypes.c_int32, ctypes.c_int64, ctypes.c_int32,
                                      ctypes.POINTER(_VP)]),
    "ea_chan_export": (ctypes.c_int, [_VP, ctypes.c_void_p]),
    "ea_chan_connect": (ctypes.c_int, [_VP, ctypes.c_void_p]),
    "ea_chan_pair": (ctypes.c_int, [_VP, _VP]),
    "ea_chan_send": (ctypes.c_int, [_VP, _VP, ctypes.c_int64, _VP]),
    "ea_chan_recv": (ctypes.c_int, [_VP, _VP, ctypes.c_int64, _VP]),
    "ea_chan_count": (ctypes.c_int64, [_VP]),
    "ea_chan_destroy": (ctypes.c_int, [_VP]),
    "ea_chan_last_error": (ctypes.c_char_p, [_VP]),
}

_lib = None


def load_library(path: str = LIB_PATH) -> ctypes.CDLL:
    """Load (once) and type the C ABI.  Raises LibraryNotBuilt if absent."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise LibraryNotBuilt(f"{path} not found: run `python -m paper_conf_ppopp_chen0qz23_b200.build` "
                              "(or __graft_entry__.build()); there is no CPU fallback")
    try:
        import torch  # noqa: F401  -- map torch's libnccl.so.2 first so one NCCL is loaded
    except Exception:
        pass
    lib = ctypes.CDLL(path, mode=ctypes.RTLD_GLOBAL)
    for name, (res, args) in SIGNATURES.items():
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    if lib.ea_abi_version() != ABI_VERSION:
        raise LibraryNotBuilt(f"ABI version mismatch: library {lib.ea_abi_version()} vs binding {ABI_VERSION}")
    _lib = lib
    return lib


def last_error(handle=None) -> str:
    return (load_library().ea_last_error(handle) or b"").decode()


def _check(status: int, handle=None):
    if status != EA_OK:
        raise EAError(status, last_error(handle))


def get_unique_id() -> bytes:
    buf = (ctypes.c_uint8 * UNIQUE_ID_BYTES)()
    _check(load_library().ea_get_unique_id(buf))
    return bytes(buf)


def schedule(K: int, M: int, stage: int, advance: int) -> List[Tuple[str, int]]:
    """Advance-forward order of `stage` (0-based) as [('F'|'B', micro_batch)]."""
    lib = load_library()
    cap = max(2 * M, 0)
    out = (EAOp * max(cap, 1))()
    n = lib.ea_schedule(K, M, stage, advance, out, cap)
    if n < 0:
        raise EAError(-n, f"ea_schedule(K={K}, M={M}, stage={stage}, advance={advance}) rejected")
    return [("F" if out[i].kind == 0 else "B", out[i].micro_batch) for i in range(n)]


def _make_profile(m, n, dt, phi, t_gpu, t_comm, f_mod, f_dat):
    """Marshal a profile (sequences / numpy arrays) into an EAProfile; the
    returned tuple keeps the ctypes buffers alive."""
    K = len(t_gpu)
    rows = [list(map(float, r)) for r in phi] if len(phi) else [[] for _ in range(K)]
    S = len(rows[0]) if rows else 0
    if len(rows) != K or any(len(r) != S for r in rows):
        raise ValueError("phi must be K rows of equal length")
    arr = lambda v: (ctypes.c_double * max(len(v), 1))(*map(float, v))
    flat = arr([x for r in rows for x in r])
    bufs = [flat, arr(t_gpu), arr(t_comm), arr(f_mod), arr(f_dat)]
    prof = EAProfile(K, int(m), int(n), S, float(dt), *[ctypes.cast(b, ctypes.POINTER(ctypes.c_double)) for b in bufs])
    return prof, bufs


def predict(m, n, dt, phi, t_gpu, t_comm, f_mod, f_dat, m_star, n_star):
    """ea_predict: per-GPU predictions (list of dicts), iteration time, peak memory."""
    prof, _keep = _make_profile(m, n, dt, phi, t_gpu, t_comm, f_mod, f_dat)
    out = (EAGpuPrediction * prof.n_gpus)()
    it, pk = ctypes.c_double(), ctypes.c_double()
    st = load_library().ea_predict(ctypes.byref(prof), int(m_star), int(n_star), out, ctypes.byref(it),
                                   ctypes.byref(pk))
    if st != EA_OK:
        raise EAError(st, "ea_predict rejected the profile or (m*, n*)")
    per = [{f: getattr(o, f) for f, _ in EAGpuPrediction._fields_} for o in out]
    return per, it.value, pk.value


def tune(m, n, dt, phi, t_gpu, t_comm, f_mod, f_dat, m_cands, n_cands, mem_limit, objective="throughput"):
    """ea_tune: (m*, n*, iteration time) or None if no candidate fits mem_limit."""
    prof, _keep = _make_profile(m, n, dt, phi, t_gpu, t_comm, f_mod, f_dat)
    mc = (ctypes.c_int32 * len(m_cands))(*m_cands)
    nc = (ctypes.c_int32 * len(n_cands))(*n_cands)
    bm, bn, bt = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_double()
    st = load_library().ea_tune(ctypes.byref(prof), mc, len(m_cands), nc, len(n_cands), float(mem_limit),
                                {"throughput": 0, "time": 1}[objective], ctypes.byref(bm), ctypes.byref(bn),
                                ctypes.byref(bt))
    if st == EA_ESTATE:
        return None
    if st != EA_OK:
        raise EAError(st, "ea_tune rejected its arguments")
    return bm.value, bn.value, bt.value


def _stream_ptr(stream) -> Optional[int]:
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return stream.cuda_stream


def _ptr(t, what: str) -> int:
    import torch
    if not isinstance(t, torch.Tensor) or t.dtype != torch.float32 or not t.is_cuda or not t.is_contiguous():
        raise TypeError(f"{what} must be a contiguous float32 CUDA tensor")
    return t.data_ptr()


def _numel(t, want: int, what: str):
    """The C ABI takes bare pointers: a tensor of the wrong size would be read or written past its end."""
    if t.numel() != want:
        raise ValueError(f"{what} has {t.numel()} elements, the library expects {want}")


def _host_ptr(t, what: str) -> int:
    import torch
    if not isinstance(t, torch.Tensor) or t.dtype != torch.float32 or t.is_cuda or not t.is_contiguous():
        raise TypeError(f"{what} must be a contiguous float32 CPU tensor (pinned for asynchronous copies)")
    return t.data_ptr()


class Channel:
    """One end of a point-to-point activation channel (``ea_chan_*``, row f2): role "send" or "recv", a ring
    of `slots` messages of at most `slot_bytes` on `device`.  Wire the two ends with ``export()`` /
    ``connect(peer_handle)`` across processes, or ``Channel.pair(send_end, recv_end)`` in one process.
    ``send(t)`` / ``recv(t)`` enqueue on `stream` (default: the current stream); the host never waits."""

    def __init__(self, role: str, slot_bytes: int, slots: int, device: Optional[int] = None):
        import torch
        self._lib = load_library()
        self.role = role
        self.slot_bytes, self.slots = int(slot_bytes), int(slots)
        self.device = torch.cuda.current_device() if device is None else int(device)
        h = ctypes.c_void_p()
        st = self._lib.ea_chan_create(self.device, {"send": 0, "recv": 1}[role], self.slot_bytes, self.slots,
                                      ctypes.byref(h))
        if st != EA_OK:
            raise EAError(st, (self._lib.ea_chan_last_error(None) or b"").decode())
        self._h = h

    def _check(self, st):
        if st != EA_OK:
            raise EAError(st, (self._lib.ea_chan_last_error(self._h) or b"").decode())

    def export(self) -> bytes:
        buf = (ctypes.c_uint8 * CHAN_HANDLE_BYTES)()
        self._check(self._lib.ea_chan_export(self._h, buf))
        return bytes(buf)

    def connect(self, peer_handle: bytes):
        if len(peer_handle) != CHAN_HANDLE_BYTES:
            raise ValueError(f"peer handle must be {CHAN_HANDLE_BYTES} bytes")
        self._check(self._lib.ea_chan_connect(self._h,
                                              (ctypes.c_uint8 * CHAN_HANDLE_BYTES).from_buffer_copy(peer_handle)))

    @staticmethod
    def pair(send_end: "Channel", recv_end: "Channel"):
        send_end._check(send_end._lib.ea_chan_pair(send_end._h, recv_end._h))

    @staticmethod
    def _buf(t):
        import torch
        if not isinstance(t, torch.Tensor) or not t.is_cuda or not t.is_contiguous():
            raise TypeError("channel buffers must be contiguous CUDA tensors")
        return t.data_ptr(), t.numel() * t.element_size()

    def send(self, t, stream=None):
        p, n = self._buf(t)
        self._check(self._lib.ea_chan_send(self._h, p, n, _stream_ptr(stream)))

    def recv(self, t, stream=None):
        p, n = self._buf(t)
        self._check(self._lib.ea_chan_recv(self._h, p, n, _stream_ptr(stream)))

    @property
    def count(self) -> int:
        return int(self._lib.ea_chan_count(self._h))

    def close(self):
        if getattr(self, "_h", None):
            self._lib.ea_chan_destroy(self._h)
            self._h = None

    def __del__(self):  # pragma: no cover
        # not at interpreter shutdown: ea_chan_destroy synchronises the device, which would never return if a
        # stream still waits for a message from a peer that is gone (the process teardown frees the buffer)
        import sys
        if sys.is_finalizing():
            return
        try:
            self.close()
        except Exception:
            pass


class ElasticAveraging:
    """Handle over ``ea_init`` for the stages this process hosts.

    stage_params: P_s per hosted stage.  alpha defaults to 1/N.
    layout "colocated": all N replicas of a stage on this GPU; "spread": one
    replica per rank, world == N, center sharded (needs ``nccl_id``)."""

    def __init__(self, stage_params: Sequence[int], n_pipelines: int, *, alpha: Optional[float] = None,
                 beta: float = 0.0, rho: float = 1.0, lr: float = 0.05, momentum: float = 0.0,
                 weight_decay: float = 0.0, nesterov: bool = False, layout: str = "colocated", rank: int = 0,
                 world: int = 1, device: Optional[int] = None, kernel_variant: str = "auto",
                 nccl_id: Optional[bytes] = None, optimizer: str = "sgd", betas=(0.9, 0.999), eps: float = 1e-8,
                 exchange: str = "nccl", staleness: int = 0, asgd_lambd: float = 1e-4, asgd_alpha: float = 0.75,
                 asgd_t0: float = 1e6):
        import torch
        self._lib = load_library()
        self.n = int(n_pipelines)
        self.stage_params = [int(p) for p in stage_params]
        self.layout = layout
        if device is None:
            device = torch.cuda.current_device()
        self.device = int(device)
        self._sp = (ctypes.c_int64 * len(self.stage_params))(*self.stage_params)
        self.optimizer = optimizer
        cfg = EAConfig(self.n, len(self.stage_params), self._sp,
                       1.0 / self.n if alpha is None else float(alpha), float(beta), float(rho), float(lr),
                       float(momentum), float(weight_decay), int(bool(nesterov)), LAYOUTS[layout], int(rank),
                       int(world), self.device, VARIANTS[kernel_variant], OPTIMIZERS[optimizer],
                       float(betas[0]), float(betas[1]), float(eps), EXCHANGES[exchange], int(staleness),
                       float(asgd_lambd), float(asgd_alpha), float(asgd_t0))
        self._cfg = cfg
        self.rank, self.world = int(rank), int(world)
        idbuf = None
        if nccl_id is not None:
            if len(nccl_id) != UNIQUE_ID_BYTES:
                raise ValueError("nccl_id must be 128 bytes")
            idbuf = (ctypes.c_uint8 * UNIQUE_ID_BYTES).from_buffer_copy(nccl_id)
        h = ctypes.c_void_p()
        _check(self._lib.ea_init(ctypes.byref(cfg), idbuf, ctypes.byref(h)))
        self._h = h

    # -- queries
    def center_capacity(self, stage: int) -> int:
        v = self._lib.ea_center_capacity(self._h, stage)
        if v < 0:
            raise EAError(EA_EINVAL, f"bad stage {stage}")
        return v

    def shard_elems(self, stage: int) -> int:
        v = self._lib.ea_shard_elems(self._h, stage)
        if v < 0:
            raise EAError(EA_EINVAL, f"bad stage {stage}")
        return v

    # -- the step
    def _p(self, stage: int) -> int:
        if not 0 <= int(stage) < len(self.stage_params):
            raise EAError(EA_EINVAL, f"stage {stage} out of range")
        return self.stage_params[int(stage)]

    def _check_stage_tensors(self, stage, reps, gs, center):
        want = self.n if self.layout == "colocated" else 1
        if len(reps) != want or len(gs) != want:
            raise ValueError(f"stage {stage}: need {want} replica and gradient tensors, got {len(reps)}/{len(gs)}")
        p = self._p(stage)
        for t in reps:
            _numel(t, p, f"stage {stage} replica")
        for t in gs:
            _numel(t, p, f"stage {stage} gradient")
        _numel(center, self.center_capacity(stage), f"stage {stage} center (ea_center_capacity)")

    def step(self, stage: int, replicas, grads, center, stream=None):
        reps = list(replicas)
        gs = list(grads)
        rp = (ctypes.c_void_p * max(len(reps), 1))(*[_ptr(t, "replica") for t in reps])
        gp = (ctypes.c_void_p * max(len(gs), 1))(*[_ptr(t, "grad") for t in gs])
        self._check_stage_tensors(stage, reps, gs, center)
        _check(self._lib.ea_step(self._h, stage, rp, gp, _ptr(center, "center"), _stream_ptr(stream)), self._h)

    def step_many(self, stages, replicas, grads, centers, stream=None):
        """Several stages in one call (one launch co-located, N <= 8).
        replicas[j] / grads[j]: the tensors of stages[j]; centers[j] its center."""
        stages = [int(s) for s in stages]
        want = self.n if self.layout == "colocated" else 1
        if not (len(replicas) == len(grads) == len(centers) == len(stages)):
            raise ValueError("stages, replicas, grads, centers must have the same length")
        rp, gp = [], []
        for j in range(len(stages)):
            self._check_stage_tensors(stages[j], list(replicas[j]), list(grads[j]), centers[j])
            rp += [_ptr(t, "replica") for t in replicas[j]]
            gp += [_ptr(t, "grad") for t in grads[j]]
        k = max(len(stages), 1)
        st = (ctypes.c_int32 * k)(*stages)
        ra = (ctypes.c_void_p * max(len(rp), 1))(*rp)
        ga = (ctypes.c_void_p * max(len(gp), 1))(*gp)
        ca = (ctypes.c_void_p * k)(*[_ptr(c, "center") for c in centers])
        _check(self._lib.ea_step_many(self._h, len(stages), st, ra, ga, ca, _stream_ptr(stream)), self._h)

    def step_many_host(self, stages, replicas, host_grads, centers, host_centers_out, stream=None):
        """ea_step_many with gradients in (pinned) host tensors and the new
        centers copied back into host tensors; copies and kernels overlap."""
        stages = [int(s) for s in stages]
        rp, gp = [], []
        for j in range(len(stages)):
            self._check_stage_tensors(stages[j], list(replicas[j]), list(host_grads[j]), centers[j])
            _numel(host_centers_out[j], self._p(stages[j]), f"stage {stages[j]} host center output")
            rp += [_ptr(t, "replica") for t in replicas[j]]
            gp += [_host_ptr(t, "host grad") for t in host_grads[j]]
        k = max(len(stages), 1)
        st = (ctypes.c_int32 * k)(*stages)
        ra = (ctypes.c_void_p * max(len(rp), 1))(*rp)
        ga = (ctypes.c_void_p * max(len(gp), 1))(*gp)
        ca = (ctypes.c_void_p * k)(*[_ptr(c, "center") for c in centers])
        oa = (ctypes.c_void_p * k)(*[_host_ptr(c, "host center out") for c in host_centers_out])
        _check(self._lib.ea_step_many_host(self._h, len(stages), st, ra, ga, ca, oa, _stream_ptr(stream)), self._h)

    @staticmethod
    def p2p_connect(handles):
        """Connect in-process EA_XCHG_P2P ranks (handles[q] = rank q)."""
        lib = load_library()
        arr = (ctypes.c_void_p * len(handles))(*[h._h.value for h in handles])
        for h in handles:
            _check(lib.ea_p2p_connect(h._h, arr, len(handles)), h._h)

    def p2p_export(self) -> bytes:
        """This rank's exchange-buffer CUDA IPC handle (64 bytes)."""
        buf = (ctypes.c_uint8 * 64)()
        _check(self._lib.ea_p2p_export(self._h, buf), self._h)
        return bytes(buf)

    def p2p_open(self, handles):
        """Map every rank's exchange buffer from the list of all ranks' handles."""
        blob = b"".join(handles)
        if len(blob) != 64 * self.world:
            raise ValueError("need world x 64-byte handles")
        buf = (ctypes.c_uint8 * len(blob)).from_buffer_copy(blob)
        _check(self._lib.ea_p2p_open(self._h, buf, self.world), self._h)

    def sync(self, stream=None):
        _check(self._lib.ea_sync(self._h, _stream_ptr(stream)), self._h)

    def spread_local(self, stage: int, replica, grad, center, contrib, stream=None):
        p, cap = self._p(stage), self.center_capacity(stage)
        _numel(replica, p, "replica")
        _numel(grad, p, "gradient")
        _numel(center, cap, "center (ea_center_capacity)")
        _numel(contrib, cap, "contribution buffer (ea_center_capacity)")
        _check(self._lib.ea_spread_local(self._h, stage, _ptr(replica, "replica"), _ptr(grad, "grad"),
                                         _ptr(center, "center"), _ptr(contrib, "contrib"), _stream_ptr(stream)),
               self._h)

    def spread_apply(self, stage: int, center_shard, reduced, stream=None):
        k = self.shard_elems(stage)
        _numel(center_shard, k, "center shard (ea_shard_elems)")
        _numel(reduced, k, "reduced shard (ea_shard_elems)")
        _check(self._lib.ea_spread_apply(self._h, stage, _ptr(center_shard, "center_shard"),
                                         _ptr(reduced, "reduced"), _stream_ptr(stream)), self._h)

    # -- optimizer state
    def state(self, stage: int, replica: int, slot: int = 0):
        """Zero-copy torch view of library-owned optimizer state: slot 0 = SGD
        momentum / Adam first moment / ASGD average ax, slot 1 = Adam second moment,
        SLOT_CENTER_PREV = the stale center x~_{t-1} (staleness 1, replica 0)."""
        ptr = ctypes.c_void_p()
        _check(self._lib.ea_get_state(self._h, stage, replica, slot, ctypes.byref(ptr)), self._h)
        return _device_view(ptr.value, self.stage_params[stage], self.device)

    def momentum(self, stage: int, replica: int):
        return self.state(stage, replica, 0)

    def set_state(self, stage: int, replica: int, src, slot: int = 0, stream=None):
        _numel(src, self._p(stage), "state source")
        _check(self._lib.ea_set_state(self._h, stage, replica, slot, _ptr(src, "state"), _stream_ptr(stream)),
               self._h)

    def set_momentum(self, stage: int, replica: int, src, stream=None):
        self.set_state(stage, replica, src, 0, stream)

    def get_step(self, stage: int) -> int:
        t = ctypes.c_int64()
        _check(self._lib.ea_get_step(self._h, stage, ctypes.byref(t)), self._h)
        return t.value

    def set_step(self, stage: int, step: int):
        _check(self._lib.ea_set_step(self._h, stage, int(step)), self._h)

    def set_hyper(self, **kw):
        """Change hyper-parameters (alpha, beta, rho, lr, momentum, weight_decay,
        nesterov, beta1, beta2, eps, asgd_lambd, asgd_alpha, asgd_t0) for the steps enqueued afterwards."""
        cfg = EAConfig.from_buffer_copy(self._cfg)
        for k, v in kw.items():
            if k not in ("alpha", "beta", "rho", "lr", "momentum", "weight_decay", "nesterov", "beta1", "beta2",
                         "eps", "asgd_lambd", "asgd_alpha", "asgd_t0"):
                raise KeyError(k)
            setattr(cfg, k, int(bool(v)) if k == "nesterov" else float(v))
        _check(self._lib.ea_set_hyper(self._h, ctypes.byref(cfg)), self._h)
        self._cfg = cfg

    def close(self):
        if getattr(self, "_h", None) is not None and self._h.value:
            self._lib.ea_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()


def _device_view(ptr: int, n: int, device: int):
    """Zero-copy float32 torch view of library-owned device memory."""
    import torch

    class _Arr:
        __cuda_array_interface__ = {"shape": (n,), "typestr": "<f4", "data": (ptr, False), "version": 3,
                                    "strides": None}

    return torch.as_tensor(_Arr(), device=f"cuda:{device}")
