#!/usr/bin/env python
"""Benchmark of the elastic-averaging step (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

One "step" = one elastic-averaging iteration over every stage of the
workload (rows a1-a8 of SURVEY §8): N=1 runs configs[1] (C2: ResNet-50-sized
25M params, K=4 stages, N=4 pipelines, all replicas co-located on the GPU);
N>1 (torchrun, one rank per GPU) runs the spread layout with N pipelines
(C3 for 2/4 GPUs, C4 for 8) -- one replica of every stage per GPU, the
center sharded and exchanged by NCCL reduce-scatter / all-gather.

value = replica-params/s = (pipelines x params) / step time, whole job,
inputs resident in HBM, timed with CUDA events (max over ranks).  `e2e`
repeats the measurement through the same API with the gradients coming
from pinned HOST memory and the new center read back every step.
`--impl reference` times the float64 CPU oracle (the only reference that
exists: the paper ships no code) on a bounded per-step sample.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "elastic-avg step params/sec and HBM/NVLink GB/s (% roofline) at 1/2/4/8 B200"
_JSON_OUT = None


def emit(obj):
    out = _JSON_OUT or sys.stdout
    out.write(json.dumps(obj) + "\n")
    out.flush()
UNIT = "replica-params/s"
MODE = "combined"   # rho=1, beta=N*alpha, alpha=1/N; every mode moves the same bytes


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=1000)
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--impl", choices=("ours", "reference"), default="ours")
    ap.add_argument("--variant", choices=("auto", "regloop", "laneshfl", "bulkpipe", "split", "warprep", "warpspec"), default="auto")
    ap.add_argument("--optimizer", choices=("sgd", "adam", "adamw", "asgd"), default="sgd",
                    help="local optimizer (BASELINE configs: SGD+momentum; Adam(W) and ASGD are row f1)")
    ap.add_argument("--staleness", type=int, choices=(0, 1), default=0,
                    help="1: replicas see the center one step late (row f4; co-located SGD)")
    ap.add_argument("--exchange", choices=("nccl", "p2p"), default="nccl",
                    help="N>1 spread exchange: NCCL RS/AG or the fused peer-memory kernel")
    ap.add_argument("--no-graph", action="store_true",
                    help="launch ea_step_many every step instead of replaying one captured CUDA graph (SGD)")
    ap.add_argument("--per-stage", action="store_true", help="one ea_step launch per stage instead of ea_step_many")
    ap.add_argument("--e2e-steps", type=int, default=20)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    ap.add_argument("--config", default=None, help="override workload key (synth.CONFIGS)")
    ap.add_argument("--n", type=int, default=None, help="override the number of pipelines (co-located, 1 GPU)")
    ap.add_argument("--layout", choices=("auto", "colocated", "spread"), default="auto",
                    help="auto: co-located on 1 GPU, spread on N>1; spread on 1 GPU runs the N>1 code path at world 1")
    return ap.parse_args()


# ----------------------------------------------------------------------------- env
def dist_env():
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


def shared_gpu_test_mode():
    """AVGPIPE_BENCH_SHARED_GPU=1 (tests only): every rank on cuda:0, a gloo control group, the P2P
    exchange wired over CUDA IPC -- exercises the N>1 code path of this script on a one-GPU box, where
    NCCL refuses two ranks on one device.  The ranks' kernels are time-sliced, so its numbers mean nothing."""
    return os.environ.get("AVGPIPE_BENCH_SHARED_GPU") == "1"


def max_over_ranks(ms, dev):
    """Max of a per-rank device time over the process group (NCCL: a device tensor; gloo: host)."""
    import torch
    import torch.distributed as dist
    on_dev = dist.get_backend() == "nccl"
    tt = torch.tensor([ms], device=dev if on_dev else "cpu")
    dist.all_reduce(tt, op=dist.ReduceOp.MAX)
    return float(tt.item())


def measured_peaks():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(path):
        d = json.load(open(path))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy burst)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


NVLINK_PEAK_GBS = 770.0   # B200_PROFILING.md: measured peer copy per direction per GPU (900 GB/s nominal)
NVLINK_PEAK_SOURCE = ("measured reference in /opt/skills/guides/B200_PROFILING.md: peer copy 770 GB/s per direction "
                      "per GPU (8-rank all-reduce busBW 725 GB/s at 1 GiB; 900 GB/s nominal NVLink 5)")


def nccl_debug_setup(rank):
    """NCCL_DEBUG=INFO into a per-rank file (unless the caller set NCCL_DEBUG), so the line can report the
    algorithm / protocol / NVLS NCCL chose for the library's communicator."""
    if os.environ.get("NCCL_DEBUG_FILE"):
        return os.environ["NCCL_DEBUG_FILE"]
    import tempfile
    path = os.path.join(tempfile.gettempdir(), f"avgpipe_nccl_{os.getpid()}_{rank}.log")
    os.environ["NCCL_DEBUG"] = "INFO"
    os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT,TUNING,NVLS")
    os.environ["NCCL_DEBUG_FILE"] = path
    return path


def nccl_debug_summary(path, limit=12):
    """Distinct NCCL INFO lines that name the algorithm / protocol / NVLS / channels of the communicators."""
    if not path or not os.path.exists(path):
        return None
    import re
    keep, seen = [], set()
    pat = re.compile(r"(algo|proto|nvls|collnet|channel \d+/|channels|ring|tree|nranks|p2p/|via )", re.I)
    for line in open(path, errors="replace"):
        if "NCCL INFO" not in line or not pat.search(line):
            continue
        msg = re.sub(r"^.*NCCL INFO ", "", line.strip())
        msg = re.sub(r"0x[0-9a-f]+", "0x..", msg)
        if msg not in seen:
            seen.add(msg)
            keep.append(msg)
        if len(keep) >= limit:
            break
    return keep


class ClockSampler:
    """NVML clocks + throttle reasons sampled DURING the timed region."""
    REASONS = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
               0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
               0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, index: int, period_s: float = 0.001):
        self.samples, self.reasons, self.ok = [], set(), False
        self.max_mhz = None
        self.period = period_s
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception as e:  # pragma: no cover
            self.err = repr(e)

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                bits = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for b, name in self.REASONS.items():
                    if bits & b:
                        self.reasons.add(name)
            except Exception:
                pass
            self._stop.wait(self.period)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *exc):
        self._stop.set()
        if self.ok:
            self.t.join()

    def summary(self):
        if not self.ok or not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                    "samples": len(self.samples)}
        s = sorted(self.samples)
        return {"sm_mhz": s[len(s) // 2], "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons - {"gpu_idle"}),
                "samples": len(s)}


def workload_key(gpus: int, override):
    if override:
        return override
    return {1: "C2", 2: "C3N2", 4: "C3N4", 8: "C4"}.get(gpus, "C4")


# ----------------------------------------------------------------------------- our arm
def stale_fused(n, optimizer, variant):
    """ea_api.cu: under the default variant the stale center runs one launch per <= 8 stages for N <= 4, SGD/ASGD
    N = 5 and Adam(W) N <= 8 (bulk-copy pipeline / lane / warp-per-replica / warp-specialised kernels per N,
    ea_kernels.cu); else the replica loop per stage."""
    two = optimizer in ("adam", "adamw")
    return ((variant == "auto" and (n <= 4 or (n == 5 and not two) or (two and n <= 8)))
            or (variant in ("warprep", "warpspec") and n <= 8))


def kernel_name(variant, optimizer, n, staleness=0):
    """The co-located kernel the library runs (its per-N default, ea_kernels.cu / ea_api.cu)."""
    force_wide = os.environ.get("AVGPIPE_EA_FORCE_WIDE", "")[:1] == "1"   # ea_api.cu measurement knob
    if force_wide:
        return "colocated_wide" + ("<stale>" if staleness else "")
    if staleness:
        if stale_fused(n, optimizer, variant):   # ea_api.cu: x~_{t-1} staged beside x~_t, <= 8 stages per launch
            two = optimizer in ("adam", "adamw")
            kern = ("colocated_warpspec" if variant == "warpspec" or (variant == "auto" and two and n not in (2, 4))
                    else
                    "colocated_warprep" if variant == "warprep" or (not two and n in (2, 5)) else
                    "colocated_laneshfl" if 2 <= n <= 4 else "colocated_bulkpipe")
            return kern + "<stale" + ("" if optimizer == "sgd" else "," + optimizer) + ">"
        return "colocated_wide<stale>"
    two_state = optimizer in ("adam", "adamw")
    if n > 8:
        name = "colocated_wide"
    elif two_state:
        if variant == "auto":
            variant = ("laneshfl" if n == 1 else "regloop" if n <= 3 else "bulkpipe" if n == 4 else
                       "warprep" if n == 5 else "warpspec")
        name = "colocated_" + variant
    elif variant == "auto":   # ea_kernels.cu: SGD / ASGD warp per replica, N = 2 lane kernel, N = 5 warp-specialised
        name = "colocated_laneshfl" if n == 2 else "colocated_warpspec" if n == 5 else "colocated_warprep"
    else:
        name = "colocated_" + variant
    return name + ("" if optimizer == "sgd" else "<" + optimizer + ">")


def colocated_launches(n, k, args, batched):
    """Our kernels per co-located step: the fused kernel(s) plus, for Adam(W) and
    ASGD, the step-counter kernel that precedes each launch."""
    coef = args.optimizer != "sgd"
    two_state = args.optimizer in ("adam", "adamw")
    stale_lane = args.staleness and stale_fused(n, args.optimizer, args.variant)
    force_wide = os.environ.get("AVGPIPE_EA_FORCE_WIDE", "")[:1] == "1"   # ea_api.cu measurement knob
    per_stage = (n > 8 or not batched
                 or (args.staleness and not stale_lane) or force_wide)
    launches = k if per_stage else (k + 7) // 8
    return launches * (2 if coef else 1)


def bytes_colocated(n, p, optimizer="sgd"):
    """Algorithmic HBM bytes of one co-located launch (fp32): read x~ and, per
    replica, x_i, g_i and the optimizer state; write x_i, the state and x~.
    SGD-momentum / ASGD (one state vector): (20 N + 8) P; Adam(W) (two): (28 N + 8) P."""
    return ((28 if optimizer in ("adam", "adamw") else 20) * n + 8) * p


def bytes_spread_local(p, optimizer="sgd"):
    """HBM bytes of the spread local kernel: read x, g, state, x~; write x, state, r:
    28 P (SGD) / 36 P (Adam)."""
    return (36 if optimizer in ("adam", "adamw") else 28) * p


def run_ours(args, rank, world, local):
    import torch
    import torch.distributed as dist
    from paper_conf_ppopp_chen0qz23_b200 import synth
    from paper_conf_ppopp_chen0qz23_b200.binding import ElasticAveraging
    from paper_conf_ppopp_chen0qz23_b200 import parallel

    shared = shared_gpu_test_mode()
    nccl_log = None
    if shared:
        local = 0
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    key = workload_key(world, args.config)
    cfg = synth.CONFIGS[key]
    spread = world > 1 or args.layout == "spread"
    if args.layout == "colocated" and world > 1:
        raise SystemExit("--layout colocated runs one process per GPU with all N replicas: use --gpus 1")
    n = (args.n or cfg.n_pipelines) if not spread else world
    sizes = cfg.stage_sizes
    a, b, r = synth.mode_coeffs(MODE, n)
    lr = synth.LR if args.optimizer in ("sgd", "asgd") else 1e-3
    stream = torch.cuda.current_stream(dev)
    if spread:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ.setdefault("MASTER_PORT", "29531")
        os.environ.setdefault("RANK", str(rank))
        os.environ.setdefault("WORLD_SIZE", str(world))
        if shared:
            if args.exchange != "p2p" and world > 1:
                raise SystemExit("AVGPIPE_BENCH_SHARED_GPU=1 needs --exchange p2p (NCCL refuses two ranks on one GPU)")
            dist.init_process_group("gloo")
            uid = None
        else:
            nccl_log = nccl_debug_setup(rank)
            dist.init_process_group("nccl", device_id=dev)
            uid = parallel.broadcast_unique_id()
        h = ElasticAveraging(sizes, n, alpha=a, beta=b, rho=r, lr=lr, momentum=synth.MOMENTUM,
                             layout="spread", rank=rank, world=world, device=local, nccl_id=uid,
                             optimizer=args.optimizer, exchange=args.exchange, staleness=args.staleness)
        if shared and world > 1:
            parallel.connect_p2p(h)      # IPC handles over the gloo group
        state = []
        for s, p in enumerate(sizes):
            reps, c0, grads = synth.device_state(1, p, dev, seed=1000 * s)   # same center on every rank
            cc = torch.zeros(h.center_capacity(s), device=dev)
            cc[:p] = c0
            state.append((reps, grads, cc))
    else:
        h = ElasticAveraging(sizes, n, alpha=a, beta=b, rho=r, lr=lr, momentum=synth.MOMENTUM,
                             device=local, kernel_variant=args.variant, optimizer=args.optimizer,
                             staleness=args.staleness)
        state = [synth.device_state(n, p, dev, seed=s) for s, p in enumerate(sizes)]
        state = [(reps, grads, c) for (reps, c, grads) in state]
    order = parallel.stage_order(len(sizes))

    batched = not spread and not args.per_stage

    def one_step(evs=None):
        if batched:    # all stages in ONE launch (ea_step_many)
            if evs is not None:
                evs[0][0].record(stream)
            h.step_many(order, [state[s][0] for s in order], [state[s][1] for s in order],
                        [state[s][2] for s in order], stream=stream)
            if evs is not None:
                evs[0][1].record(stream)
            return
        for s in order:
            reps, grads, c = state[s]
            if evs is not None:
                evs[s][0].record(stream)
            h.step(s, reps, grads, c, stream=stream)
            if evs is not None:
                evs[s][1].record(stream)
        if spread:
            h.sync(stream)

    for _ in range(args.warmup):
        one_step()
    torch.cuda.synchronize()
    use_graph = not args.no_graph and not spread and batched
    if use_graph:
        # the whole step as one CUDA graph (no per-step host work at all; Adam's step
        # counter and bias corrections are advanced on the device inside the graph)
        graph = torch.cuda.CUDAGraph()
        cap = torch.cuda.Stream()
        cap.wait_stream(stream)
        with torch.cuda.stream(cap):
            with torch.cuda.graph(graph, stream=cap):
                h.step_many(order, [state[s_][0] for s_ in order], [state[s_][1] for s_ in order],
                            [state[s_][2] for s_ in order], stream=cap)
        torch.cuda.synchronize()

        def one_step(evs=None):  # noqa: F811
            if evs is not None:
                evs[0][0].record(stream)
            graph.replay()
            if evs is not None:
                evs[0][1].record(stream)
        one_step()
        torch.cuda.synchronize()
    if spread:
        dist.barrier()
    # per-launch events for the dominant kernel (co-located: every ea_step is one kernel)
    # spread: events bracket each stage's local kernel (the exchange is on the library's side stream)
    ev = [[(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
           for _ in (range(1) if batched else sizes)] for _ in range(args.steps)]
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with ClockSampler(local) as clk:
        torch.cuda.synchronize()
        t0.record(stream)
        for k in range(args.steps):
            one_step(None if ev is None else ev[k])
        t1.record(stream)
        torch.cuda.synchronize()
    ms = t0.elapsed_time(t1) / args.steps
    if spread:
        ms = max_over_ranks(ms, dev)
    total_params = sum(sizes)
    value = n * total_params / (ms * 1e-3)
    peak, peak_src = measured_peaks()
    out = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True, "scaling": "weak",
           "vs_baseline": None, "dtype": "f32", "data": "synthetic (seeded: x0~N(0,0.02^2), replicas +N(0,1e-3^2), "
                                                        "grads~N(0,1e-2^2); torch.Generator on device)"}
    ws_bytes = (n * 3 + 1) * 4 * total_params if not spread else 5 * 4 * total_params
    out["config"] = {"workload": cfg.name, "n_pipelines": n, "n_stages": len(sizes), "params": total_params,
                     "stage_params": sizes, "layout": "spread" if spread else "colocated", "mode": MODE,
                     "exchange": args.exchange if spread else None,
                     "nccl_env": {k: v for k, v in os.environ.items() if k.startswith("NCCL_")} if spread else None,
                     "optimizer": "sgd-momentum(0.9)" if args.optimizer == "sgd" else args.optimizer,
                     "kernel": args.variant,
                     "knobs": {k: v for k, v in os.environ.items() if k.startswith("AVGPIPE_EA_")} or None,
                     "l2": f"no flush: working set {ws_bytes / 1e9:.2f} GB per GPU > 126 MB L2"}
    if not spread:
        step_bytes = sum(bytes_colocated(n, p, args.optimizer) + 8 * p * args.staleness for p in sizes)
        launches_per_step = 1 if batched else len(sizes)
        kern_ms = [ev[k][j][0].elapsed_time(ev[k][j][1]) for k in range(args.steps) for j in range(launches_per_step)]
        # per launch (batched: all stages; per-stage: averaged over the equal-sized stages)
        per_launch_bytes = step_bytes / launches_per_step
        avg_ms = sum(kern_ms) / len(kern_ms)
        achieved = per_launch_bytes / (avg_ms * 1e-3) / 1e9
        out["gbps"] = step_bytes / (ms * 1e-3) / 1e9
        q = sorted(kern_ms)
        pct = {f"p{k}": q[min(len(q) - 1, len(q) * k // 100)] for k in (10, 50, 90)}
        out["roofline"] = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                           "frac": achieved / peak,
                           "traffic": traffic_from_profiles(cfg.name if n == cfg.n_pipelines else f"{cfg.name}@N{n}",
                                                            kernel_name(args.variant, args.optimizer, n,
                                                                        args.staleness)),
                           "launch_ms_pct": pct,
                           "kernel": kernel_name(args.variant, args.optimizer, n, args.staleness),
                           "bytes_per_launch": per_launch_bytes, "avg_launch_ms": avg_ms,
                           "share_of_step": sum(kern_ms) / args.steps / ms, "peak_source": peak_src}
        out["gpu_launches"] = args.steps * colocated_launches(n, len(sizes), args, batched)
        out["config"]["launch"] = ("CUDA graph replay of ea_step_many (1 kernel/step)" if use_graph
                                   else "ea_step_many (1 launch/step)" if batched else "ea_step per stage")
    else:
        step_bytes = sum(bytes_spread_local(p, args.optimizer) for p in sizes)
        nv_bytes = sum(2 * (n - 1) / n * 4 * h.center_capacity(s) for s in range(len(sizes)))
        out["gbps"] = step_bytes / (ms * 1e-3) / 1e9
        nv_gbs = nv_bytes / (ms * 1e-3) / 1e9
        nvlink = {"bound": "nvlink", "achieved": nv_gbs, "peak": NVLINK_PEAK_GBS, "unit": "GB/s",
                  "frac": nv_gbs / NVLINK_PEAK_GBS, "traffic": None, "peak_source": NVLINK_PEAK_SOURCE,
                  "traffic_note": "ncu has no NVLink byte counter on a one-GPU capture; the bytes are the "
                                  "algorithmic (ring busBW) volume",
                  "bytes_per_step": nv_bytes,
                  "note": "whole step: per-GPU NVLink bytes 2(N-1)/N*4*P_pad (ring busBW convention) / step time"}
        # the local kernel (rows a1-a4; p2p: + the pushes into the owners' inboxes) runs on the caller's stream
        # between each stage's events; the exchange runs on the library's side stream, outside them
        kern = ("p2p_push" if args.exchange == "p2p" else "spread_bulkpipe") + \
            ("" if args.optimizer == "sgd" else "<" + args.optimizer + ">")
        kern_ms = [ev[k][j][0].elapsed_time(ev[k][j][1]) for k in range(args.steps) for j in range(len(sizes))]
        avg_ms = sum(kern_ms) / len(kern_ms)
        if args.exchange == "p2p":   # the push kernel reads/writes the padded vectors (28 / 36 B per element)
            launch_bytes = [bytes_spread_local(h.center_capacity(s), args.optimizer) for s in range(len(sizes))]
        else:
            launch_bytes = [bytes_spread_local(p, args.optimizer) for p in sizes]
        per_launch_bytes = sum(launch_bytes) / len(sizes)
        achieved = per_launch_bytes / (avg_ms * 1e-3) / 1e9
        local = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                 "traffic": traffic_from_profiles(cfg.name, kern), "kernel": kern,
                 "bytes_per_launch": per_launch_bytes, "avg_launch_ms": avg_ms,
                 "share_of_step": sum(kern_ms) / args.steps / ms, "peak_source": peak_src}
        if world == 1:
            out["roofline"] = local     # no NVLink traffic at world 1: the local kernel is the bound
            local["note"] = ("world 1: each stage's local kernel is timed while the previous stage's exchange "
                             "(side stream) shares HBM")
            # world 1 the exchange is local HBM work too: NCCL's reduce-scatter is a copy (8 B), the shard update
            # 12 B, the in-place all-gather nothing; p2p phase B 16 B; the stale snapshot + 8 B per element
            xb = (20 if args.exchange == "nccl" else 16) + 8 * args.staleness
            sb = step_bytes + sum(xb * h.center_capacity(s) for s in range(len(sizes)))
            out["step_hbm"] = {"bytes_per_step": sb, "achieved": sb / (ms * 1e-3) / 1e9, "peak": peak,
                               "frac": sb / (ms * 1e-3) / 1e9 / peak, "unit": "GB/s",
                               "note": f"whole step at world 1: local kernels 28 B + exchange {xb} B per element, "
                                       "both streams sharing HBM"}
        else:
            out["roofline"] = nvlink
            out["local_kernel_roofline"] = local
        if args.exchange == "nccl":
            out["config"]["nccl"] = nccl_debug_summary(nccl_log)
        # ours per stage: the local kernel + the shard update (NCCL) or the exchange kernel (p2p), and the
        # step-counter kernel when something on the device consumes the step count (Adam/ASGD, the p2p epoch)
        per_stage = 2 + (1 if (args.optimizer != "sgd" or args.exchange == "p2p") else 0)
        out["gpu_launches"] = args.steps * per_stage * len(sizes)   # NCCL's own kernels excluded
    out["clocks"] = clk.summary()
    if not spread:
        out["copy_gbs_same_box"] = same_box_copy_gbs(dev)
    if not spread and not args.no_e2e:
        out["e2e"] = e2e_colocated(h, state, sizes, n, args, stream, dev, order)
    elif spread and not args.no_e2e:
        out["e2e"] = e2e_spread(h, state, sizes, args, stream, dev, order, rank, world)
    h.close()
    if rank == 0 and not args.no_cpu_baseline:
        # N > 1: one stage-shard (P_s/N elements x N replicas) on rank 0, per-element rate extrapolated
        out["cpu_baseline"] = cpu_baseline(cfg, n, seconds=args.cpu_seconds, shard=world > 1)
    if rank == 0:
        emit(out)
    if spread:
        dist.destroy_process_group()


def same_box_copy_gbs(dev, nbytes=2 << 30, reps=10):
    """torch copy_ of 2 GiB (read + write bytes / best time): this box's copy
    bandwidth, for context next to MEASURED_PEAKS.json (same recipe)."""
    import torch
    a = torch.empty(nbytes // 2, dtype=torch.bfloat16, device=dev)
    b = torch.empty_like(a)
    best = None
    for _ in range(reps + 2):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        b.copy_(a)
        e1.record()
        e1.synchronize()
        t = e0.elapsed_time(e1)
        best = t if best is None else min(best, t)
    del a, b
    torch.cuda.empty_cache()
    return 2 * nbytes / (best * 1e-3) / 1e9


def same_box_h2d_gbs(dev, pinned, reps=5):
    """Pinned host -> device copy bandwidth of this box (best of `reps` copies of
    the given pinned tensor): the PCIe bound of the e2e line."""
    import torch
    d = torch.empty_like(pinned, device=dev)
    best = None
    for _ in range(reps + 1):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        d.copy_(pinned, non_blocking=True)
        e1.record()
        e1.synchronize()
        t = e0.elapsed_time(e1)
        best = t if best is None else min(best, t)
    return pinned.numel() * pinned.element_size() / (best * 1e-3) / 1e9


def traffic_from_profiles(workload, kernel):
    """ncu dram__bytes_read.sum + dram__bytes_write.sum per launch of this exact
    (workload, kernel), from profiles/traffic.json; None when not captured."""
    path = os.path.join(ROOT, "profiles", "traffic.json")
    if not os.path.exists(path):
        return None
    d = json.load(open(path))
    return d.get(f"{workload}|{kernel}", {}).get("dram_bytes_per_launch")


def e2e_colocated(h, state, sizes, n, args, stream, dev, order):
    """Same step through the public API with HOST buffers: ea_step_many_host
    takes the gradients from pinned host memory and writes the new centers
    back to pinned host memory every step (the library pipelines H2D, kernel
    and D2H in 4 Mi-element chunks on its own copy streams)."""
    import torch
    host_g = [[g.cpu().pin_memory() for g in grads] for (_, grads, _) in state]
    host_c = [torch.empty(p, dtype=torch.float32).pin_memory() for p in sizes]

    def step():
        h.step_many_host(order, [state[s][0] for s in order], [host_g[s] for s in order],
                         [state[s][2] for s in order], [host_c[s] for s in order], stream=stream)

    for _ in range(3):
        step()
    torch.cuda.synchronize()
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0.record(stream)
    for _ in range(args.e2e_steps):
        step()
    t1.record(stream)
    torch.cuda.synchronize()
    ms = t0.elapsed_time(t1) / args.e2e_steps
    h2d = 4 * n * sum(sizes)
    pcie = same_box_h2d_gbs(dev, host_g[0][0])
    return {"value": n * sum(sizes) / (ms * 1e-3), "unit": UNIT, "ms_per_step": ms,
            "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": 4 * sum(sizes),
            "h2d_gbs": h2d / (ms * 1e-3) / 1e9, "h2d_gbs_same_box": pcie,
            "pcie_frac": h2d / (ms * 1e-3) / 1e9 / pcie,
            "path": "ea_step_many_host: pinned host grads -> device (chunked, copy stream), fused kernel per chunk, "
                    "center chunks -> pinned host (second copy stream)"}


def e2e_spread(h, state, sizes, args, stream, dev, order, rank, world):
    """Spread layout end to end through the public API: every step each rank
    copies its replica's gradients of every stage from pinned HOST memory
    (non_blocking, on the step stream), runs ea_step per stage (local kernel +
    exchange on the library side stream), joins the exchange (ea_sync) and
    reads its owned center shard of every stage back to pinned host memory.
    Timed with CUDA events on the step stream, max over ranks."""
    import torch
    import torch.distributed as dist
    host_g = [state[s][1][0].cpu().pin_memory() for s in range(len(sizes))]
    shard = [h.shard_elems(s) for s in range(len(sizes))]
    host_c = [torch.empty(shard[s], dtype=torch.float32).pin_memory() for s in range(len(sizes))]

    def step():
        for s in order:
            reps, grads, cc = state[s]
            grads[0].copy_(host_g[s], non_blocking=True)
            h.step(s, reps, grads, cc, stream=stream)
        h.sync(stream)
        for s in order:
            cc = state[s][2]
            host_c[s].copy_(cc[rank * shard[s]:(rank + 1) * shard[s]], non_blocking=True)

    for _ in range(3):
        step()
    torch.cuda.synchronize()
    dist.barrier()
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0.record(stream)
    for _ in range(args.e2e_steps):
        step()
    t1.record(stream)
    torch.cuda.synchronize()
    ms = max_over_ranks(t0.elapsed_time(t1) / args.e2e_steps, dev)
    return {"value": world * sum(sizes) / (ms * 1e-3), "unit": UNIT, "ms_per_step": ms,
            "h2d_bytes_per_step": 4 * world * sum(sizes), "d2h_bytes_per_step": 4 * world * sum(shard),
            "path": "per rank: pinned host grads -> device (non_blocking copy on the step stream), ea_step per "
                    "stage, ea_sync, owned center shards -> pinned host; bytes summed over ranks"}


# ----------------------------------------------------------------------------- oracle (CPU) legs
def _oracle_sample(n, p_sample, seed=0):
    import numpy as np
    from paper_conf_ppopp_chen0qz23_b200 import synth
    reps, c = synth.host_state(n, p_sample, seed=synth.WEIGHT_SEED + seed)
    gs = synth.GradStream(n, p_sample).next()
    return reps, [np.zeros(p_sample, dtype=np.float32) for _ in range(n)], c, gs


def cpu_model():
    """The host CPU's model name (/proc/cpuinfo), reported beside the oracle timings."""
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def cpu_baseline(cfg, n, seconds=10.0, shard=False):
    """The float64 oracle, as it stands (single-threaded numpy), on a bounded
    sample: one full stage of the workload (shard=True, the N>1 lines: one
    stage-shard of P_s/N elements x N replicas, SURVEY §8(d) -- the full C3-C5
    float64 state exceeds host RAM), repeated until `seconds` pass."""
    from oracle.ea_oracle import Hyper, ea_step
    from paper_conf_ppopp_chen0qz23_b200 import synth
    p = cfg.stage_sizes[0] // (n if shard else 1)
    a, b, r = synth.mode_coeffs(MODE, n)
    hp = Hyper(alpha=a, beta=b, rho=r, lr=synth.LR, momentum=synth.MOMENTUM)
    xs, ms, c, g = _oracle_sample(n, p)
    steps, t0 = 0, time.perf_counter()
    while True:
        xs, ms, c = ea_step(xs, ms, c, g, hp)
        steps += 1
        el = time.perf_counter() - t0
        if el >= seconds:
            break
    what = f"stage-shard (P_s/N of {cfg.stage_sizes[0]})" if shard else "stage"
    out = {"value": n * p * steps / el, "unit": UNIT, "cores": 1, "kind": "oracle",
           "sample": f"{steps} oracle steps of one {p}-element {what} x N={n} (float64 numpy, 1 thread), "
                     f"{el:.1f} s", "host_cores_available": len(os.sched_getaffinity(0)), "cpu_model": cpu_model()}
    if shard:
        out["extrapolated"] = ("per-element rate of one stage-shard; the whole job's state does not fit host RAM "
                               "in float64 (SURVEY §8(d))")
    out["all_cores"] = cpu_baseline_all_cores(xs, ms, c, g, hp, seconds=seconds / 2)
    return out


def cpu_baseline_all_cores(xs, ms, c, g, hp, seconds=5.0):
    """The same oracle step, unchanged, called on contiguous element ranges by a
    thread pool with one worker per host core (the update is elementwise over j,
    and numpy's ufuncs release the GIL) -- SURVEY §8(d)'s all-core variant."""
    from concurrent.futures import ThreadPoolExecutor
    from oracle.ea_oracle import ea_step
    cores = len(os.sched_getaffinity(0))
    p, n = len(c), len(xs)
    bounds = [(p * k // cores, p * (k + 1) // cores) for k in range(cores)]

    def part(b):
        a, e = b
        return ea_step([x[a:e] for x in xs], [m[a:e] for m in ms], c[a:e], [gi[a:e] for gi in g], hp)

    steps, t0 = 0, time.perf_counter()
    with ThreadPoolExecutor(max_workers=cores) as pool:
        while True:
            list(pool.map(part, bounds))
            steps += 1
            el = time.perf_counter() - t0
            if el >= seconds:
                break
    return {"value": n * p * steps / el, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": f"{steps} oracle steps of one {p}-element stage x N={n}, split into {cores} element ranges "
                      f"on {cores} threads (float64 numpy), {el:.1f} s"}


REFERENCE_BUDGET_S = 150.0   # the reference arm's timed steps + warm-up stay within a few minutes


def run_reference(args, rank, world):
    """--impl reference: the float64 oracle, as it stands, on host cores; rank 0 only.

    N = 1: the WHOLE workload (every stage, every replica, full size) per step when K + W steps fit
    REFERENCE_BUDGET_S (C2: ~2.3 s per step on one core), else the same leading fraction of every stage.
    N > 1: one stage-shard (P_s/N elements x N replicas) per step, per-element rate extrapolated to the job
    (the full C3-C5 float64 state does not fit host RAM)."""
    if rank != 0:
        return
    import numpy as np
    from oracle.ea_oracle import Hyper, ea_step
    from paper_conf_ppopp_chen0qz23_b200 import synth
    key = workload_key(world, args.config)
    cfg = synth.CONFIGS[key]
    n = cfg.n_pipelines if world == 1 else world
    a, b, r = synth.mode_coeffs(MODE, n)
    hp = Hyper(alpha=a, beta=b, rho=r, lr=synth.LR, momentum=synth.MOMENTUM)
    if world == 1:
        parts = list(cfg.stage_sizes)
    else:
        parts = [cfg.stage_sizes[0] // n]
    states = [_oracle_sample(n, p, seed=s) for s, p in enumerate(parts)]

    def one_step(states, frac=1.0):
        out = []
        for xs, ms, c, g in states:
            if frac < 1.0:
                k = max(1, int(len(c) * frac))
                xk, mk, ck = ea_step([x[:k] for x in xs], [m[:k] for m in ms], c[:k], [gi[:k] for gi in g], hp)
                for x, v in zip(xs, xk):
                    x[:k] = v
                for m, v in zip(ms, mk):
                    m[:k] = v
                c[:k] = ck
                out.append((xs, ms, c, g))
            else:
                xs2, ms2, c2 = ea_step(xs, ms, c, g, hp)
                out.append((xs2, ms2, c2, g))
        return out

    t0 = time.perf_counter()
    states = one_step(states)                # calibration (counts as one warm-up step)
    t_full = time.perf_counter() - t0
    frac = min(1.0, REFERENCE_BUDGET_S / max(t_full * (args.steps + max(args.warmup - 1, 0)), 1e-9))
    for _ in range(max(args.warmup - 1, 0)):
        states = one_step(states, frac)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        states = one_step(states, frac)
    el = time.perf_counter() - t0
    elems = sum(max(1, int(p * frac)) if frac < 1.0 else p for p in parts)
    ms_step = el / args.steps * 1e3
    value = n * elems / (el / args.steps)
    if world == 1 and frac >= 1.0:
        sample = f"the whole workload each step: {len(parts)} stages x {parts[0]} elements x N={n} replicas"
    elif world == 1:
        sample = (f"each step: the leading {frac:.3f} of every stage ({elems} of {sum(parts)} elements) x N={n} "
                  f"replicas (K + W steps of the whole workload exceed {REFERENCE_BUDGET_S:.0f} s)")
    else:
        sample = f"each step: one stage-shard, {parts[0]} elements (P_s/N) x N={n} replicas; rate extrapolated"
    same = world == 1 and frac >= 1.0
    out = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "weak",
           "vs_baseline": None, "dtype": "f64", "data": "synthetic (seeded numpy PCG64, synth.host_state)",
           "impl": "reference",
           "config": {"workload": cfg.name, "n_pipelines": n, "params_per_step_sample": elems, "mode": MODE,
                      "same_config": same},
           "cpu_baseline": {"value": value, "unit": UNIT, "cores": 1, "kind": "oracle",
                            "sample": sample + " (float64 numpy, 1 thread)", "cpu_model": cpu_model(),
                            "host_cores_available": len(os.sched_getaffinity(0))},
           "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
           "gpu_launches": 0}
    if not same:
        out["cpu_baseline"]["extrapolated"] = "per-element rate of the sample"
    emit(out)


def main():
    args = parse()
    # exactly ONE JSON line on stdout: whatever native libraries print there (NCCL's
    # version banner at communicator init, ...) goes to stderr instead
    json_out = os.fdopen(os.dup(1), "w")
    sys.stdout.flush()
    os.dup2(2, 1)
    global _JSON_OUT
    _JSON_OUT = json_out
    rank, world, local = dist_env()
    if world != args.gpus and rank == 0:
        print(f"note: WORLD_SIZE={world} but --gpus={args.gpus}; using WORLD_SIZE", file=sys.stderr)
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    run_ours(args, rank, world, local)


if __name__ == "__main__":
    main()
