"""Parity helpers: run the CUDA path (through the C ABI) and the float64
oracle on the same seeded inputs and compare with the c13 metric.

c13: for each tensor T,
    max_j |T_gpu[j] - T_ref[j]| / max(|T_ref[j]|, rms(T_ref))  <=  1e-5
after the run.  The rms floor is what makes the north star's "max relative
error 1e-5" attainable in fp32 at all: a pure elementwise ratio is dominated by
elements that pass near zero (DESIGN.md derives the budget: ~100 steps x a few
fp32 roundings of 6e-8 each -> ~1.5e-6 measured in an fp32 numpy model).
"""
from __future__ import annotations

import os

import numpy as np

from oracle.ea_oracle import (Hyper, ea_step, ea_step_adam, ea_step_adam_stale, ea_step_asgd, ea_step_asgd_stale,
                               ea_step_stale)
from paper_conf_ppopp_chen0qz23_b200 import synth

TOL = 1e-5

# Worst c13 error seen by rel_err during the running test (tests/conftest.py resets it per test and appends it,
# with the test id, to the margins log: AVGPIPE_PARITY_LOG, default gpurun_out/parity_margins.jsonl on a GPU).
WORST = {"err": None}


def rel_err(gpu: np.ndarray, ref: np.ndarray) -> float:
    gpu = np.asarray(gpu, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    if ref.size == 0:
        return 0.0
    floor = float(np.sqrt(np.mean(ref * ref)))
    denom = np.maximum(np.abs(ref), floor if floor > 0 else 1e-30)
    e = float(np.max(np.abs(gpu - ref) / denom))
    WORST["err"] = e if WORST["err"] is None else max(WORST["err"], e)
    return e


def to_np(t) -> np.ndarray:
    return t.detach().cpu().numpy()


def f32(v: float) -> float:
    """The value a float32 field of ea_config actually carries (AVGPIPE_PARITY_F64_HYPER=1: the unrounded value,
    for measuring what the rounding is worth -- profiles/r02_parity_margins*.jsonl)."""
    if os.environ.get("AVGPIPE_PARITY_F64_HYPER") == "1":
        return float(v)
    return float(np.float32(v))


ASGD_TEST = dict(asgd_lambd=1e-2, asgd_alpha=0.75, asgd_t0=5.0)   # averaging starts within a short test


def hyper(n, mode, alpha=None, lr=synth.LR, momentum=synth.MOMENTUM, wd=0.0, nesterov=False, betas=(0.9, 0.999),
          eps=1e-8, asgd=ASGD_TEST):
    """Oracle hyper-parameters equal to what the ABI carries (reading c12: the
    oracle consumes the same fp32 values upcast): alpha, beta, rho, lr,
    momentum, weight_decay, eps are float32 fields; beta1/beta2 and the ASGD
    fields are double.  float32(0.01) is 2.2e-8 relative below 0.01,
    float32(1e-3) 4.7e-8 above, float32(0.9) 2.6e-8 below.  Mostly harmless
    (lr enters Delta linearly: ~1e-7 of rms(x) after 100 steps), except for
    Adam with L2 decay where g' = g + lambda*x nearly cancels (|g'| <~ eps):
    there Delta has slope lr/eps = 1e5 in g', and the 4.5e-12 the rounding of
    lambda moves lambda*x becomes ~2e-5 of rms(x) -- measured: the C2 full-size
    Adam test fails its first step with unrounded values
    (profiles/r02_parity_margins.md)."""
    a, b, r = synth.mode_coeffs(mode, n, alpha)
    return Hyper(alpha=f32(a), beta=f32(b), rho=f32(r), lr=f32(lr), momentum=f32(momentum), weight_decay=f32(wd),
                 nesterov=nesterov, beta1=betas[0], beta2=betas[1], eps=f32(eps), **asgd)


def asgd_kw(hp):
    """ElasticAveraging keyword arguments carrying hp's ASGD fields."""
    return dict(asgd_lambd=hp.asgd_lambd, asgd_alpha=hp.asgd_alpha, asgd_t0=hp.asgd_t0)


class OracleStage:
    """float64 oracle state of one stage (optimizer 'sgd' | 'adam' | 'adamw' | 'asgd'; ms holds the
    momentum / first moment / ASGD average)."""

    def __init__(self, reps, center, optimizer="sgd", staleness=0):
        self.xs = [np.asarray(x, dtype=np.float64) for x in reps]
        self.ms = [np.zeros_like(self.xs[0]) for _ in reps]
        self.vs = [np.zeros_like(self.xs[0]) for _ in reps]
        self.c = np.asarray(center, dtype=np.float64)
        self.c_prev = self.c.copy()        # x~_{-1} := x~_0 (c28)
        self.opt = optimizer
        self.staleness = staleness
        self.t = 0

    def step(self, grads, hp):
        self.t += 1
        if self.staleness == 1 and self.opt == "sgd":
            self.xs, self.ms, self.c, self.c_prev = ea_step_stale(self.xs, self.ms, self.c, self.c_prev, grads, hp)
        elif self.staleness == 1 and self.opt == "asgd":
            self.xs, self.ms, self.c, self.c_prev = ea_step_asgd_stale(self.xs, self.ms, self.c, self.c_prev, grads,
                                                                       hp, self.t)
        elif self.staleness == 1:
            self.xs, self.ms, self.vs, self.c, self.c_prev = ea_step_adam_stale(
                self.xs, self.ms, self.vs, self.c, self.c_prev, grads, hp, self.t, decoupled=self.opt == "adamw")
        elif self.opt == "sgd":
            self.xs, self.ms, self.c = ea_step(self.xs, self.ms, self.c, grads, hp)
        elif self.opt == "asgd":
            self.xs, self.ms, self.c = ea_step_asgd(self.xs, self.ms, self.c, grads, hp, self.t)
        else:
            self.xs, self.ms, self.vs, self.c = ea_step_adam(self.xs, self.ms, self.vs, self.c, grads, hp, self.t,
                                                             decoupled=self.opt == "adamw")
