"""Oracle of AvgPipe's profiling-based tuning predictor (§5.2, Eqs. (1)-(8)).

TEST INFRASTRUCTURE ONLY -- see ``oracle/__init__.py``.

From one profiled setting (M = m micro-batches, N = n pipelines) the predictor
estimates, for a candidate (m*, n*), per GPU k of K:

  Eq. (2)  T_gpu*  = (m* n)/(m n*) * ( T_gpu + Int max( (m n*)/(m* n) phi(t) - 1, 0 ) dt )
  Eq. (4)  T_com*  = n*/(m* n) TT + (m*-1)/m* * max( (n*/n) TT - T_gpu*, 0 )
  Eq. (5)  T_bub*  = T_up* + T_down*
  Eq. (6)  T_up^1* = 0,  T_up^k*   = T_up^{k-1}*   + ( TT^{k-1}* + T_gpu^{k-1}* ) / m*
  Eq. (7)  T_down^K* = 0, T_down^k* = T_down^{k+1}* + ( TT^{k+1}* + T_gpu^{k+1}* ) / m*
  Eq. (1)  T*      = T_gpu* + T_com* + T_bub*
  Eq. (8)  F*      = (n*/n) F_mod + (m n*)/(m* n) F_dat
and picks "the setting that achieves the optimal prediction of performance and
satisfies the given memory constraint".

(phi = GPU utilisation curve, TT = total communication time of the
profile, F_mod / F_dat = model / data footprints.)

Readings (DESIGN.md c22-c26):
  c22  phi^k is given as samples at a uniform step dt over the profiled window;
       the integral of Eq. (2) is the left Riemann sum of the sampled curve.
  c23  TT^{k-1}* in Eqs. (6)/(7) is the predicted total communication time,
       (n*/n) TT^{k-1} (as in Eq. (4)).
  c24  the iteration time of a setting is max_k T^k*; "optimal" = the highest
       throughput n*/T* (n* batches per iteration), ties broken by the
       lower peak memory, then the smaller (n*, m*).  Objective "time" =
       the lowest T*.
  c25  memory feasibility: max_k F^k* <= limit.
  c26  the profile must not saturate: phi in [0, 1] is accepted.
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import List, Sequence

import numpy as np


@dataclass
class Profile:
    m: int                    # profiled micro-batches per batch
    n: int                    # profiled parallel pipelines
    dt: float                 # seconds per utilisation sample
    phi: np.ndarray           # K x S utilisation samples in [0, 1]
    t_gpu: Sequence[float]    # K: T_gpu^k
    t_comm: Sequence[float]   # K: total communication time TT^k
    f_mod: Sequence[float]    # K: F_mod^k
    f_dat: Sequence[float]    # K: F_dat^k

    @property
    def K(self) -> int:
        return len(self.t_gpu)


def t_gpu_star(prof: Profile, k: int, m_star: int, n_star: int) -> float:
    """Eq. (2) for GPU k (0-based)."""
    c = (prof.m * n_star) / (m_star * prof.n)
    phi = np.asarray(prof.phi[k], dtype=np.float64)
    extra = float(np.sum(np.maximum(c * phi - 1.0, 0.0)) * prof.dt)      # c22
    return (m_star * prof.n) / (prof.m * n_star) * (prof.t_gpu[k] + extra)


def tt_star(prof: Profile, k: int, n_star: int) -> float:
    """(TT^k)* = (n*/n) TT^k (text before Eq. (4))."""
    return n_star / prof.n * prof.t_comm[k]


def t_com_star(prof: Profile, k: int, m_star: int, n_star: int, tg_star: float) -> float:
    """Eq. (4)."""
    return (n_star / (m_star * prof.n)) * prof.t_comm[k] + \
        (m_star - 1) / m_star * max(tt_star(prof, k, n_star) - tg_star, 0.0)


def memory_star(prof: Profile, k: int, m_star: int, n_star: int) -> float:
    """Eq. (8)."""
    return n_star / prof.n * prof.f_mod[k] + (prof.m * n_star) / (m_star * prof.n) * prof.f_dat[k]


def predict(prof: Profile, m_star: int, n_star: int) -> dict:
    """Per-GPU predictions and the iteration time / peak memory (c24, c25)."""
    K = prof.K
    tg = [t_gpu_star(prof, k, m_star, n_star) for k in range(K)]
    tc = [t_com_star(prof, k, m_star, n_star, tg[k]) for k in range(K)]
    up = [0.0] * K
    for k in range(1, K):                                                   # Eq. (6)
        up[k] = up[k - 1] + (tt_star(prof, k - 1, n_star) + tg[k - 1]) / m_star
    down = [0.0] * K
    for k in range(K - 2, -1, -1):                                          # Eq. (7)
        down[k] = down[k + 1] + (tt_star(prof, k + 1, n_star) + tg[k + 1]) / m_star
    bub = [up[k] + down[k] for k in range(K)]                               # Eq. (5)
    total = [tg[k] + tc[k] + bub[k] for k in range(K)]                      # Eq. (1)
    mem = [memory_star(prof, k, m_star, n_star) for k in range(K)]
    return {"t_gpu": tg, "t_com": tc, "t_up": up, "t_down": down, "t_bub": bub, "t_total": total, "mem": mem,
            "iter_time": max(total), "peak_mem": max(mem)}


def tune(prof: Profile, m_cands: Sequence[int], n_cands: Sequence[int], mem_limit: float,
         objective: str = "throughput"):
    """Brute force over the candidates (c24/c25).  Returns (m*, n*, iter_time)
    or None if nothing fits the memory limit."""
    best = None
    for n_star in n_cands:
        for m_star in m_cands:
            p = predict(prof, m_star, n_star)
            if p["peak_mem"] > mem_limit:
                continue
            score = n_star / p["iter_time"] if objective == "throughput" else -p["iter_time"]
            key = (score, -p["peak_mem"], -n_star, -m_star)
            if best is None or key > best[0]:
                best = (key, m_star, n_star, p["iter_time"])
    return None if best is None else (best[1], best[2], best[3])
