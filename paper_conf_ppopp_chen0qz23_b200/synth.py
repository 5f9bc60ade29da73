"""Seeded synthetic inputs shared by the tests, bench.py and smoke().

Holds NONE of the method's arithmetic: only random draws, the stage split and
the coefficient table of the three modes.  It is
the one module both the oracle-side tests and the CUDA-side calls use.

Recipe:
  weights   x0 ~ N(0, 0.02^2) fp32 (GPT-2 init scale); replica i = x0 + N(0, 1e-3^2);
            center = x0; momentum = 0.
  gradients g ~ N(0, 1e-2^2) fp32, fresh every step.
  host      numpy PCG64, seeds 1234 (weights) / 1235 (gradients).
  device    torch.Generator('cuda') (perf runs; values do not affect timing).
  stages    P_s = floor(P / K), remainder on the last stage.
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import Dict, List, Tuple

import numpy as np

WEIGHT_SEED = 1234
GRAD_SEED = 1235
INIT_STD = 0.02
REPLICA_STD = 1e-3
GRAD_STD = 1e-2
LR = 0.05
MOMENTUM = 0.9


def mode_coeffs(mode: str, n: int, alpha: float | None = None) -> Tuple[float, float, float]:
    """(alpha, beta, rho) of a named mode (reading c5).

    paper    rho=1, beta=0          (P:116 steps 4-5 on the local updates)
    easgd    rho=0, beta=N*alpha    (EASGD / Crossbow center pull, refs [35]/[18])
    combined rho=1, beta=N*alpha
    alpha defaults to 1/N."""
    a = 1.0 / n if alpha is None else float(alpha)
    if mode == "paper":
        return a, 0.0, 1.0
    if mode == "easgd":
        return a, n * a, 0.0
    if mode == "combined":
        return a, n * a, 1.0
    raise ValueError(f"unknown mode {mode!r}")


MODES = ("paper", "easgd", "combined")


def stage_split(total_params: int, n_stages: int) -> List[int]:
    """P_s = floor(P/K); the remainder goes to the last stage."""
    base = total_params // n_stages
    sizes = [base] * n_stages
    sizes[-1] += total_params - base * n_stages
    return sizes


@dataclass(frozen=True)
class Config:
    name: str
    n_pipelines: int     # N
    n_stages: int        # K
    total_params: int    # P
    gpus: int
    layout: str          # "colocated" | "spread"

    @property
    def stage_sizes(self) -> List[int]:
        return stage_split(self.total_params, self.n_stages)


# BASELINE.json configs.
CONFIGS: Dict[str, Config] = {
    "C1": Config("C1-2pipe-2stage-2M", 2, 2, 2_000_000, 1, "colocated"),
    "C2": Config("C2-resnet50-25M-N4-K4", 4, 4, 25_000_000, 1, "colocated"),
    "C3N2": Config("C3-bert-large-340M-N2-K4", 2, 4, 340_000_000, 2, "spread"),
    "C3N4": Config("C3-bert-large-340M-N4-K4", 4, 4, 340_000_000, 4, "spread"),
    "C4": Config("C4-gpt2-medium-355M-N8-K8", 8, 8, 355_000_000, 8, "spread"),
    "C5": Config("C5-gpt2-xl-1.5B-N8-K8", 8, 8, 1_500_000_000, 8, "spread"),
}


def host_state(n: int, p: int, seed: int = WEIGHT_SEED):
    """fp32 numpy (replicas[n], center) for one stage of p elements."""
    rng = np.random.Generator(np.random.PCG64(seed))
    x0 = rng.standard_normal(p, dtype=np.float32) * np.float32(INIT_STD)
    reps = [x0 + rng.standard_normal(p, dtype=np.float32) * np.float32(REPLICA_STD) for _ in range(n)]
    return reps, x0.copy()


class GradStream:
    """Fresh fp32 gradients every step from one PCG64 stream (seed GRAD_SEED)."""

    def __init__(self, n: int, p: int, seed: int = GRAD_SEED):
        self.n, self.p = n, p
        self.rng = np.random.Generator(np.random.PCG64(seed))

    def next(self) -> List[np.ndarray]:
        return [self.rng.standard_normal(self.p, dtype=np.float32) * np.float32(GRAD_STD)
                for _ in range(self.n)]


def device_state(n: int, p: int, device, seed: int = 0):
    """Same recipe drawn on the GPU with torch.Generator (perf runs)."""
    import torch
    gen = torch.Generator(device=device)
    gen.manual_seed(seed)
    x0 = torch.randn(p, generator=gen, device=device, dtype=torch.float32) * INIT_STD
    reps = [x0 + torch.randn(p, generator=gen, device=device, dtype=torch.float32) * REPLICA_STD
            for _ in range(n)]
    grads = [torch.randn(p, generator=gen, device=device, dtype=torch.float32) * GRAD_STD
             for _ in range(n)]
    return reps, x0.clone(), grads
