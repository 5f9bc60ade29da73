"""Live advance-forward pipeline runtime for one stage (row f2).

One process per pipeline stage k (rank k of a K-rank process group).  Every
iteration each of the N parallel pipelines pushes its batch of M
micro-batches through the stages in the order Algorithm 1 prescribes for
this stage (``ea_schedule`` -- `advance` forwards first, then forward/backward
pairs, then the cool-down), exchanging activations forward and
activation-gradients backward with the neighbouring stages (point-to-point,
tagged by pipeline and micro-batch).  After the last backward of the
iteration the stage's N replicas are coupled by ONE elastic-averaging step
(``ElasticAveraging.step``, co-located layout: this GPU holds stage k of all
N pipelines plus the reference model), and the run-time controller of
Algorithm 1 (lines 9-10, ``ea_advance_*``) decides whether the next
iteration forwards one more micro-batch in advance.

The compute of a stage is the caller's ``torch.nn.Module`` (autograd); the
runtime owns the order, the transfers, the activation stash and the
averaging.  Pipelines run one after another within an iteration (the simple
policy; the paper overlaps them with one process per pipeline per GPU).
"""
from __future__ import annotations

import time
from typing import Callable, List, Optional, Sequence

from .binding import AdvanceController, schedule


class PipelineStage:
    """Stage `stage` (0-based) of K; `replicas` = this stage's module of each of
    the N pipelines (structurally identical).  `ea` (optional) is an
    ElasticAveraging handle whose stage `ea_stage` holds these parameters,
    flattened in `flat_params[i]` / `flat_grads[i]` (views the modules use)."""

    def __init__(self, replicas: Sequence, stage: int, K: int, M: int, group=None, *, ea=None, ea_stage: int = 0,
                 center=None, flat_params=None, flat_grads=None, mem_limit: Optional[float] = None,
                 mem_per_microbatch: float = 0.0, extra_advance: int = 0, dynamic: bool = False):
        import torch.distributed as dist
        self.replicas = list(replicas)
        self.N = len(self.replicas)
        self.stage, self.K, self.M = stage, K, M
        self.group = group
        self.rank = dist.get_rank(group)
        self.prev = self.rank - 1 if stage > 0 else None
        self.next = self.rank + 1 if stage < K - 1 else None
        self.ea, self.ea_stage, self.center = ea, ea_stage, center
        self.flat_params, self.flat_grads = flat_params, flat_grads
        self.ctl = AdvanceController(K, M)
        self.ctl.ctl.advance_num = min(self.ctl.ctl.advance_num + max(extra_advance, 0), M)  # beyond 1F1B (c15)
        self.backend = dist.get_backend(group)
        self.dynamic = dynamic
        self.mem_limit = mem_limit
        self.mem_per_microbatch = mem_per_microbatch
        self.peak_stash = 0
        self.history: List[dict] = []

    # ------------------------------------------------------------------ transfers
    def _tag(self, pipeline: int, j: int, backward: bool) -> int:
        return ((pipeline * self.M + j) << 1) | int(backward)

    def _send(self, t, dst, tag):
        import torch.distributed as dist
        t = t.detach().contiguous()
        if self.backend == "gloo" and t.is_cuda:      # gloo moves host tensors
            t = t.cpu()
        return dist.isend(t, dst=dst, group=self.group, tag=tag)

    def _recv(self, like_shape, dtype, device, src, tag):
        import torch
        import torch.distributed as dist
        host = self.backend == "gloo"
        buf = torch.empty(like_shape, dtype=dtype, device="cpu" if host else device)
        dist.recv(buf, src=src, group=self.group, tag=tag)
        return buf.to(device) if host else buf

    # ------------------------------------------------------------------ one iteration
    def run_iteration(self, inputs=None, targets=None, loss_fn: Optional[Callable] = None, act_shape=None,
                      act_dtype=None, device="cpu"):
        """inputs[i][j] (stage 0) / targets[i][j] (last stage): micro-batch j of
        pipeline i.  act_shape: shape of the activation this stage receives
        (stage > 0) -- and, for the backward, the shape it sends.  Returns the
        per-pipeline summed loss on the last stage (else None)."""
        import torch
        advance = self.ctl.advance_for_stage(self.stage)
        ops = schedule(self.K, self.M, self.stage, advance)
        t0 = time.perf_counter()
        losses = [0.0] * self.N
        pending = []
        peak = 0
        for i, mod in enumerate(self.replicas):
            stash = {}
            for kind, j in ops:
                if kind == "F":
                    if self.prev is None:
                        x = inputs[i][j]
                    else:
                        x = self._recv(act_shape, act_dtype, device, self.prev, self._tag(i, j, False))
                        x.requires_grad_(True)
                    y = mod(x)
                    if self.next is None:
                        loss = loss_fn(y, targets[i][j]) / self.M
                        losses[i] += float(loss.detach())
                        stash[j] = (x, loss)
                    else:
                        pending.append(self._send(y, self.next, self._tag(i, j, False)))
                        stash[j] = (x, y)
                    peak = max(peak, len(stash))
                else:
                    x, y = stash.pop(j)
                    if self.next is None:
                        y.backward()
                    else:
                        gy = self._recv(y.shape, y.dtype, device, self.next, self._tag(i, j, True))
                        y.backward(gy)
                    if self.prev is not None:
                        pending.append(self._send(x.grad, self.prev, self._tag(i, j, True)))
        if self.ea is not None:
            # this stage's last backward is done: the averaging step goes onto the stream now, so it overlaps
            # the activation-gradient sends still in flight (they never read the parameters; "not block")
            self.ea.step(self.ea_stage, self.flat_params, self.flat_grads, self.center)
        for w in pending:
            w.wait()
        if torch.cuda.is_available() and str(device).startswith("cuda"):
            torch.cuda.synchronize()
        dt = time.perf_counter() - t0
        self.peak_stash = peak
        rec = {"advance": advance, "peak_stash": peak, "time": dt}
        if self.dynamic and self.mem_limit is not None and self.stage == 0:
            self.ctl.update(dt, peak * self.mem_per_microbatch, self.mem_per_microbatch, self.mem_limit)
        if self.dynamic and self.mem_limit is not None:
            self._agree_on_advance()
            rec["next_advance"] = self.ctl.advance_num
        self.history.append(rec)
        return losses if self.next is None else None

    def _agree_on_advance(self):
        """Algorithm 1 runs its adjustment on the first GPU; the other
        stages follow it (a_k = min(M, K-k+e), c15), which keeps the per-stage
        advances feasible (c16).  Broadcast GPU 1's decision."""
        import torch
        import torch.distributed as dist
        t = torch.tensor([self.ctl.advance_num], dtype=torch.int64)
        src = dist.get_global_rank(self.group, 0) if self.group is not None else 0
        dist.broadcast(t, src=src, group=self.group)
        self.ctl.ctl.advance_num = int(t.item())
