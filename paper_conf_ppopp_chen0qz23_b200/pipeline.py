"""Live advance-forward pipeline runtime for one stage (row f2).

One process per pipeline stage k (rank k of a K-rank process group).  Every
iteration each of the N parallel pipelines pushes its batch of M
micro-batches through the stages in the order Algorithm 1 prescribes for
this stage (``ea_schedule`` -- `advance` forwards first, then forward/backward
pairs, then the cool-down), exchanging activations forward and
activation-gradients backward with the neighbouring stages (point-to-point).
After the last backward of the iteration the stage's N replicas are coupled
by ONE elastic-averaging step (``ElasticAveraging.step``, co-located layout:
this GPU holds stage k of all N pipelines plus the reference model),
and the run-time controller of Algorithm 1 (lines 9-10, ``ea_advance_*``)
decides whether the next iteration forwards one more micro-batch in advance.

Concurrency ("a parallel pipeline launches a process on each GPU"):
with ``concurrent=True`` the N pipelines of a stage run at the same time, one
host thread and one CUDA stream per pipeline, each pipeline's transfers on its
own process group (``make_pipeline_groups``) -- so NCCL's in-order matching of
point-to-point operations holds per pipeline, and the pipelines' activation
transfers and compute interleave freely.  The elastic-averaging step goes on
its own stream (``ea_stream``): it waits only for every pipeline's last
backward (CUDA events), the host does not wait for it, and the next
iteration's forward of pipeline i waits for it on the GPU (it reads x_i) --
P:112 "in an asynchronous manner ... to prevent the inter-process
communication blocking the pipeline".

Transfers (``transport``): "dist" -- torch.distributed point-to-point, device
tensors over NCCL (NVLink) with the ``nccl`` backend, staged through host
memory with ``gloo``; "ipc" -- the library's own activation channels
(``binding.Channel``, ``ea_chan_*``): copy-engine copies straight into the
receiving stage's device memory over a CUDA IPC peer mapping, handshaken by
stream memory operations, so neither host waits for a transfer (the process
group only carries the one-time handle exchange; two processes may share a
GPU).  The compute of a stage is the caller's ``torch.nn.Module`` (autograd);
the runtime owns the order, the transfers, the activation stash and the
averaging.
"""
from __future__ import annotations

import threading
import time
from typing import Callable, List, Optional, Sequence

from .binding import AdvanceController, Channel, schedule


def wait_streams(streams, timeout_s: float, what: str = "streams"):
    """Host wait for CUDA streams with a deadline (failure detection for the activation channels: a stream that
    waits on the GPU for a message the peer stage never sends -- it died or stalled -- would make synchronize()
    block forever).  Raises TimeoutError naming `what`; the streams stay blocked."""
    import torch
    evs = []
    for s in streams:
        e = torch.cuda.Event()
        e.record(s)
        evs.append(e)
    t0 = time.monotonic()
    while not all(e.query() for e in evs):
        if time.monotonic() - t0 > timeout_s:
            raise TimeoutError(f"{what}: GPU work not finished after {timeout_s:.0f} s (a peer stage stalled?)")
        time.sleep(0.0002)


def make_pipeline_groups(n_pipelines: int, ranks: Optional[Sequence[int]] = None, backend: Optional[str] = None):
    """One process group per parallel pipeline over the K stage ranks (a collective call: every stage rank
    creates the N groups in the same order).  Pipeline i's activations and gradients travel only on group i."""
    import torch.distributed as dist
    ranks = list(range(dist.get_world_size())) if ranks is None else list(ranks)
    return [dist.new_group(ranks, backend=backend) for _ in range(n_pipelines)]


class PipelineStage:
    """Stage `stage` (0-based) of K; `replicas` = this stage's module of each of
    the N pipelines (structurally identical).  `ea` (optional) is an
    ElasticAveraging handle whose stage `ea_stage` holds these parameters,
    flattened in `flat_params[i]` / `flat_grads[i]` (views the modules use).
    `concurrent`: run the N pipelines at once (threads + streams; `groups` =
    per-pipeline process groups, default `make_pipeline_groups(N)`)."""

    def __init__(self, replicas: Sequence, stage: int, K: int, M: int, group=None, *, ea=None, ea_stage: int = 0,
                 center=None, flat_params=None, flat_grads=None, mem_limit: Optional[float] = None,
                 mem_per_microbatch: float = 0.0, extra_advance: int = 0, dynamic: bool = False,
                 concurrent: bool = False, groups=None, transport: str = "dist", act_bytes: int = 0,
                 device=None, timeout_s: float = 600.0):
        import torch.distributed as dist
        self.replicas = list(replicas)
        self.N = len(self.replicas)
        self.stage, self.K, self.M = stage, K, M
        self.group = group
        self.rank = dist.get_rank(group)
        self.prev = stage - 1 if stage > 0 else None      # neighbour stage indices = ranks of `group`
        self.next = stage + 1 if stage < K - 1 else None
        self.ea, self.ea_stage, self.center = ea, ea_stage, center
        self.flat_params, self.flat_grads = flat_params, flat_grads
        self.ctl = AdvanceController(K, M)
        self.ctl.ctl.advance_num = min(self.ctl.ctl.advance_num + max(extra_advance, 0), M)  # beyond 1F1B (c15)
        self.backend = dist.get_backend(group)
        self.dynamic = dynamic
        self.mem_limit = mem_limit
        self.mem_per_microbatch = mem_per_microbatch
        self.concurrent = concurrent
        if concurrent and groups is None:
            groups = make_pipeline_groups(self.N)
        self.groups = list(groups) if groups is not None else [group] * self.N
        self.peak_stash = 0
        self.history: List[dict] = []
        self._streams = None      # per-pipeline CUDA streams (concurrent, on a GPU)
        self._ea_stream = None
        self._ea_done = None      # event: the last EA step (the next forward of every pipeline waits for it)
        if transport not in ("dist", "ipc"):
            raise ValueError("transport must be 'dist' or 'ipc'")
        self.transport = transport
        self.timeout_s = float(timeout_s)    # ipc: deadline for an iteration's streams (a stalled peer stage)
        self._chan = {}
        if transport == "ipc":
            self._open_channels(act_bytes, device)

    # ------------------------------------------------------------------ activation channels (transport "ipc")
    def _open_channels(self, act_bytes: int, device):
        """Per pipeline i: a forward channel to the next stage and a backward channel from it (and the mirror
        ends toward the previous stage), M slots of act_bytes each -- a sender never waits for a free slot, as at
        most M messages of one direction are in flight per iteration.  The IPC handles travel once over the
        stage process group (all_gather_object); every end then maps its peer's buffer."""
        import os
        import torch
        import torch.distributed as dist
        if act_bytes <= 0:
            raise ValueError("transport 'ipc' needs act_bytes (bytes of the largest activation message)")
        if os.environ.get("CUDA_MODULE_LOADING", "LAZY").upper() != "EAGER":
            # a stream of this process may wait on the GPU for a message the peer sends only after this process
            # enqueued more work; with lazy loading, the first launch of a kernel synchronises the context and
            # would wait for that stream -> deadlock across the two processes
            raise RuntimeError("transport 'ipc' needs CUDA_MODULE_LOADING=EAGER in the environment before CUDA "
                               "is initialised (lazy kernel loading synchronises the context, which cannot finish "
                               "while a stream waits on the GPU for the peer stage's message)")
        dev = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        mine = {}
        for i in range(self.N):
            if self.next is not None:
                self._chan[("F", i, "send")] = Channel("send", act_bytes, self.M, dev.index)
                self._chan[("B", i, "recv")] = Channel("recv", act_bytes, self.M, dev.index)
                mine[("F", i, self.stage, "send")] = self._chan[("F", i, "send")].export()
                mine[("B", i, self.stage + 1, "recv")] = self._chan[("B", i, "recv")].export()
            if self.prev is not None:
                self._chan[("F", i, "recv")] = Channel("recv", act_bytes, self.M, dev.index)
                self._chan[("B", i, "send")] = Channel("send", act_bytes, self.M, dev.index)
                mine[("F", i, self.stage - 1, "recv")] = self._chan[("F", i, "recv")].export()
                mine[("B", i, self.stage, "send")] = self._chan[("B", i, "send")].export()
        allh = [None] * dist.get_world_size(self.group)
        dist.all_gather_object(allh, mine, group=self.group)
        for i in range(self.N):
            if self.next is not None:      # F: stage -> stage+1 (key: source stage); B: stage+1 -> stage
                self._chan[("F", i, "send")].connect(allh[self.stage + 1][("F", i, self.stage, "recv")])
                self._chan[("B", i, "recv")].connect(allh[self.stage + 1][("B", i, self.stage + 1, "send")])
            if self.prev is not None:
                self._chan[("F", i, "recv")].connect(allh[self.stage - 1][("F", i, self.stage - 1, "send")])
                self._chan[("B", i, "send")].connect(allh[self.stage - 1][("B", i, self.stage, "recv")])

    def close(self):
        """Free the activation channels (every stage past its last iteration first: a collective barrier)."""
        import torch.distributed as dist
        if self._chan:
            dist.barrier(group=self.group)
            for c in self._chan.values():
                c.close()
            self._chan = {}

    # ------------------------------------------------------------------ transfers
    def _peer(self, stage_index, group):
        import torch.distributed as dist
        return dist.get_global_rank(group, stage_index) if group is not None else stage_index

    def _tag(self, pipeline: int, j: int, backward: bool) -> int:
        return ((pipeline * self.M + j) << 1) | int(backward)

    def _send(self, t, dst_stage, tag, group, pipeline=0, backward=False):
        import torch.distributed as dist
        t = t.detach().contiguous()
        if self.transport == "ipc":     # stream-ordered; t was produced on this stream, so its reuse is ordered
            self._chan[("B" if backward else "F", pipeline, "send")].send(t)
            return None
        if self.backend == "gloo" and t.is_cuda:      # gloo moves host tensors
            t = t.cpu()
        return dist.isend(t, dst=self._peer(dst_stage, group), group=group, tag=tag)

    def _recv(self, like_shape, dtype, device, src_stage, tag, group, pipeline=0, backward=False):
        import torch
        import torch.distributed as dist
        if self.transport == "ipc":     # the GPU waits for the message, not the host
            buf = torch.empty(like_shape, dtype=dtype, device=device)
            self._chan[("B" if backward else "F", pipeline, "recv")].recv(buf)
            return buf
        host = self.backend == "gloo"
        buf = torch.empty(like_shape, dtype=dtype, device="cpu" if host else device)
        dist.recv(buf, src=self._peer(src_stage, group), group=group, tag=tag)
        return buf.to(device) if host else buf

    # ------------------------------------------------------------------ one pipeline's share of an iteration
    def _run_pipeline(self, i, ops, inputs, targets, loss_fn, act_shape, act_dtype, device):
        """Pipeline i's ops on this stage, in Algorithm 1's order.  Returns (loss, pending sends, peak stash)."""
        mod = self.replicas[i]
        group = self.groups[i]
        stash, pending, loss_sum, peak = {}, [], 0.0, 0
        for kind, j in ops:
            if kind == "F":
                if self.prev is None:
                    x = inputs[i][j]
                else:
                    x = self._recv(act_shape, act_dtype, device, self.prev, self._tag(i, j, False), group, i)
                    x.requires_grad_(True)
                y = mod(x)
                if self.next is None:
                    loss = loss_fn(y, targets[i][j]) / self.M
                    loss_sum += float(loss.detach())
                    stash[j] = (x, loss)
                else:
                    pending.append(self._send(y, self.next, self._tag(i, j, False), group, i))
                    stash[j] = (x, y)
                peak = max(peak, len(stash))
            else:
                x, y = stash.pop(j)
                if self.next is None:
                    y.backward()
                else:
                    gy = self._recv(y.shape, y.dtype, device, self.next, self._tag(i, j, True), group, i, True)
                    y.backward(gy)
                if self.prev is not None:
                    pending.append(self._send(x.grad, self.prev, self._tag(i, j, True), group, i, True))
        return loss_sum, pending, peak

    def _cuda(self, device):
        import torch
        return torch.cuda.is_available() and str(device).startswith("cuda")

    # ------------------------------------------------------------------ one iteration
    def run_iteration(self, inputs=None, targets=None, loss_fn: Optional[Callable] = None, act_shape=None,
                      act_dtype=None, device="cpu", zero_grads: bool = False, sync: bool = True):
        """inputs[i][j] (stage 0) / targets[i][j] (last stage): micro-batch j of
        pipeline i.  act_shape: shape of the activation this stage receives
        (stage > 0) -- and, for the backward, the shape it sends.  zero_grads:
        zero flat_grads[i] on pipeline i's stream first (ordered after the last
        EA step, which reads them).  sync=False returns once the pipelines'
        streams are done and leaves the EA step running on its stream (the next
        iteration's forwards wait for it on the GPU).  Returns the per-pipeline
        summed loss on the last stage (else None)."""
        import torch
        advance = self.ctl.advance_for_stage(self.stage)
        ops = schedule(self.K, self.M, self.stage, advance)
        t0 = time.perf_counter()
        cuda = self._cuda(device)
        results = [None] * self.N
        if self.concurrent:
            if cuda and self._streams is None:
                self._streams = [torch.cuda.Stream(device=device) for _ in range(self.N)]
            errors = []

            def work(i):
                try:
                    if cuda:
                        s = self._streams[i]
                        if self._ea_done is not None:
                            s.wait_event(self._ea_done)        # x_i was updated by the last EA step
                        with torch.cuda.stream(s):
                            if zero_grads and self.flat_grads is not None:
                                self.flat_grads[i].zero_()
                            results[i] = self._run_pipeline(i, ops, inputs, targets, loss_fn, act_shape,
                                                            act_dtype, device)
                    else:
                        results[i] = self._run_pipeline(i, ops, inputs, targets, loss_fn, act_shape, act_dtype,
                                                        device)
                except BaseException as e:  # pragma: no cover
                    errors.append(e)

            threads = [threading.Thread(target=work, args=(i,)) for i in range(self.N)]
            for t in threads:
                t.start()
            for t in threads:
                t.join()
            if errors:
                raise errors[0]
        else:
            for i in range(self.N):
                if cuda and self._ea_done is not None:
                    torch.cuda.current_stream(device).wait_event(self._ea_done)
                if zero_grads and self.flat_grads is not None:
                    self.flat_grads[i].zero_()
                results[i] = self._run_pipeline(i, ops, inputs, targets, loss_fn, act_shape, act_dtype, device)
        pending = [w for r in results for w in r[1] if w is not None]
        peak = max(r[2] for r in results)
        if self.ea is not None:
            # every pipeline's last backward of this stage is done: the averaging step goes onto its own stream
            # behind them (events), and the host moves on -- it overlaps the activation-gradient sends still in
            # flight (they never read the parameters) and whatever else is queued ("not block")
            if cuda:
                if self._ea_stream is None:
                    self._ea_stream = torch.cuda.Stream(device=device)
                    self._ea_done = torch.cuda.Event()
                streams = self._streams if self.concurrent else [torch.cuda.current_stream(device)]
                for s in streams:
                    self._ea_stream.wait_stream(s)
                self.ea.step(self.ea_stage, self.flat_params, self.flat_grads, self.center, stream=self._ea_stream)
                self._ea_done.record(self._ea_stream)
            else:
                self.ea.step(self.ea_stage, self.flat_params, self.flat_grads, self.center)
        for w in pending:
            w.wait()
        streams = (self._streams if self.concurrent else [torch.cuda.current_stream(device)]) if cuda else []
        if cuda and self.transport == "ipc":
            # a stream waiting on the GPU for a message the peer never sends would block synchronize() forever:
            # wait with a deadline instead (the EA stream too when sync)
            wait_streams(streams + ([self._ea_stream] if sync and self._ea_stream is not None else []),
                         self.timeout_s, f"stage {self.stage}")
        elif cuda and sync:
            torch.cuda.synchronize(device)
        elif cuda:
            for s in streams:
                s.synchronize()
        dt = time.perf_counter() - t0
        self.peak_stash = peak
        rec = {"advance": advance, "peak_stash": peak, "time": dt}
        if self.dynamic and self.mem_limit is not None and self.stage == 0:
            self.ctl.update(dt, peak * self.mem_per_microbatch, self.mem_per_microbatch, self.mem_limit)
        if self.dynamic and self.mem_limit is not None:
            self._agree_on_advance()
            rec["next_advance"] = self.ctl.advance_num
        self.history.append(rec)
        return [r[0] for r in results] if self.next is None else None

    def _agree_on_advance(self):
        """Algorithm 1 runs its adjustment on the first GPU; the other
        stages follow it (a_k = min(M, K-k+e), c15), which keeps the per-stage
        advances feasible (c16).  Broadcast GPU 1's decision."""
        import torch
        import torch.distributed as dist
        t = torch.tensor([self.ctl.advance_num], dtype=torch.int64)
        if self.backend == "nccl":
            t = t.cuda()
        src = dist.get_global_rank(self.group, 0) if self.group is not None else 0
        dist.broadcast(t, src=src, group=self.group)
        self.ctl.ctl.advance_num = int(t.item())
