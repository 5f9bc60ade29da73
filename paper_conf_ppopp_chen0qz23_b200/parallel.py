"""Host-side logic of the spread (multi-GPU) layout: placement, center
sharding, NCCL-id bootstrap, and a torch.distributed driver for the
external-collective mode of ``EA_SPREAD``.

Placement: with G = N ranks and K stages, replica i of stage s
lives on rank (i + s) mod N, so every rank holds exactly one replica of every
stage and the N replicas of a stage sit on N distinct GPUs -- the paper's N
pipelines each spanning the GPUs, with the co-partitioned reference
model sharded 1/N over the same GPUs.

Center sharding: stage s's center is padded to P_pad = round_up(P_s, 32 N)
floats (zero padding is a fixed point of the update) and rank r owns
[r P_pad/N, (r+1) P_pad/N).  One exchange step per stage and iteration:
reduce-scatter(sum) of the contributions into the owner shard, shard update,
all-gather.  All ranks issue the per-stage collectives in one global order,
stage K-1 first (the order backward finishes them).
"""
from __future__ import annotations

from typing import Callable, List, Optional, Tuple

SHARD_ALIGN = 32  # floats; must match the library (ea_center_capacity)


def replica_of(rank: int, stage: int, n: int) -> int:
    """Which replica of `stage` rank `rank` hosts."""
    return (rank - stage) % n


def rank_of(replica: int, stage: int, n: int) -> int:
    """Which rank hosts replica `replica` of `stage`."""
    return (replica + stage) % n


def padded_size(p: int, n: int) -> int:
    q = SHARD_ALIGN * n
    return (p + q - 1) // q * q


def shard_bounds(p_pad: int, n: int, rank: int) -> Tuple[int, int]:
    if p_pad % n:
        raise ValueError("P_pad must be a multiple of N")
    s = p_pad // n
    return rank * s, (rank + 1) * s


def stage_order(n_stages: int) -> List[int]:
    """Global order in which every rank issues the per-stage exchanges."""
    return list(range(n_stages - 1, -1, -1))


def broadcast_unique_id(group=None, make_id: Optional[Callable[[], bytes]] = None) -> bytes:
    """Rank 0 creates a 128-byte NCCL unique id; every rank receives it over
    the torch process group (the library's communicator is its own)."""
    import torch
    import torch.distributed as dist
    if make_id is None:
        from .binding import get_unique_id as make_id
    rank = dist.get_rank(group)
    backend = dist.get_backend(group)
    dev = torch.device("cuda", torch.cuda.current_device()) if backend == "nccl" else torch.device("cpu")
    buf = torch.zeros(128, dtype=torch.uint8, device=dev)
    if rank == 0:
        uid = make_id()
        buf.copy_(torch.frombuffer(bytearray(uid), dtype=torch.uint8))
    src = dist.get_global_rank(group, 0) if group is not None else 0
    dist.broadcast(buf, src=src, group=group)
    return bytes(buf.cpu().tolist())


class CollectiveSpread:
    """Drive ``EA_SPREAD`` in external-collective mode with torch.distributed.

    local_fn(stage, replica, grad, center, contrib) and
    apply_fn(stage, center_shard, reduced) default to the library's
    ``ea_spread_local`` / ``ea_spread_apply`` of `handle`; the collectives
    are torch.distributed's (reduce_scatter on NCCL; on gloo, which has no
    reduce-scatter, an all-reduce followed by taking the own shard)."""

    def __init__(self, handle=None, group=None, local_fn=None, apply_fn=None):
        import torch.distributed as dist
        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        self.handle = handle
        self.local_fn = local_fn or handle.spread_local
        self.apply_fn = apply_fn or handle.spread_apply
        self._scratch = {}

    def _buf(self, key, n, like):
        import torch
        b = self._scratch.get(key)
        if b is None or b.numel() != n or b.device != like.device:
            b = torch.empty(n, dtype=like.dtype, device=like.device)
            self._scratch[key] = b
        return b

    def step(self, stage: int, replica, grad, center):
        import torch.distributed as dist
        # the library writes P_pad = ea_center_capacity floats of contribution: size everything from it
        p_pad = self.handle.center_capacity(stage) if self.handle is not None else center.numel()
        if center.numel() != p_pad:
            raise ValueError(f"stage {stage}: center has {center.numel()} elements, the library expects {p_pad}")
        lo, hi = shard_bounds(p_pad, self.world, self.rank)
        contrib = self._buf(("c", stage), p_pad, center)
        self.local_fn(stage, replica, grad, center, contrib)
        if dist.get_backend(self.group) == "nccl":
            reduced = self._buf(("r", stage), hi - lo, center)
            dist.reduce_scatter_tensor(reduced, contrib, group=self.group)
        else:
            dist.all_reduce(contrib, group=self.group)
            reduced = contrib[lo:hi]
        own = center[lo:hi]
        self.apply_fn(stage, own, reduced)
        parts = list(center.view(self.world, hi - lo).unbind(0))
        dist.all_gather(parts, own.clone(), group=self.group)


def connect_p2p(handle, group=None):
    """Wire an EA_XCHG_P2P handle to its peers over a torch process group
    (any backend): all-gather the 64-byte CUDA IPC handles and open them.
    Needed only when the handle was created without an NCCL id."""
    import torch
    import torch.distributed as dist
    mine = handle.p2p_export()
    world = dist.get_world_size(group)
    backend = dist.get_backend(group)
    dev = torch.device("cuda", torch.cuda.current_device()) if backend == "nccl" else torch.device("cpu")
    t = torch.frombuffer(bytearray(mine), dtype=torch.uint8).to(dev)
    out = [torch.empty_like(t) for _ in range(world)]
    dist.all_gather(out, t, group=group)
    handle.p2p_open([bytes(o.cpu().tolist()) for o in out])
