"""Probe: can two NCCL ranks share one GPU on this box (torchrun --nproc-per-node 2, both on cuda:0)?"""
import os

import torch
import torch.distributed as dist

rank = int(os.environ["RANK"])
dev = torch.device("cuda", 0)
torch.cuda.set_device(dev)
dist.init_process_group("nccl", device_id=dev)
t = torch.full((4,), float(rank + 1), device=dev)
try:
    dist.all_reduce(t)
    torch.cuda.synchronize()
    print(f"rank {rank}: all_reduce ok {t.tolist()}", flush=True)
except Exception as e:  # noqa: BLE001
    print(f"rank {rank}: all_reduce failed: {e}", flush=True)
dist.destroy_process_group()
