"""Data parallelism over torch.distributed (NCCL over NVLink / NVSwitch).

The only cross-GPU step of the method: the mini-batch is sharded
along N (rank r owns samples [r N/p, (r+1) N/p)); Forward and BackwardData are
independent per GPU; each layer's filter gradient dw (a plain sum
over samples) is summed across ranks with an allreduce issued asynchronously
right after that layer's last BackwardFilter micro-batch, so it overlaps the
remaining backward layers.  `GradAllreduce` is backend-agnostic (the CPU tests
run it over gloo; the GPU path over nccl).
"""
from __future__ import annotations

import os
from typing import List, Optional

import torch
import torch.distributed as dist


def init_from_env(backend: Optional[str] = None) -> bool:
    """Initialise the default process group from torchrun's env (127.0.0.1 rendezvous)."""
    if int(os.environ.get("WORLD_SIZE", "1")) <= 1:
        return False
    if not dist.is_initialized():
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        backend = backend or ("nccl" if torch.cuda.is_available() else "gloo")
        if backend == "nccl":
            torch.cuda.set_device(int(os.environ.get("LOCAL_RANK", "0")))
        dist.init_process_group(backend=backend)
    return True


def shard_range(n_global: int, rank: int, world: int):
    """Samples owned by `rank` when the global mini-batch is split along N."""
    base, rem = divmod(n_global, world)
    start = rank * base + min(rank, rem)
    return start, start + base + (1 if rank < rem else 0)


class GradAllreduce:
    """grad_hook for ConvNet.iteration: async sum-allreduce of each dw as soon
    as it is final; `wait()` before the optimizer would consume the grads."""

    def __init__(self, group=None, average: bool = False):
        self.group = group
        self.average = average
        self.works: List = []
        self.tensors: List[torch.Tensor] = []

    def __call__(self, layer: int, dw: torch.Tensor):
        if not dist.is_initialized() or dist.get_world_size(self.group) == 1:
            return
        self.works.append(dist.all_reduce(dw, op=dist.ReduceOp.SUM, group=self.group, async_op=True))
        self.tensors.append(dw)

    def wait(self):
        for w in self.works:
            w.wait()
        if self.average and dist.is_initialized():
            ws = dist.get_world_size(self.group)
            for t in self.tensors:
                t.div_(ws)
        self.works, self.tensors = [], []


def max_over_ranks(value: float, device=None) -> float:
    """Max of a host scalar over all ranks (timings are reported as the max)."""
    if not dist.is_initialized():
        return value
    dev = device if device is not None else (torch.device("cuda", torch.cuda.current_device())
                                             if dist.get_backend() == "nccl" else torch.device("cpu"))
    t = torch.tensor([value], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())
