"""Data parallelism over torch.distributed (NCCL over NVLink / NVSwitch).

The only cross-GPU step of the method: the mini-batch is sharded
along N (rank r owns samples [r N/p, (r+1) N/p)); Forward and BackwardData are
independent per GPU; each layer's filter gradient dw (a plain sum
over samples) is summed across ranks with an allreduce issued asynchronously
right after that layer's last BackwardFilter micro-batch, so it overlaps the
remaining backward layers.  `GradAllreduce` is backend-agnostic (the CPU tests
run it over gloo; the GPU path over nccl).

`NvlsGradReduce` (NEXT-3) replaces the NCCL call: the reduction is
fused into BackwardFilter's epilogue, which adds each final dw value to an NVLink
multicast buffer (`multimem.red`, summed by NVSwitch into every rank's copy); the
host side here only sets up the buffer (fd exchange over the process group) and
enqueues the two NVLS barriers of an iteration.
"""
from __future__ import annotations

import ctypes
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


# ------------------------------------------------------------------ NEXT-3 --
_SYS_PIDFD_GETFD = 438  # x86_64 / aarch64 syscall number


def share_fd(fd: Optional[int], group=None) -> int:
    """Rank 0's open file descriptor `fd`, duplicated into every rank (pidfd_getfd
    of rank 0's process; rank 0 gets its own fd back).  Collective over `group`."""
    obj = [(os.getpid(), fd) if dist.get_rank(group) == 0 else None]
    dist.broadcast_object_list(obj, src=dist.get_global_rank(group, 0) if group is not None else 0, group=group)
    pid, rfd = obj[0]
    if dist.get_rank(group) == 0:
        return rfd
    pidfd = os.pidfd_open(pid)
    try:
        libc = ctypes.CDLL(None, use_errno=True)
        out = libc.syscall(_SYS_PIDFD_GETFD, pidfd, rfd, 0)
        if out < 0:
            e = ctypes.get_errno()
            raise OSError(e, f"pidfd_getfd({pid}, {rfd}): {os.strerror(e)}")
        return out
    finally:
        os.close(pidfd)


class NvlsGradReduce:
    """Cross-rank dW sum through NVLink multicast, fused into BackwardFilter.

    `sums` is this rank's copy of the multicast buffer as an fp32 tensor with the
    layout of ConvNet.dw_flat; after an iteration run with ``nvls=self`` every
    rank's `sums` holds the sum over ranks of dw_flat.  Collective constructor."""

    def __init__(self, numel: int, device: int, group=None):
        from . import _lib as L
        self.group = group
        world = dist.get_world_size(group) if dist.is_initialized() else 1
        rank = dist.get_rank(group) if dist.is_initialized() else 0
        nbytes = max(int(numel), 1) * 4
        if rank == 0:
            self.nv = L.Nvls(device, world, nbytes)
            fd = self.nv.export() if world > 1 else None
        else:
            fd = None
        if world > 1:
            fd = share_fd(fd, group)
            if rank != 0:
                self.nv = L.Nvls(device, world, nbytes, fd=fd)
                os.close(fd)
        local, mc = self.nv.bind()
        self.mc_base = mc
        self.numel = int(numel)
        self.sums = _tensor_at(local, self.numel, device)

    def mc_ptr(self, local_view: torch.Tensor, flat: torch.Tensor) -> int:
        """Multicast address of the element of `sums` matching `local_view` of `flat`."""
        return self.mc_base + (local_view.data_ptr() - flat.data_ptr())

    def begin(self):
        """Stream-ordered: zero this rank's copy, then wait for every rank's."""
        self.sums.zero_()
        self.nv.barrier(torch.cuda.current_stream().cuda_stream)

    def end(self):
        """Stream-ordered: every rank's reductions are complete and visible."""
        self.nv.barrier(torch.cuda.current_stream().cuda_stream)


class _CudaMem:
    def __init__(self, ptr: int, numel: int):
        self.__cuda_array_interface__ = {"shape": (numel,), "typestr": "<f4", "data": (ptr, False), "version": 3,
                                         "strides": None}


def _tensor_at(ptr: int, numel: int, device: int) -> torch.Tensor:
    """fp32 tensor over library-owned device memory (no copy)."""
    return torch.as_tensor(_CudaMem(ptr, numel), device=torch.device("cuda", device))
