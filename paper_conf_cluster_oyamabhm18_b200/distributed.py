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


class FusedGradReduce:
    """Cross-rank dW sum fused into BackwardFilter (NEXT-3).

    kind "nvls": one NVLink multicast buffer (mucu_nvls_*), the kernels issue one
    multimem.red per value and NVSwitch adds it into every rank's copy.
    kind "p2p": one buffer per rank (torch symmetric memory for the peer mappings),
    the kernels issue one red.global.add per rank over NVLink P2P.
    `sums` is this rank's buffer with the layout of ConvNet.dw_flat; after an
    iteration run with ``net.nvls = self`` every rank's `sums` holds the sum over
    ranks of dw_flat.  Collective constructor."""

    def __init__(self, numel: int, device: int, kind: str = "nvls", group=None):
        from . import _lib as L
        self.L = L
        self.kind = kind
        self.group = group
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        rank = dist.get_rank(group) if dist.is_initialized() else 0
        self.numel = int(numel)
        flag_at = (self.numel + 63) // 64 * 64  # 256-B aligned flag word after the sums
        self.epoch = 0
        if kind == "nvls":
            nbytes = flag_at * 4
            if rank == 0:
                self.nv = L.Nvls(device, self.world, nbytes)
                fd = self.nv.export() if self.world > 1 else None
            else:
                fd = None
            if self.world > 1:
                fd = share_fd(fd, group)
                if rank != 0:
                    self.nv = L.Nvls(device, self.world, nbytes, fd=fd)
                    os.close(fd)
            local, mc = self.nv.bind()
            self.sums = _tensor_at(local, self.numel, device)
            self.bases = [mc]
        elif kind == "p2p":
            self.nv = None
            if self.world == 1:
                self._buf = torch.zeros(flag_at + 64, dtype=torch.float32, device=torch.device("cuda", device))
                self.bases = [self._buf.data_ptr()]
            else:
                import torch.distributed._symmetric_memory as symm_mem
                self._buf = symm_mem.empty(flag_at + 64, dtype=torch.float32, device=torch.device("cuda", device))
                self._buf.zero_()
                hdl = symm_mem.rendezvous(self._buf, (group or dist.group.WORLD).group_name)
                self.bases = list(hdl.buffer_ptrs)
            self.sums = self._buf[:self.numel]
            self._flags = L.reduce_target([b + 4 * flag_at for b in self.bases])
            self._own = self._buf.data_ptr() + 4 * flag_at
        else:
            raise ValueError(f"unknown fused reduction kind {kind!r}")

    def target(self, offset_bytes: int):
        """Reduction target of the dw view at byte offset `offset_bytes` of dw_flat."""
        return self.L.reduce_target([b + offset_bytes for b in self.bases], multicast=self.kind == "nvls")

    def _barrier(self):
        stream = torch.cuda.current_stream().cuda_stream
        if self.kind == "nvls":
            self.nv.barrier(stream)
        else:
            self.epoch += 1
            self.L.peer_barrier(self._flags, self._own, self.epoch * self.world, stream)

    def begin(self):
        """Stream-ordered: zero this rank's buffer, then wait for every rank's."""
        self.sums.zero_()
        self._barrier()

    def end(self):
        """Stream-ordered: every rank's reductions are complete and visible."""
        self._barrier()

    def close(self):
        if self.nv is not None:
            self.nv.close()


NvlsGradReduce = FusedGradReduce


class _CudaMem:
    def __init__(self, ptr: int, numel: int):
        self.__cuda_array_interface__ = {"shape": (numel,), "typestr": "<f4", "data": (ptr, False), "version": 3,
                                         "strides": None}


def _tensor_at(ptr: int, numel: int, device: int) -> torch.Tensor:
    """fp32 tensor over library-owned device memory (no copy)."""
    return torch.as_tensor(_CudaMem(ptr, numel), device=torch.device("cuda", device))
