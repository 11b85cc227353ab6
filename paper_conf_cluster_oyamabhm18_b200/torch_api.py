"""PyTorch-facing wrappers: tensors -> raw device pointers for the C ABI.

PyTorch provides only device memory (tensors, the uint8 workspace, benchmark
scratch) and the stream (``torch.cuda.current_stream()``); every convolution
step runs in libmucudnn's sm_100a kernels.  Activations are contiguous NHWC
tensors [N,H,W,C] / [N,P,Q,K], filters contiguous KRSC [K,R,S,C]; dtype
float32 for MATH_F32 / MATH_TF32, bfloat16 for MATH_BF16; dw is float32.
"""
from __future__ import annotations

from typing import List, Optional, Sequence, Tuple

import torch

from . import _lib as L


def _dtype(math: int):
    return torch.bfloat16 if math == L.MATH_BF16 else torch.float32


def _check_tensor(t: torch.Tensor, shape, dtype, name):
    if not t.is_cuda:
        raise ValueError(f"{name} must be a CUDA tensor (no CPU fallback)")
    if tuple(t.shape) != tuple(shape):
        raise ValueError(f"{name} shape {tuple(t.shape)} != {tuple(shape)}")
    if t.dtype != dtype:
        raise ValueError(f"{name} dtype {t.dtype} != {dtype}")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous (NHWC / KRSC)")


def _stream():
    return torch.cuda.current_stream().cuda_stream


def shapes(d: L.ConvDesc):
    p, q = L.output_dims(d)
    return (d.n, d.h, d.w, d.c), (d.k, d.r, d.s, d.c), (d.n, p, q, d.k)


def plan_workspace(d: L.ConvDesc, conv_type: int, plan: Sequence[Tuple[int, int]]) -> int:
    return max(L.workspace_size(d, conv_type, a, b) for a, b in plan)


def _ws(workspace: Optional[torch.Tensor]):
    if workspace is None:
        return 0, 0
    if not workspace.is_cuda or workspace.dtype != torch.uint8:
        raise ValueError("workspace must be a CUDA uint8 tensor")
    return workspace.data_ptr(), workspace.numel()


def conv_forward(h: L.Handle, d: L.ConvDesc, plan, x, w, y=None, alpha=1.0, beta=0.0, workspace=None):
    xs, ws_, ys = shapes(d)
    dt = _dtype(d.math)
    _check_tensor(x, xs, dt, "x")
    _check_tensor(w, ws_, dt, "w")
    if y is None:
        y = torch.empty(ys, dtype=dt, device=x.device)
    _check_tensor(y, ys, dt, "y")
    wp, wb = _ws(workspace)
    h.conv_forward(d, plan, alpha, x.data_ptr(), w.data_ptr(), beta, y.data_ptr(), wp, wb, _stream())
    return y


def conv_backward_data(h: L.Handle, d: L.ConvDesc, plan, dy, w, dx=None, alpha=1.0, beta=0.0, workspace=None):
    xs, ws_, ys = shapes(d)
    dt = _dtype(d.math)
    _check_tensor(dy, ys, dt, "dy")
    _check_tensor(w, ws_, dt, "w")
    if dx is None:
        dx = torch.empty(xs, dtype=dt, device=dy.device)
    _check_tensor(dx, xs, dt, "dx")
    wp, wb = _ws(workspace)
    h.conv_backward_data(d, plan, alpha, dy.data_ptr(), w.data_ptr(), beta, dx.data_ptr(), wp, wb, _stream())
    return dx


def conv_backward_filter(h: L.Handle, d: L.ConvDesc, plan, x, dy, dw=None, alpha=1.0, beta=0.0, workspace=None):
    xs, ws_, ys = shapes(d)
    dt = _dtype(d.math)
    _check_tensor(x, xs, dt, "x")
    _check_tensor(dy, ys, dt, "dy")
    if dw is None:
        dw = torch.zeros(ws_, dtype=torch.float32, device=x.device)
    _check_tensor(dw, ws_, torch.float32, "dw")
    wp, wb = _ws(workspace)
    h.conv_backward_filter(d, plan, alpha, x.data_ptr(), dy.data_ptr(), beta, dw.data_ptr(), wp, wb, _stream())
    return dw


def conv_backward_filter_reduce(h: L.Handle, d: L.ConvDesc, plan, x, dy, dw, target: "L.ReduceTarget", alpha=1.0,
                                beta=0.0, workspace=None):
    """conv_backward_filter + the fused cross-rank sum (NEXT-3): the final dw values
    are also added to `target` (a multicast address or one buffer per rank, each
    element-aligned with dw)."""
    xs, ws_, ys = shapes(d)
    dt = _dtype(d.math)
    _check_tensor(x, xs, dt, "x")
    _check_tensor(dy, ys, dt, "dy")
    _check_tensor(dw, ws_, torch.float32, "dw")
    wp, wb = _ws(workspace)
    h.conv_backward_filter_reduce(d, plan, alpha, x.data_ptr(), dy.data_ptr(), beta, dw.data_ptr(), target, wp, wb,
                                  _stream())
    return dw


def run(h: L.Handle, d: L.ConvDesc, conv_type: int, plan, a, b, out=None, alpha=1.0, beta=0.0, workspace=None):
    """Dispatch by conv type: FWD (x, w) -> y; DGRAD (dy, w) -> dx; WGRAD (x, dy) -> dw."""
    fn = {L.FWD: conv_forward, L.BWD_DATA: conv_backward_data, L.BWD_FILTER: conv_backward_filter}[conv_type]
    return fn(h, d, plan, a, b, out, alpha=alpha, beta=beta, workspace=workspace)


def make_scratch(d: L.ConvDesc, conv_type: int, ws_limit: int, device="cuda", seed=0) -> torch.Tensor:
    """Benchmark scratch (P:L88 step 1 runs on scratch tensors) filled with N(0,1)
    data of the layer's dtype so the timed kernels see realistic values."""
    nbytes = L.benchmark_scratch_size(d, conv_type, ws_limit)
    buf = torch.empty(nbytes + 256, dtype=torch.uint8, device=device)
    off = (-buf.data_ptr()) % 256
    buf = buf[off:off + nbytes]
    g = torch.Generator(device=device)
    g.manual_seed(seed)
    if d.math == L.MATH_BF16:
        v = buf[: nbytes // 2 * 2].view(torch.bfloat16)
    else:
        v = buf[: nbytes // 4 * 4].view(torch.float32)
    v.normal_(generator=g)
    return buf


def plan_layer(h: L.Handle, d: L.ConvDesc, conv_type: int, ws_limit: int, scratch: Optional[torch.Tensor] = None):
    """WR: benchmark every (algo, b) within ws_limit, then the DP."""
    if scratch is None:
        scratch = make_scratch(d, conv_type, ws_limit)
    return h.plan_layer(d, conv_type, ws_limit, scratch.data_ptr(), scratch.numel(), _stream())


def benchmark(h: L.Handle, d: L.ConvDesc, conv_type: int, ws_limit: int, scratch: Optional[torch.Tensor] = None):
    if scratch is None:
        scratch = make_scratch(d, conv_type, ws_limit)
    return h.benchmark(d, conv_type, ws_limit, scratch.data_ptr(), scratch.numel(), _stream())
