"""Helpers shared by the GPU parity tests (test-side only)."""
import numpy as np
import torch

import oracle
import paper_conf_cluster_oyamabhm18_b200 as mu
from paper_conf_cluster_oyamabhm18_b200 import torch_api as T

_HANDLE = None


def handle():
    global _HANDLE
    if _HANDLE is None:
        _HANDLE = mu.Handle(0)
    return _HANDLE


def dev_dtype(math):
    return torch.bfloat16 if math == mu.MATH_BF16 else torch.float32


def to_dev(a, math):
    return torch.from_numpy(np.ascontiguousarray(a)).to("cuda").to(dev_dtype(math)).contiguous()


def stored(a, math):
    """The exact values the device holds (bf16 rounding RNE), as float32 numpy."""
    return torch.from_numpy(np.ascontiguousarray(a)).to(dev_dtype(math)).float().numpy()


def oracle_ref(shape, conv_type, x, w, dy, alpha=1.0, beta=0.0, out0=None):
    n, c, h, wd, k, r, s, pad, st = shape
    if conv_type == mu.FWD:
        return oracle.conv_forward(x, w, pad, st, alpha, beta, out0)
    if conv_type == mu.BWD_DATA:
        return oracle.conv_backward_data(dy, w, h, wd, pad, st, alpha, beta, out0)
    return oracle.conv_backward_filter(x, dy, r, s, pad, st, alpha, beta, out0)


def run_gpu(d, conv_type, plan, x, w, dy, alpha=1.0, beta=0.0, out0=None, ws_extra=0, canary=False):
    """Execute `plan` through the C ABI; returns (out float64 numpy, workspace-canary-intact)."""
    h = handle()
    math = d.math
    ws_bytes = max(T.plan_workspace(d, conv_type, plan), 0)
    pad_bytes = 4096 if canary else 0
    buf = torch.full((ws_bytes + ws_extra + 2 * pad_bytes + 256,), 0xA5, dtype=torch.uint8, device="cuda")
    off = (-buf.data_ptr()) % 256
    ws = buf[off + pad_bytes: off + pad_bytes + ws_bytes + ws_extra] if (ws_bytes + ws_extra) else None
    if conv_type == mu.FWD:
        a, b = to_dev(x, math), to_dev(w, math)
    elif conv_type == mu.BWD_DATA:
        a, b = to_dev(dy, math), to_dev(w, math)
    else:
        a, b = to_dev(x, math), to_dev(dy, math)
    out = None
    if out0 is not None:
        out = torch.from_numpy(np.ascontiguousarray(out0)).to("cuda")
        out = out.float() if conv_type == mu.BWD_FILTER else out.to(dev_dtype(math))
        out = out.contiguous()
    res = T.run(h, d, conv_type, plan, a, b, out, alpha=alpha, beta=beta, workspace=ws)
    torch.cuda.synchronize()
    intact = True
    if canary:
        lo = buf[off: off + pad_bytes]
        hi = buf[off + pad_bytes + ws_bytes + ws_extra: off + 2 * pad_bytes + ws_bytes + ws_extra]
        intact = bool((lo == 0xA5).all().item() and (hi == 0xA5).all().item())
    return res.double().cpu().numpy(), intact


def normwise_err(got, ref):
    scale = max(float(np.max(np.abs(ref))), 1e-30)
    return float(np.max(np.abs(got - ref))) / scale
