"""synthetic -- seeded input generators shared by tests, bench.py and smoke().

Holds NONE of the method's arithmetic: only random tensors of the shapes,
layouts and value distributions of the paper's workloads, random timing tables
for the planner, and the network layer tables (workload definitions).  Both the
oracle side and the CUDA side receive their inputs from here; neither imports
the other.

Recipe:
* timing tensors: x, dy ~ N(0, 1); w ~ N(0, 1/(C*R*S)),
* exactness tensors: integers uniform in {-2..2} (or {-1,0,1}),
* seeds: seed = 1000 * layer_index + {0: x, 1: w, 2: dy},
* layouts: activations NHWC, filters KRSC, all float32 on the host
  (bf16 tensors are produced by rounding these on the device side).
"""
from __future__ import annotations

import numpy as np

from .networks import ConvLayer, alexnet, resnet18, resnet50, network  # noqa: F401

SEED_X, SEED_W, SEED_DY = 0, 1, 2


def out_dims(H, W, R, S, pad, stride):
    return (H + 2 * pad - R) // stride + 1, (W + 2 * pad - S) // stride + 1


def _rng(seed):
    return np.random.default_rng(int(seed))


def conv_inputs(n, c, h, w, k, r, s, pad, stride, seed=0, kind="normal", lo=-2, hi=2):
    """x (N,H,W,C), w (K,R,S,C), dy (N,P,Q,K) float32, seeded.

    kind="normal": x, dy ~ N(0,1), w ~ N(0, 1/(C R S)).
    kind="int":    all entries uniform integers in [lo, hi] (exact in fp32/tf32/bf16)."""
    p, q = out_dims(h, w, r, s, pad, stride)
    gx, gw, gd = _rng(seed * 1000 + SEED_X), _rng(seed * 1000 + SEED_W), _rng(seed * 1000 + SEED_DY)
    if kind == "int":
        x = gx.integers(lo, hi + 1, size=(n, h, w, c)).astype(np.float32)
        wt = gw.integers(lo, hi + 1, size=(k, r, s, c)).astype(np.float32)
        dy = gd.integers(lo, hi + 1, size=(n, p, q, k)).astype(np.float32)
    else:
        x = gx.standard_normal((n, h, w, c), dtype=np.float32)
        wt = (gw.standard_normal((k, r, s, c), dtype=np.float32) / np.float32(np.sqrt(c * r * s)))
        dy = gd.standard_normal((n, p, q, k), dtype=np.float32)
    return x, wt.astype(np.float32), dy


def torch_conv_inputs(layer, n, seed, device, dtype, kind="normal"):
    """Large device-side timing tensors (values irrelevant to timing): generated
    with a seeded torch.Generator on `device`."""
    import torch
    g = torch.Generator(device=device)
    p, q = out_dims(layer.h, layer.w, layer.r, layer.s, layer.pad, layer.stride)
    out = []
    for i, shape in enumerate([(n, layer.h, layer.w, layer.c), (layer.k, layer.r, layer.s, layer.c),
                               (n, p, q, layer.k)]):
        g.manual_seed(1000 * seed + i)
        if kind == "int":
            t = torch.randint(-2, 3, shape, generator=g, device=device, dtype=torch.int32).to(torch.float32)
        else:
            t = torch.randn(shape, generator=g, device=device, dtype=torch.float32)
            if i == 1:
                t = t / float(np.sqrt(layer.c * layer.r * layer.s))
        out.append(t.to(dtype).contiguous())
    return out


def random_timing_table(n, n_algos=3, seed=0, p_absent=0.2, t_max=1000, ws_max=1 << 20,
                        ties=False, sizes=None):
    """Random planner input: time[a][b] int64 (-1 = absent) and ws[a][b] uint64,
    b = 0..n (column 0 unused).  ties=True draws from a tiny value range so that
    ties are frequent (exercises the canonical tie-breaks)."""
    g = _rng(seed)
    time = np.full((n_algos, n + 1), -1, dtype=np.int64)
    ws = np.zeros((n_algos, n + 1), dtype=np.uint64)
    for a in range(n_algos):
        for b in range(1, n + 1):
            if sizes is not None and b not in sizes:
                continue
            if g.random() < p_absent:
                continue
            if ties:
                time[a, b] = int(g.integers(1, 6)) * b // max(1, int(g.integers(1, 3)))
                ws[a, b] = int(g.integers(0, 4)) * 256
            else:
                time[a, b] = int(g.integers(1, t_max)) * b // int(g.integers(1, 4)) + int(g.integers(0, 50))
                ws[a, b] = int(g.integers(0, ws_max)) * b // n
    return time, ws
