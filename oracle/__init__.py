"""oracle -- TEST INFRASTRUCTURE ONLY (not part of the product path).

Plain CPU reference for mu-cuDNN's hot path (Oyama, Ben-Nun, Hoefler,
Matsuoka, CLUSTER 2018; /root/reference/PAPER.md):

* ``conv_forward`` / ``conv_backward_data`` / ``conv_backward_filter``: the
  fp64 seven-loop direct convolution of Alg. 1 (Sec. II) and its two
  backward operations, in ``conv_oracle.c`` (plain C + OpenMP over
  the independent output elements).
* ``planner_bf``: brute-force enumeration of the WR / WD optimisation problems
  of Sec. III-B / III-C.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  It
shares no code with ``paper_conf_cluster_oyamabhm18_b200`` and never imports
it; the product never imports this.

Parity status: the conv functions are pinned by tests/test_oracle_conv.py
(torch fp64 library routines, the adjoint identity, one-hot closed forms,
1x1 == matmul); the planner by tests/test_oracle_planner.py (closed forms,
the paper's worked examples, scipy.optimize.milp).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "conv_oracle.c")
_lib = None


def build(force: bool = False) -> str:
    """Compile conv_oracle.c into oracle/liboracle.so (gcc -O2 -fopenmp)."""
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-o", _LIB_PATH, _SRC])
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        i, d = ctypes.c_int, ctypes.c_double
        pd = ctypes.POINTER(ctypes.c_double)
        pf = ctypes.POINTER(ctypes.c_float)
        for name, ptrs in (("oracle_conv_forward", (pd, pd, pd)),
                           ("oracle_conv_backward_data", (pd, pd, pd)),
                           ("oracle_conv_backward_filter", (pd, pd, pd))):
            fn = getattr(lib, name)
            fn.restype = i
            fn.argtypes = [i] * 9 + [d, ptrs[0], ptrs[1], d, ptrs[2]]
        lib.oracle_forward_at.restype = d
        lib.oracle_forward_at.argtypes = [i] * 8 + [pf, pf] + [i] * 4
        lib.oracle_backward_data_at.restype = d
        lib.oracle_backward_data_at.argtypes = [i] * 8 + [pf, pf] + [i] * 4
        lib.oracle_backward_filter_at.restype = d
        lib.oracle_backward_filter_at.argtypes = [i] * 9 + [pf, pf] + [i] * 4
        _lib = lib
    return _lib


def output_dims(H, W, R, S, pad, stride):
    """P = (H + 2 pad - R) // stride + 1 (standard extent)."""
    return (H + 2 * pad - R) // stride + 1, (W + 2 * pad - S) // stride + 1


def _f64(a):
    return np.ascontiguousarray(a, dtype=np.float64)


def _ptr(a, ct=ctypes.c_double):
    return a.ctypes.data_as(ctypes.POINTER(ct))


def conv_forward(x, w, pad, stride, alpha=1.0, beta=0.0, y=None):
    """y = alpha * conv(x, w) + beta * y.  x: (N,H,W,C), w: (K,R,S,C) -> y: (N,P,Q,K), fp64."""
    x, w = _f64(x), _f64(w)
    N, H, W, C = x.shape
    K, R, S, C2 = w.shape
    assert C == C2
    P, Q = output_dims(H, W, R, S, pad, stride)
    out = np.zeros((N, P, Q, K)) if y is None else _f64(y).copy()
    rc = _load().oracle_conv_forward(N, C, H, W, K, R, S, pad, stride, alpha, _ptr(x), _ptr(w), beta, _ptr(out))
    assert rc == 0
    return out


def conv_backward_data(dy, w, H, W, pad, stride, alpha=1.0, beta=0.0, dx=None):
    """dx = alpha * conv^T(dy, w) + beta * dx.  dy: (N,P,Q,K), w: (K,R,S,C) -> dx: (N,H,W,C)."""
    dy, w = _f64(dy), _f64(w)
    N, P, Q, K = dy.shape
    K2, R, S, C = w.shape
    assert K == K2 and output_dims(H, W, R, S, pad, stride) == (P, Q)
    out = np.zeros((N, H, W, C)) if dx is None else _f64(dx).copy()
    rc = _load().oracle_conv_backward_data(N, C, H, W, K, R, S, pad, stride, alpha, _ptr(dy), _ptr(w), beta, _ptr(out))
    assert rc == 0
    return out


def conv_backward_filter(x, dy, R, S, pad, stride, alpha=1.0, beta=0.0, dw=None):
    """dw = alpha * sum_n x_n (*) dy_n + beta * dw.  x: (N,H,W,C), dy: (N,P,Q,K) -> dw: (K,R,S,C)."""
    x, dy = _f64(x), _f64(dy)
    N, H, W, C = x.shape
    N2, P, Q, K = dy.shape
    assert N == N2 and output_dims(H, W, R, S, pad, stride) == (P, Q)
    out = np.zeros((K, R, S, C)) if dw is None else _f64(dw).copy()
    rc = _load().oracle_conv_backward_filter(N, C, H, W, K, R, S, pad, stride, alpha, _ptr(x), _ptr(dy), beta, _ptr(out))
    assert rc == 0
    return out


def _f32(a):
    return np.ascontiguousarray(a, dtype=np.float32)


def forward_at(x32, w32, pad, stride, idx):
    """One element y[n,p,q,k] (alpha=1, beta=0) from fp32-stored inputs, accumulated in fp64."""
    x32, w32 = _f32(x32), _f32(w32)
    N, H, W, C = x32.shape
    K, R, S, _ = w32.shape
    n, p, q, k = idx
    return _load().oracle_forward_at(C, H, W, K, R, S, pad, stride, _ptr(x32, ctypes.c_float),
                                     _ptr(w32, ctypes.c_float), n, p, q, k)


def backward_data_at(dy32, w32, H, W, pad, stride, idx):
    dy32, w32 = _f32(dy32), _f32(w32)
    K, R, S, C = w32.shape
    n, h, w, c = idx
    return _load().oracle_backward_data_at(C, H, W, K, R, S, pad, stride, _ptr(dy32, ctypes.c_float),
                                           _ptr(w32, ctypes.c_float), n, h, w, c)


def backward_filter_at(x32, dy32, R, S, pad, stride, idx):
    x32, dy32 = _f32(x32), _f32(dy32)
    N, H, W, C = x32.shape
    K = dy32.shape[3]
    k, r, s, c = idx
    return _load().oracle_backward_filter_at(N, C, H, W, K, R, S, pad, stride, _ptr(x32, ctypes.c_float),
                                             _ptr(dy32, ctypes.c_float), k, r, s, c)
