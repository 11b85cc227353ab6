"""Pins for the fp64 conv oracle (oracle/conv_oracle.c) -- CPU only.

The oracle is checked against things other than itself (SURVEY 8(c) "What
pins each part"):
* library routines: torch.nn.functional.conv2d / torch.nn.grad.conv2d_input /
  conv2d_weight in float64 on the CPU (a different implementation, NCHW);
* the adjoint identity <F(x,w),dy> = <x,D(dy,w)> = <w,G(x,dy)>, which ties the
  three operations to each other (a wrong sign/index in one of them breaks it);
* closed forms: one-hot x gives a filter slice; 1x1/stride-1/pad-0 is a
  matrix product (numpy.matmul); alpha/beta scaling.
"""
import numpy as np
import pytest
import torch

import oracle
from synthetic import conv_inputs

SHAPES = [
    # n, c, h, w, k, r, s, pad, stride
    (2, 3, 7, 6, 4, 3, 3, 1, 1),
    (1, 2, 9, 9, 3, 5, 5, 2, 1),
    (2, 3, 11, 10, 2, 3, 3, 1, 2),
    (1, 4, 12, 12, 3, 11, 11, 2, 4),   # AlexNet conv1 geometry, shrunk
    (2, 5, 8, 8, 6, 1, 1, 0, 2),       # ResNet downsample geometry
    (1, 3, 9, 9, 2, 7, 7, 3, 2),       # ResNet conv1 geometry
    (3, 2, 5, 5, 2, 3, 3, 0, 1),
    (1, 1, 4, 4, 1, 4, 4, 0, 1),       # P = Q = 1
]


def _nchw(a):
    return torch.from_numpy(np.ascontiguousarray(a.transpose(0, 3, 1, 2))).double()


def _kcrs(w):
    return torch.from_numpy(np.ascontiguousarray(w.transpose(0, 3, 1, 2))).double()


@pytest.mark.parametrize("shape", SHAPES)
def test_forward_matches_torch_conv2d(shape):
    n, c, h, w, k, r, s, pad, st = shape
    x, wt, _ = conv_inputs(n, c, h, w, k, r, s, pad, st, seed=7)
    y = oracle.conv_forward(x, wt, pad, st)
    ref = torch.nn.functional.conv2d(_nchw(x), _kcrs(wt), stride=st, padding=pad).numpy().transpose(0, 2, 3, 1)
    assert y.shape == ref.shape
    assert np.max(np.abs(y - ref)) <= 1e-12 * max(1.0, np.max(np.abs(ref)))


@pytest.mark.parametrize("shape", SHAPES)
def test_backward_data_matches_torch(shape):
    n, c, h, w, k, r, s, pad, st = shape
    _, wt, dy = conv_inputs(n, c, h, w, k, r, s, pad, st, seed=8)
    dx = oracle.conv_backward_data(dy, wt, h, w, pad, st)
    ref = torch.nn.grad.conv2d_input((n, c, h, w), _kcrs(wt), _nchw(dy), stride=st, padding=pad)
    ref = ref.numpy().transpose(0, 2, 3, 1)
    assert np.max(np.abs(dx - ref)) <= 1e-12 * max(1.0, np.max(np.abs(ref)))


@pytest.mark.parametrize("shape", SHAPES)
def test_backward_filter_matches_torch(shape):
    n, c, h, w, k, r, s, pad, st = shape
    x, _, dy = conv_inputs(n, c, h, w, k, r, s, pad, st, seed=9)
    dw = oracle.conv_backward_filter(x, dy, r, s, pad, st)
    ref = torch.nn.grad.conv2d_weight(_nchw(x), (k, c, r, s), _nchw(dy), stride=st, padding=pad)
    ref = ref.numpy().transpose(0, 2, 3, 1)
    assert np.max(np.abs(dw - ref)) <= 1e-12 * max(1.0, np.max(np.abs(ref)))


@pytest.mark.parametrize("shape", SHAPES)
def test_adjoint_identity(shape):
    """<F(x,w), dy> = <x, D(dy,w)> = <w, G(x,dy)>: the three ops of P:L56 are
    one bilinear form read three ways."""
    n, c, h, w, k, r, s, pad, st = shape
    x, wt, dy = conv_inputs(n, c, h, w, k, r, s, pad, st, seed=10)
    a = np.sum(oracle.conv_forward(x, wt, pad, st) * dy)
    b = np.sum(x.astype(np.float64) * oracle.conv_backward_data(dy, wt, h, w, pad, st))
    g = np.sum(wt.astype(np.float64) * oracle.conv_backward_filter(x, dy, r, s, pad, st))
    scale = max(1.0, abs(a))
    assert abs(a - b) <= 1e-11 * scale
    assert abs(a - g) <= 1e-11 * scale


def test_one_hot_input_gives_filter_slice():
    """x = e_(n0,h0,w0,c0)  =>  y[n0,p,q,k] = w[k, h0 - p*st + pad, w0 - q*st + pad, c0]."""
    n, c, h, w, k, r, s, pad, st = 2, 3, 9, 8, 4, 3, 5, 2, 2
    _, wt, _ = conv_inputs(n, c, h, w, k, r, s, pad, st, seed=11)
    x = np.zeros((n, h, w, c), np.float32)
    n0, h0, w0, c0 = 1, 4, 3, 2
    x[n0, h0, w0, c0] = 1.0
    y = oracle.conv_forward(x, wt, pad, st)
    P, Q = oracle.output_dims(h, w, r, s, pad, st)
    expect = np.zeros_like(y)
    for p in range(P):
        for q in range(Q):
            rr, ss = h0 - p * st + pad, w0 - q * st + pad
            if 0 <= rr < r and 0 <= ss < s:
                expect[n0, p, q, :] = wt[:, rr, ss, c0]
    assert np.array_equal(y, expect)


def test_1x1_is_matmul():
    n, c, h, w, k = 2, 5, 4, 3, 6
    x, wt, dy = conv_inputs(n, c, h, w, k, 1, 1, 0, 1, seed=12)
    y = oracle.conv_forward(x, wt, 0, 1)
    ref = np.matmul(x.astype(np.float64), wt[:, 0, 0, :].astype(np.float64).T)
    assert np.max(np.abs(y - ref)) <= 1e-13
    dx = oracle.conv_backward_data(dy, wt, h, w, 0, 1)
    assert np.max(np.abs(dx - np.matmul(dy.astype(np.float64), wt[:, 0, 0, :].astype(np.float64)))) <= 1e-13
    dw = oracle.conv_backward_filter(x, dy, 1, 1, 0, 1)
    ref_dw = np.matmul(dy.reshape(-1, k).astype(np.float64).T, x.reshape(-1, c).astype(np.float64))
    assert np.max(np.abs(dw[:, 0, 0, :] - ref_dw)) <= 1e-12


def test_alpha_beta():
    """Output scale of P:L58 (reading G5): out = alpha * op + beta * out."""
    n, c, h, w, k, r, s, pad, st = 2, 3, 6, 6, 4, 3, 3, 1, 1
    x, wt, dy = conv_inputs(n, c, h, w, k, r, s, pad, st, seed=13)
    y0 = conv_inputs(n, k, h, w, c, r, s, pad, st, seed=14)[0]
    base = oracle.conv_forward(x, wt, pad, st)
    got = oracle.conv_forward(x, wt, pad, st, alpha=0.5, beta=-2.0, y=y0)
    assert np.max(np.abs(got - (0.5 * base - 2.0 * y0))) <= 1e-12
    dw0 = conv_inputs(1, c, r, s, k, 1, 1, 0, 1, seed=15)[0].reshape(1, r, s, c).repeat(k, 0)
    base = oracle.conv_backward_filter(x, dy, r, s, pad, st)
    got = oracle.conv_backward_filter(x, dy, r, s, pad, st, alpha=1.0, beta=1.0, dw=dw0)
    assert np.max(np.abs(got - (base + dw0))) <= 1e-12


def test_gradient_sum_over_samples():
    """dL/dw = sum_n dl_n/dw -- WGRAD of the batch equals the sum of
    per-sample WGRADs (the property micro-batching relies on)."""
    n, c, h, w, k, r, s, pad, st = 4, 2, 7, 7, 3, 3, 3, 1, 2
    x, _, dy = conv_inputs(n, c, h, w, k, r, s, pad, st, seed=16)
    full = oracle.conv_backward_filter(x, dy, r, s, pad, st)
    parts = sum(oracle.conv_backward_filter(x[i:i + 1], dy[i:i + 1], r, s, pad, st) for i in range(n))
    assert np.max(np.abs(full - parts)) <= 1e-12


@pytest.mark.parametrize("shape", SHAPES[:4])
def test_single_element_helpers_match_full(shape):
    n, c, h, w, k, r, s, pad, st = shape
    x, wt, dy = conv_inputs(n, c, h, w, k, r, s, pad, st, seed=17)
    y = oracle.conv_forward(x, wt, pad, st)
    dx = oracle.conv_backward_data(dy, wt, h, w, pad, st)
    dw = oracle.conv_backward_filter(x, dy, r, s, pad, st)
    g = np.random.default_rng(0)
    for _ in range(5):
        idx = tuple(int(g.integers(0, d)) for d in y.shape)
        assert oracle.forward_at(x, wt, pad, st, idx) == pytest.approx(y[idx], abs=1e-12)
        idx = tuple(int(g.integers(0, d)) for d in dx.shape)
        assert oracle.backward_data_at(dy, wt, h, w, pad, st, idx) == pytest.approx(dx[idx], abs=1e-12)
        idx = tuple(int(g.integers(0, d)) for d in dw.shape)
        assert oracle.backward_filter_at(x, dy, r, s, pad, st, idx) == pytest.approx(dw[idx], abs=1e-12)
