"""Full-size parity (BASELINE.json configs, N = 256) in the launch configuration
bench.py times: the WR plans from a real benchmark pass (64 MiB, powerOfTwo)
executed through ConvNet, checked on sampled output elements that the fp64
oracle computes one by one (oracle.*_at).  Tolerance (north_star): 1e-2 for
TF32 / BF16, 1e-5 for F32, relative to the largest magnitude among the
oracle's sampled values (never to the GPU output's own norm)."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_cluster_oyamabhm18_b200 as mu
from paper_conf_cluster_oyamabhm18_b200.network import ConvNet
from synthetic import network

pytestmark = pytest.mark.gpu

N = 256
SAMPLES = 24


TOL = {mu.MATH_F32: 1e-5, mu.MATH_TF32: 1e-2, mu.MATH_BF16: 1e-2}


def _check_layer(net, i, layer, rng, tol=1e-2):
    t = net.tensors[i]
    x = t["x"].float().cpu().numpy()
    w = t["w"].float().cpu().numpy()
    dy = t["dy"].float().cpu().numpy()
    y = t["y"].float().cpu().numpy()
    dx = t["dx"].float().cpu().numpy()
    dw = t["dw"].cpu().numpy()
    for out, fn in ((y, "fwd"), (dx, "dgrad"), (dw, "wgrad")):
        assert np.isfinite(out).all()
        idxs, refs = [], []
        for _ in range(SAMPLES):
            idx = tuple(int(rng.integers(0, d)) for d in out.shape)
            if fn == "fwd":
                ref = oracle.forward_at(x, w, layer.pad, layer.stride, idx)
            elif fn == "dgrad":
                ref = oracle.backward_data_at(dy, w, layer.h, layer.w, layer.pad, layer.stride, idx)
            else:
                ref = oracle.backward_filter_at(x, dy, layer.r, layer.s, layer.pad, layer.stride, idx)
            idxs.append(idx)
            refs.append(ref)
        scale = max(abs(r) for r in refs)
        assert scale > 0
        for idx, ref in zip(idxs, refs):
            assert abs(float(out[idx]) - ref) <= tol * scale, (layer.name, fn, idx, float(out[idx]), ref)


def _run(config, math, names=None):
    h = mu.Handle(0)
    h.set_policy(mu.POLICY_POW2)
    layers = network(config)
    if names:
        layers = [l for l in layers if l.name in names]
    net = ConvNet(h, layers, N, math, device="cuda")
    net.allocate(seed=3)
    limit = 64 << 20
    net.benchmark_all(limit)
    net.plan_wr(limit)
    net.iteration()
    torch.cuda.synchronize()
    rng = np.random.default_rng(0)
    for i, layer in enumerate(layers):
        _check_layer(net, i, layer, rng, TOL[math])


def test_alexnet_tf32_full_size_sampled():
    _run("alexnet", mu.MATH_TF32)


def test_resnet50_bf16_full_size_sampled():
    """BASELINE config 4 (ResNet-50, BF16, N = 256), every one of the 53 layers."""
    _run("resnet50", mu.MATH_BF16)


def test_resnet18_bf16_full_size_sampled():
    """BASELINE config 3 (ResNet-18, BF16, N = 256), every layer."""
    _run("resnet18", mu.MATH_BF16)


def test_alexnet_bf16_concurrent_full_size_sampled():
    """The bench step's executor (BackwardFilter on a side stream) at full size."""
    h = mu.Handle(0)
    h.set_policy(mu.POLICY_POW2)
    layers = network("alexnet")
    net = ConvNet(h, layers, N, mu.MATH_BF16, device="cuda")
    net.allocate(seed=4)
    limit = 64 << 20
    net.benchmark_all(limit)
    net.plan_wr(limit)
    net.iteration(concurrent=True)
    torch.cuda.synchronize()
    rng = np.random.default_rng(1)
    for i, layer in enumerate(layers):
        _check_layer(net, i, layer, rng, TOL[mu.MATH_BF16])


def test_alexnet_f32_full_size_sampled():
    """BASELINE config 2 at the paper's precision (fp32 CUDA-core path)."""
    _run("alexnet", mu.MATH_F32)


def test_alexnet_conv2_cfg1_f32():
    """BASELINE config 1: AlexNet conv2 forward, N = 8, F32, WR 8 MiB, `all`
    policy (b = 1..8): benchmark, DP, execute; the whole output against the
    fp64 oracle (normwise 1e-5)."""
    import paper_conf_cluster_oyamabhm18_b200.torch_api as T
    h = mu.Handle(0)
    h.set_policy(mu.POLICY_ALL)
    layer = [l for l in network("alexnet") if l.name == "conv2"][0]
    net = ConvNet(h, [layer], 8, mu.MATH_F32, device="cuda", types=(mu.FWD,))
    net.allocate(seed=9)
    limit = 8 << 20
    net.benchmark_all(limit)
    t, w = net.kernels[(0, mu.FWD)].table
    assert (t[mu.WINOGRAD] < 0).all()                      # 5x5: Winograd ineligible
    assert (t[mu.IM2COL_GEMM, 2:] < 0).all() and t[mu.IM2COL_GEMM, 1] > 0  # 4,665,600 B/sample: b = 1 only
    net.plan_wr(limit)
    net.iteration()
    torch.cuda.synchronize()
    tt = net.tensors[0]
    ref = oracle.conv_forward(tt["x"].cpu().numpy(), tt["w"].cpu().numpy(), layer.pad, layer.stride)
    got = tt["y"].double().cpu().numpy()
    assert np.max(np.abs(got - ref)) <= 1e-5 * np.max(np.abs(ref))
    h.set_policy(mu.POLICY_POW2)
