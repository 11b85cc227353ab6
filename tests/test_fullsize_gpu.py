"""Full-size parity (BASELINE.json configs, N = 256) in the launch configuration
bench.py times: the WR plans from a real benchmark pass (64 MiB, powerOfTwo)
executed through ConvNet, checked on sampled output elements that the fp64
oracle computes one by one (oracle.*_at).  Tolerance: normwise 1e-2 for
TF32 / BF16, scaled by the inf-norm of the full GPU output."""
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


def _check_layer(net, i, layer, rng):
    t = net.tensors[i]
    x = t["x"].float().cpu().numpy()
    w = t["w"].float().cpu().numpy()
    dy = t["dy"].float().cpu().numpy()
    y = t["y"].float().cpu().numpy()
    dx = t["dx"].float().cpu().numpy()
    dw = t["dw"].cpu().numpy()
    for out, fn in ((y, "fwd"), (dx, "dgrad"), (dw, "wgrad")):
        scale = float(np.max(np.abs(out)))
        assert np.isfinite(scale) and scale > 0
        for _ in range(SAMPLES):
            idx = tuple(int(rng.integers(0, d)) for d in out.shape)
            if fn == "fwd":
                ref = oracle.forward_at(x, w, layer.pad, layer.stride, idx)
            elif fn == "dgrad":
                ref = oracle.backward_data_at(dy, w, layer.h, layer.w, layer.pad, layer.stride, idx)
            else:
                ref = oracle.backward_filter_at(x, dy, layer.r, layer.s, layer.pad, layer.stride, idx)
            assert abs(float(out[idx]) - ref) <= 1e-2 * scale, (layer.name, fn, idx, float(out[idx]), ref)


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
        _check_layer(net, i, layer, rng)


def test_alexnet_tf32_full_size_sampled():
    _run("alexnet", mu.MATH_TF32)


def test_resnet50_bf16_full_size_sampled_layers():
    _run("resnet50", mu.MATH_BF16, names={"conv1", "layer1.0.conv2", "layer2.0.conv2", "layer3.0.downsample",
                                          "layer4.2.conv3", "layer1.0.conv1"})


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
        _check_layer(net, i, layer, rng)
