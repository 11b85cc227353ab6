"""NEXT-3 on one GPU: BackwardFilter with the cross-rank dW sum fused into its
epilogue (include/mucudnn.h mucu_conv_backward_filter_reduce), for
both targets: one NVLink multicast address (multimem.red; skipped where the box
cannot create a multicast object) and per-rank buffers (red.global.add, P2P).

With one rank the sum is 0 + dw, so the buffer must equal the rank's own
dW bit for bit, for every BackwardFilter kernel family: the tensor-core epilogues
(no split, cluster split-K with ordered groups, staged small-C, window, space-to-depth,
partial slots + reduction kernel) take the reduction in the kernel that writes the
final value (no extra launch), the F32 SIMT / Winograd / FFT / atomic writers are
followed by one push kernel.  The local dw must be unchanged by the fusion.
"""
import numpy as np
import pytest
import torch

import paper_conf_cluster_oyamabhm18_b200 as mu
from paper_conf_cluster_oyamabhm18_b200 import _lib
from paper_conf_cluster_oyamabhm18_b200 import torch_api as T
from paper_conf_cluster_oyamabhm18_b200.distributed import FusedGradReduce
from paper_conf_cluster_oyamabhm18_b200.network import ConvNet
from synthetic import network

pytestmark = pytest.mark.gpu

from gpu_util import handle  # noqa: E402

IG, I2C, WG, FFT = mu.IMPLICIT_GEMM, mu.IM2COL_GEMM, mu.WINOGRAD, mu.FFT

SHAPES = {
    "3x3_c64": (16, 64, 28, 28, 64, 3, 3, 1, 1),        # cluster split-K, ordered groups
    "5x5_c64_k192": (8, 64, 27, 27, 192, 5, 5, 2, 1),   # AlexNet conv2 (256-row tiles)
    "1x1_c256": (8, 256, 14, 14, 512, 1, 1, 0, 1),      # pointwise, partial slots (I2C)
    "11x11s4_c3": (8, 3, 224, 224, 64, 11, 11, 2, 4),   # AlexNet conv1: staged / window
    "7x7s2_c3": (8, 3, 224, 224, 64, 7, 7, 3, 2),       # ResNet conv1: staged / space-to-depth
    "3x3s2_c64": (8, 64, 56, 56, 128, 3, 3, 1, 2),
    "3x3_c512_small": (4, 512, 7, 7, 512, 3, 3, 1, 1),  # few pixels, long split chains
}


@pytest.fixture(scope="module", params=["p2p", "nvls"])
def nvls(request):
    torch.cuda.set_device(0)
    if request.param == "nvls":
        if not _lib.nvls_supported(0):
            pytest.skip("no NVLink multicast on this device")
        try:
            red = FusedGradReduce(8 << 20, 0, kind="nvls")  # 32 MiB of fp32 sums, world size 1
        except mu.MucuError as e:  # e.g. no NVSwitch fabric behind a one-GPU lease
            pytest.skip(f"NVLink multicast object unavailable: {e}")
    else:
        red = FusedGradReduce(8 << 20, 0, kind="p2p")
    yield red
    red.close()


def _dev(shape, dtype, seed):
    g = torch.Generator(device="cuda")
    g.manual_seed(seed)
    return torch.randn(shape, generator=g, device="cuda").to(dtype).contiguous()


def _ws(d, plan):
    ws = T.plan_workspace(d, mu.BWD_FILTER, plan)
    return torch.empty(max(ws, 256), dtype=torch.uint8, device="cuda") if ws else None


def _check(nv, d, plan, x, dy, beta, det, expect_fused):
    h = handle()
    h.set_deterministic(det)
    try:
        xs, wsh, ys = T.shapes(d)
        out0 = _dev(wsh, torch.float32, 9)
        ws = _ws(d, plan)
        ref = out0.clone()
        n0 = _lib.launch_count()
        T.conv_backward_filter(h, d, plan, x, dy, ref, beta=beta, workspace=ws)
        torch.cuda.synchronize()
        plain = _lib.launch_count() - n0
        dw = out0.clone()
        nv.begin()
        n0 = _lib.launch_count()
        T.conv_backward_filter_reduce(h, d, plan, x, dy, dw, nv.target(0), beta=beta, workspace=ws)
        fused = _lib.launch_count() - n0
        nv.end()
        torch.cuda.synchronize()
        sums = nv.sums[:dw.numel()].view(wsh)
        if det:
            assert torch.equal(dw, ref), "the fused call changed this rank's dw"
        assert torch.equal(sums, dw), (plan, float((sums - dw).abs().max()))
        if expect_fused is not None:
            assert fused == plain + (0 if expect_fused else 1), (plan, plain, fused)
    finally:
        h.set_deterministic(True)


@pytest.mark.parametrize("math", [mu.MATH_TF32, mu.MATH_BF16], ids=["tf32", "bf16"])
@pytest.mark.parametrize("name", list(SHAPES))
def test_fused_epilogue_tensor_core(nvls, name, math):
    """Tensor-core IG / I2C: the final dw writer takes the reduction (no extra
    launch), single and micro-batched plans, beta 0 and beta != 0."""
    shape = SHAPES[name]
    n = shape[0]
    d = mu.desc(*shape, math)
    dt = torch.bfloat16 if math == mu.MATH_BF16 else torch.float32
    xs, wsh, ys = T.shapes(d)
    x, dy = _dev(xs, dt, 1), _dev(ys, dt, 2)
    for plan in ([(IG, n)], [(I2C, n)], [(IG, n // 2), (I2C, n // 4), (IG, n // 4)]):
        for beta in (0.0, -0.5):
            _check(nvls, d, plan, x, dy, beta, True, True)


@pytest.mark.parametrize("name", ["3x3_c64", "5x5_c64_k192", "3x3_c512_small"])
def test_push_fallback(nvls, name):
    """Writers that do not fuse (F32 SIMT, Winograd output transform, FFT, atomic
    split-K partials) are followed by exactly one push kernel."""
    shape = SHAPES[name]
    n, r = shape[0], shape[5]
    for math in (mu.MATH_F32, mu.MATH_TF32):
        d = mu.desc(*shape, math)
        xs, wsh, ys = T.shapes(d)
        x, dy = _dev(xs, torch.float32, 3), _dev(ys, torch.float32, 4)
        plans = [[(IG, n)]] if math == mu.MATH_F32 else []
        if r == 3:
            plans.append([(IG, n // 2), (WG, n // 2)])
        for plan in plans:
            _check(nvls, d, plan, x, dy, 1.0, True, False)
    # non-deterministic mode: split partials with L2 atomics are not final values
    d = mu.desc(*shape, mu.MATH_BF16)
    xs, wsh, ys = T.shapes(d)
    x, dy = _dev(xs, torch.bfloat16, 5), _dev(ys, torch.bfloat16, 6)
    _check(nvls, d, [(IG, n)], x, dy, 0.0, False, None)


def test_fft_push(nvls):
    shape = (2, 64, 27, 27, 48, 5, 5, 2, 1)  # FFT eligible (F = 32)
    d = mu.desc(*shape, mu.MATH_F32)
    xs, wsh, ys = T.shapes(d)
    x, dy = _dev(xs, torch.float32, 7), _dev(ys, torch.float32, 8)
    _check(nvls, d, [(FFT, 1), (IG, 1)], x, dy, 0.0, True, False)
    _check(nvls, d, [(IG, 1), (FFT, 1)], x, dy, 0.0, True, False)


@pytest.mark.parametrize("concurrent", [False, True], ids=["sequential", "concurrent"])
def test_network_iteration_sums(nvls, concurrent):
    """ConvNet.iteration with the NVLS reduction (world size 1): the multicast
    sums equal the iteration's own filter gradients for every layer."""
    h = handle()
    layers = network("alexnet")
    net = ConvNet(h, layers, 16, mu.MATH_TF32)
    net.allocate(seed=3)
    net.benchmark_all(64 << 20)
    net.plan_wr(64 << 20)
    assert net.dw_flat.numel() <= nvls.numel
    net.nvls = nvls
    try:
        net.iteration(concurrent=concurrent)
        torch.cuda.synchronize()
        sums = nvls.sums[:net.dw_flat.numel()]
        assert torch.equal(sums, net.dw_flat)
        ref = net.dw_flat.clone()
        net.nvls = None
        net.iteration(concurrent=concurrent)
        torch.cuda.synchronize()
        assert torch.equal(net.dw_flat, ref)
    finally:
        net.nvls = None
