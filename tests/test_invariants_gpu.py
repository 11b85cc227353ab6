"""GPU tests of the paper's semantic invariants at the sizes where they can
break, and of the planner entry points that run on the GPU.

* I1: micro-batched FWD / DGRAD are bitwise equal to the same
  algorithm at full N -- at N = 256, where the tile heuristics (pick_bn waves,
  256 / 512-row tiles, merged im2col boxes) change with the micro-batch size b.
* Deterministic BackwardFilter: split-K partials are
  combined in a fixed order, so two runs on random data give bitwise-equal dW.
* Workspace prefix reuse inside one call: a plan that alternates
  Winograd and im2col must rebuild Winograd's transformed filter U.
* mucu_network_plan (benchmark + fronts + MCKP on the GPU) and the file DB.
* A WD-planned network iteration checked against the fp64 oracle.
"""
import os

import numpy as np
import pytest
import torch

import oracle
import paper_conf_cluster_oyamabhm18_b200 as mu
from paper_conf_cluster_oyamabhm18_b200 import torch_api as T
from paper_conf_cluster_oyamabhm18_b200.network import ConvNet
from synthetic import conv_inputs, network

pytestmark = pytest.mark.gpu

from gpu_util import handle, oracle_ref, run_gpu  # noqa: E402

IG, I2C, WG = mu.IMPLICIT_GEMM, mu.IM2COL_GEMM, mu.WINOGRAD


def _dev(shape, dtype, seed, scale=1.0):
    g = torch.Generator(device="cuda")
    g.manual_seed(seed)
    return (torch.randn(shape, generator=g, device="cuda") * scale).to(dtype).contiguous()


def _run_plan(d, conv_type, plan, a, b, beta=0.0, out=None):
    ws = T.plan_workspace(d, conv_type, plan)
    wst = torch.empty(max(ws, 256), dtype=torch.uint8, device="cuda") if ws else None
    r = T.run(handle(), d, conv_type, plan, a, b, out, beta=beta, workspace=wst)
    torch.cuda.synchronize()
    return r


# ------------------------------------------------------------ prefix reuse --
@pytest.mark.parametrize("math", [mu.MATH_F32, mu.MATH_TF32, mu.MATH_BF16], ids=["f32", "tf32", "bf16"])
@pytest.mark.parametrize("conv_type", [mu.FWD, mu.BWD_DATA], ids=["fwd", "dgrad"])
def test_winograd_prefix_rebuilt_after_other_algorithm(conv_type, math):
    """[(WG,2),(I2C,1),(WG,1)]: im2col writes its col / dcol buffer over U at
    workspace offset 0 (R*S*C*elt % 16 == 0: no padded-filter prefix), so the
    second Winograd part must recompute U (exact on integer data)."""
    shape = (4, 32, 9, 9, 48, 3, 3, 1, 1)
    d = mu.desc(*shape, math)
    x, w, dy = conv_inputs(*shape, seed=41, kind="int")
    ref = oracle_ref(shape, conv_type, x, w, dy)
    if math == mu.MATH_BF16:
        ref = torch.from_numpy(ref).to(torch.bfloat16).double().numpy()
    for plan in ([(WG, 2), (I2C, 1), (WG, 1)], [(WG, 1), (IG, 1), (I2C, 1), (WG, 1)]):
        got, _ = run_gpu(d, conv_type, plan, x, w, dy)
        assert np.array_equal(got, ref), plan


# ------------------------------------------------------------ I1 at N=256 --
FULL = {
    "alexnet_conv2": ((256, 64, 27, 27, 192, 5, 5, 2, 1), [mu.MATH_TF32, mu.MATH_BF16]),
    "resnet50_l1_3x3": ((256, 64, 56, 56, 64, 3, 3, 1, 1), [mu.MATH_BF16, mu.MATH_TF32]),
    "alexnet_conv1": ((256, 3, 224, 224, 64, 11, 11, 2, 4), [mu.MATH_TF32, mu.MATH_BF16]),
    "resnet50_l3_1x1": ((256, 1024, 14, 14, 256, 1, 1, 0, 1), [mu.MATH_BF16]),
    "resnet50_l2_3x3s2": ((256, 128, 56, 56, 128, 3, 3, 1, 2), [mu.MATH_BF16]),
}
I1_CASES = [(name, math, t, a) for name, (shape, maths) in FULL.items() for math in maths
            for t in (mu.FWD, mu.BWD_DATA) for a in (IG, I2C, WG)
            if a != WG or (shape[5] == 3 and shape[8] == 1)]
SPLIT = [(128,), (64,), (32,), (16,), (8,), (4,), (2,), (1,), (1,)]


@pytest.mark.parametrize("env", ["default", "mt2", "mt4"])
@pytest.mark.parametrize("case", I1_CASES,
                         ids=lambda c: f"{c[0]}-{['f32', 'tf32', 'bf16'][c[1]]}-{mu.TYPE_NAMES[c[2]]}-{mu.ALGO_NAMES[c[3]]}")
def test_i1_full_size_bitwise(case, env, monkeypatch):
    """I1 at N = 256 with parts 128/64/32/16/8/4/2/1/1 -- every micro-batch size
    the powerOfTwo policy produces, each with the tiling its own size selects."""
    if env != "default":
        monkeypatch.setenv("MUCU_FORCE_MT", env[-1])
    name, math, conv_type, algo = case
    shape = FULL[name][0]
    n, c, h, w_, k, r, s, pad, st = shape
    d = mu.desc(*shape, math)
    dt = torch.bfloat16 if math == mu.MATH_BF16 else torch.float32
    xs, wsh, ys = T.shapes(d)
    a = _dev(xs if conv_type == mu.FWD else ys, dt, 1)
    b = _dev(wsh, dt, 2, 1.0 / np.sqrt(c * r * s))
    full = _run_plan(d, conv_type, [(algo, n)], a, b)
    split = _run_plan(d, conv_type, [(algo, p[0]) for p in SPLIT], a, b)
    assert torch.isfinite(full.float()).all()
    assert torch.equal(full, split)


# --------------------------------------------- deterministic BackwardFilter --
DET = {
    "3x3_c64": (32, 64, 28, 28, 64, 3, 3, 1, 1),
    "3x3_c128_k192": (16, 128, 14, 14, 192, 3, 3, 1, 1),
    "5x5_alexnet_conv2": (16, 64, 27, 27, 192, 5, 5, 2, 1),
    "1x1": (32, 256, 14, 14, 512, 1, 1, 0, 1),
    "1x1s2": (16, 256, 28, 28, 512, 1, 1, 0, 2),
    "11x11s4_c3": (16, 3, 224, 224, 64, 11, 11, 2, 4),
    "7x7s2_c3": (16, 3, 224, 224, 64, 7, 7, 3, 2),
    "3x3s2_c64": (16, 64, 56, 56, 128, 3, 3, 1, 2),
}


@pytest.mark.parametrize("math", [mu.MATH_F32, mu.MATH_TF32, mu.MATH_BF16], ids=["f32", "tf32", "bf16"])
@pytest.mark.parametrize("name", list(DET))
def test_wgrad_bitwise_reproducible(name, math):
    """Two runs of every BackwardFilter algorithm (and a micro-batched plan) on
    N(0,1) data give bitwise-equal dW, and match the oracle within tolerance on
    a sample of elements."""
    shape = DET[name]
    n, c, h, w_, k, r, s, pad, st = shape
    d = mu.desc(*shape, math)
    dt = torch.bfloat16 if math == mu.MATH_BF16 else torch.float32
    xs, wsh, ys = T.shapes(d)
    x = _dev(xs, dt, 3)
    dy = _dev(ys, dt, 4)
    algos = [IG, I2C] + ([WG] if r == 3 and s == 3 and st == 1 else [])
    plans = [[(a, n)] for a in algos] + [[(algos[-1], n // 2), (IG, n // 4), (I2C, n // 4)]]
    xh = x.float().cpu().numpy()
    dyh = dy.float().cpu().numpy()
    rng = np.random.default_rng(0)
    idx = [tuple(int(rng.integers(0, e)) for e in wsh) for _ in range(12)]
    refs = np.array([oracle.backward_filter_at(xh, dyh, r, s, pad, st, i) for i in idx])
    tol = 1e-5 if math == mu.MATH_F32 else 1e-2
    for plan in plans:
        dw1 = _run_plan(d, mu.BWD_FILTER, plan, x, dy, out=torch.full(wsh, float("nan"), device="cuda"))
        dw2 = _run_plan(d, mu.BWD_FILTER, plan, x, dy, out=torch.full(wsh, float("nan"), device="cuda"))
        assert torch.equal(dw1, dw2), plan
        got = np.array([float(dw1[i]) for i in idx])
        assert np.max(np.abs(got - refs)) <= tol * np.max(np.abs(refs)), plan


@pytest.mark.parametrize("math", [mu.MATH_TF32, mu.MATH_BF16], ids=["tf32", "bf16"])
def test_wgrad_beta_applied_once_per_tile(math):
    """The user's beta scales dw exactly once even when the reduction is split
    across CTAs (split 0 applies it, later splits add): dw = 2*op - 1*dw0 on
    integer data is exact."""
    shape = (16, 64, 28, 28, 64, 3, 3, 1, 1)
    d = mu.desc(*shape, math)
    x, w, dy = conv_inputs(*shape, seed=47, kind="int", lo=-1, hi=1)
    out0 = np.random.default_rng(2).integers(-2, 3, size=(64, 3, 3, 64)).astype(np.float32)
    ref = oracle_ref(shape, mu.BWD_FILTER, x, w, dy, alpha=2.0, beta=-1.0, out0=out0)
    for plan in ([(IG, 16)], [(I2C, 16)], [(WG, 8), (IG, 8)]):
        got, _ = run_gpu(d, mu.BWD_FILTER, plan, x, w, dy, alpha=2.0, beta=-1.0, out0=out0)
        assert np.array_equal(got, ref), plan


# ---------------------------------------------------- planner on the GPU --
def test_network_plan_on_gpu_matches_oracle():
    """mucu_network_plan: benchmark every unique (desc, type), build the fronts,
    solve the MCKP; then run each kernel's plan in its segment of one network
    workspace and compare with the oracle (integer data: exact)."""
    shapes = [(8, 32, 13, 13, 64, 3, 3, 1, 1), (8, 64, 13, 13, 64, 3, 3, 1, 1), (8, 32, 13, 13, 64, 3, 3, 1, 1)]
    math = mu.MATH_BF16
    h = handle()
    h.set_policy(mu.POLICY_ALL)
    net = mu.Network()
    ids = []
    for sh in shapes:
        for t in (mu.FWD, mu.BWD_DATA, mu.BWD_FILTER):
            ids.append((sh, t, net.add(mu.desc(*sh, math), t)))
    total = 6 << 20
    need = max(mu.benchmark_scratch_size(mu.desc(*sh, math), t, total) for sh, t, _ in ids)
    scratch = torch.empty(need + 256, dtype=torch.uint8, device="cuda")
    off = (-scratch.data_ptr()) % 256
    net.plan(h, total, scratch.data_ptr() + off, need, torch.cuda.current_stream().cuda_stream)
    segs = [net.get(kid) for _, _, kid in ids]
    end = max(o + nb for _, o, nb, _ in segs)
    assert end <= total
    for (_, o, nb, _), (_, o2, nb2, _) in zip(segs, segs[1:]):
        assert o + nb <= o2  # disjoint segments in registration order (reading G18)
    for (sh, t, kid), (plan, o, nb, est) in zip(ids, segs):
        assert sum(b for _, b in plan) == sh[0] and est > 0
        d = mu.desc(*sh, math)
        assert T.plan_workspace(d, t, plan) <= nb
        x, w, dy = conv_inputs(*sh, seed=kid, kind="int")
        ref = oracle_ref(sh, t, x, w, dy)
        if t != mu.BWD_FILTER:
            ref = torch.from_numpy(ref).to(torch.bfloat16).double().numpy()
        got, _ = run_gpu(d, t, plan, x, w, dy)
        assert np.array_equal(got, ref), (sh, t, plan)
    h.set_policy(mu.POLICY_POW2)


def test_tables_db_roundtrip(tmp_path):
    """File DB: tables saved after a benchmark pass and loaded into a
    fresh network give identical tables and identical WR / WD plans."""
    h = handle()
    layers = network("alexnet")[2:4]
    a = ConvNet(h, layers, 16, mu.MATH_TF32, device="cuda")
    limit = 8 << 20
    a.benchmark_all(limit)
    path = str(tmp_path / "db.npz")
    a.save_tables(path, limit, "pow2")
    b = ConvNet(h, layers, 16, mu.MATH_TF32, device="cuda")
    assert b.load_tables(path, limit, "pow2")
    assert not b.load_tables(path, limit + 1, "pow2")  # another limit: not in the DB
    assert b.load_tables(path, limit, "pow2")
    for key in a.kernels:
        ta, wa = a.kernels[key].table
        tb, wb = b.kernels[key].table
        assert np.array_equal(ta, tb) and np.array_equal(wa, wb)
    a.plan_wr(limit)
    b.plan_wr(limit)
    assert all(a.kernels[k].plan == b.kernels[k].plan for k in a.kernels)
    a.plan_wd(6 * limit)
    b.plan_wd(6 * limit)
    assert all(a.kernels[k].plan == b.kernels[k].plan and a.kernels[k].ws_offset == b.kernels[k].ws_offset
               for k in a.kernels)


@pytest.mark.parametrize("math", [mu.MATH_TF32, mu.MATH_BF16], ids=["tf32", "bf16"])
def test_wd_planned_iteration_matches_oracle(math):
    """A WD-planned AlexNet iteration (one shared workspace, segments from the
    MCKP, concurrent backward) checked element-wise against the fp64 oracle on
    integer data (exact), full tensors at N = 8."""
    h = handle()
    layers = network("alexnet")
    net = ConvNet(h, layers, 8, math, device="cuda")
    net.allocate(seed=7, kind="int")
    net.benchmark_all(8 << 20)
    net.plan_wd(len(net.kernels) * (8 << 20) // 2)
    assert net.net_ws is not None
    net.iteration(concurrent=True)
    torch.cuda.synchronize()
    for i, l in enumerate(layers):
        t = net.tensors[i]
        x, w, dy = (t[k].float().cpu().numpy() for k in ("x", "w", "dy"))
        refs = {"y": oracle.conv_forward(x, w, l.pad, l.stride),
                "dx": oracle.conv_backward_data(dy, w, l.h, l.w, l.pad, l.stride),
                "dw": oracle.conv_backward_filter(x, dy, l.r, l.s, l.pad, l.stride)}
        for k, ref in refs.items():
            if k != "dw" and math == mu.MATH_BF16:
                ref = torch.from_numpy(ref).to(torch.bfloat16).double().numpy()
            got = t[k].double().cpu().numpy()
            assert np.array_equal(got, ref), (l.name, k)
