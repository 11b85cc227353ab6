"""GPU parity: every (algorithm x conv type x math) of the CUDA path against the
fp64 oracle, through the C ABI, plus the paper's semantic invariants.

Tolerances (north_star):
* F32 SIMT: max|d| / ||ref||_inf <= 1e-5;
* TF32 / BF16 tensor cores and Winograd: <= 1e-2 (BF16 outputs are rounded);
* integer-valued inputs in {-2..2}: every path is exact (sums < 2^24), so the
  comparison is bit-exact against the oracle (BF16 output: RNE(oracle)).
Invariants: I1 micro-batched FWD/DGRAD bitwise equal to the same algorithm at
full N; I2 WGRAD summed over micro-batches equals full-batch dW
(P:L52-58); I6 no write outside the declared workspace.
"""
import numpy as np
import pytest
import torch

import paper_conf_cluster_oyamabhm18_b200 as mu
from synthetic import conv_inputs

pytestmark = pytest.mark.gpu

from gpu_util import normwise_err, oracle_ref, run_gpu, stored  # noqa: E402

# n, c, h, w, k, r, s, pad, stride -- several tiles and a ragged tail each
SHAPES = {
    "3x3s1": (3, 32, 13, 13, 40, 3, 3, 1, 1),
    "3x3s1_c64": (2, 64, 12, 12, 64, 3, 3, 1, 1),      # vector gather paths (C, K % 64 == 0)
    "3x3s1_c128": (2, 128, 10, 10, 192, 3, 3, 1, 1),
    "3x3s2_c64": (2, 64, 15, 15, 128, 3, 3, 1, 2),
    "3x3s1_p0_odd": (2, 16, 9, 11, 24, 3, 3, 0, 1),
    "3x3s1_p2": (2, 32, 7, 7, 32, 3, 3, 2, 1),
    "5x5s1": (2, 64, 11, 11, 48, 5, 5, 2, 1),          # AlexNet conv2 geometry
    "11x11s4_c3": (2, 3, 35, 35, 64, 11, 11, 2, 4),    # AlexNet conv1 geometry
    "7x7s2_c3": (2, 3, 23, 23, 64, 7, 7, 3, 2),        # ResNet conv1 geometry
    "11x11s4_c3_ragged": (2, 3, 30, 27, 64, 11, 11, 2, 4),  # space-to-depth with ragged super-pixel edges
    "5x5s2_c2_k32": (2, 2, 17, 19, 32, 5, 5, 2, 2),
    "4x4s3_c3_p0": (3, 3, 20, 22, 64, 4, 4, 0, 3),
    "11x11s4_c3_w32": (2, 3, 35, 32, 64, 11, 11, 2, 4),   # W*C*elt % 16 == 0: staged-row FWD / WGRAD
    "7x7s2_c3_w32": (3, 3, 30, 32, 64, 7, 7, 3, 2),
    "3x3s2": (2, 64, 14, 14, 128, 3, 3, 1, 2),
    "1x1s1": (3, 64, 10, 10, 96, 1, 1, 0, 1),
    "1x1s2": (2, 64, 14, 14, 128, 1, 1, 0, 2),
    "big_k": (1, 128, 6, 6, 256, 3, 3, 1, 1),
}

TOL = {mu.MATH_F32: 1e-5, mu.MATH_TF32: 1e-2, mu.MATH_BF16: 1e-2}


def _eligible(shape, conv_type, algo):
    n, c, h, w, k, r, s, pad, st = shape
    if algo == mu.WINOGRAD:
        return r == 3 and s == 3 and st == 1 and pad <= 2
    return True


def _inputs(shape, kind, seed=3):
    n, c, h, w, k, r, s, pad, st = shape
    return conv_inputs(n, c, h, w, k, r, s, pad, st, seed=seed, kind=kind)


CASES = [(name, t, a) for name in SHAPES for t in (mu.FWD, mu.BWD_DATA, mu.BWD_FILTER)
         for a in (mu.IMPLICIT_GEMM, mu.IM2COL_GEMM, mu.WINOGRAD) if _eligible(SHAPES[name], t, a)]


def _ids(c):
    return f"{c[0]}-{mu.TYPE_NAMES[c[1]]}-{mu.ALGO_NAMES[c[2]]}"


@pytest.mark.parametrize("math", [mu.MATH_F32, mu.MATH_TF32, mu.MATH_BF16], ids=["f32", "tf32", "bf16"])
@pytest.mark.parametrize("case", CASES, ids=_ids)
def test_parity_random(case, math):
    name, conv_type, algo = case
    shape = SHAPES[name]
    d = mu.desc(*shape, math)
    x, w, dy = _inputs(shape, "normal")
    xs, ws_, dys = stored(x, math), stored(w, math), stored(dy, math)
    ref = oracle_ref(shape, conv_type, xs, ws_, dys)
    got, _ = run_gpu(d, conv_type, [(algo, shape[0])], x, w, dy)
    assert got.shape == ref.shape
    assert normwise_err(got, ref) <= TOL[math]


@pytest.mark.parametrize("math", [mu.MATH_F32, mu.MATH_TF32, mu.MATH_BF16], ids=["f32", "tf32", "bf16"])
@pytest.mark.parametrize("case", CASES, ids=_ids)
def test_parity_integer_exact(case, math):
    name, conv_type, algo = case
    shape = SHAPES[name]
    d = mu.desc(*shape, math)
    x, w, dy = _inputs(shape, "int", seed=5)
    ref = oracle_ref(shape, conv_type, x, w, dy)
    if math == mu.MATH_BF16 and conv_type != mu.BWD_FILTER:
        ref = torch.from_numpy(ref).to(torch.bfloat16).double().numpy()  # output rounding RNE
    got, _ = run_gpu(d, conv_type, [(algo, shape[0])], x, w, dy)
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("math", [mu.MATH_F32, mu.MATH_TF32, mu.MATH_BF16], ids=["f32", "tf32", "bf16"])
@pytest.mark.parametrize("case", [c for c in CASES if c[1] != mu.BWD_FILTER], ids=_ids)
def test_micro_batch_bit_identity(case, math):
    """I1: FWD / DGRAD split into micro-batches == the same algorithm at full N, bitwise."""
    name, conv_type, algo = case
    shape = list(SHAPES[name])
    shape[0] = 5
    shape = tuple(shape)
    d = mu.desc(*shape, math)
    x, w, dy = _inputs(shape, "normal", seed=9)
    full, _ = run_gpu(d, conv_type, [(algo, 5)], x, w, dy)
    split, _ = run_gpu(d, conv_type, [(algo, 3), (algo, 1), (algo, 1)], x, w, dy)
    assert np.array_equal(full, split)


@pytest.mark.parametrize("math", [mu.MATH_F32, mu.MATH_TF32, mu.MATH_BF16], ids=["f32", "tf32", "bf16"])
@pytest.mark.parametrize("name", ["3x3s1", "11x11s4_c3", "1x1s2"])
def test_wgrad_accumulates_over_micro_batches(name, math):
    """I2: dW summed over micro-batches (beta = 1 after the first)
    equals full-batch dW: exact on integer data, within tolerance otherwise."""
    shape = list(SHAPES[name])
    shape[0] = 4
    shape = tuple(shape)
    d = mu.desc(*shape, math)
    for kind in ("int", "normal"):
        x, w, dy = _inputs(shape, kind, seed=11)
        xs, dys = stored(x, math), stored(dy, math)
        ref = oracle_ref(shape, mu.BWD_FILTER, xs, None, dys)
        first = mu.WINOGRAD if _eligible(shape, mu.BWD_FILTER, mu.WINOGRAD) else mu.IMPLICIT_GEMM
        plan = [(first, 2), (mu.IM2COL_GEMM, 1), (mu.IMPLICIT_GEMM, 1)]
        got, _ = run_gpu(d, mu.BWD_FILTER, plan, x, w, dy)
        if kind == "int":
            assert np.array_equal(got, ref)
        else:
            assert normwise_err(got, ref) <= TOL[math]


@pytest.mark.parametrize("math", [mu.MATH_F32, mu.MATH_BF16], ids=["f32", "bf16"])
@pytest.mark.parametrize("conv_type", [mu.FWD, mu.BWD_DATA, mu.BWD_FILTER], ids=["fwd", "dgrad", "wgrad"])
def test_alpha_beta_and_mixed_plan(conv_type, math):
    """out = alpha*op + beta*out (reading G5) with a plan mixing all
    eligible algorithms."""
    shape = (4, 32, 9, 9, 48, 3, 3, 1, 1)
    d = mu.desc(*shape, math)
    x, w, dy = _inputs(shape, "int", seed=13)
    algos = [mu.WINOGRAD, mu.IM2COL_GEMM, mu.IMPLICIT_GEMM]
    plan = [(algos[0], 2), (algos[1], 1), (algos[2], 1)]
    n, c, h, wd, k, r, s, pad, st = shape
    p, q = mu.output_dims(d)
    out_shape = {mu.FWD: (n, p, q, k), mu.BWD_DATA: (n, h, wd, c), mu.BWD_FILTER: (k, r, s, c)}[conv_type]
    out0 = np.random.default_rng(1).integers(-2, 3, size=out_shape).astype(np.float32)
    ref = oracle_ref(shape, conv_type, x, w, dy, alpha=2.0, beta=-1.0, out0=out0)
    if math == mu.MATH_BF16 and conv_type != mu.BWD_FILTER:
        ref = torch.from_numpy(ref).to(torch.bfloat16).double().numpy()
    got, _ = run_gpu(d, conv_type, plan, x, w, dy, alpha=2.0, beta=-1.0, out0=out0)
    assert np.array_equal(got, ref)


@pytest.mark.parametrize("math", [mu.MATH_F32, mu.MATH_BF16], ids=["f32", "bf16"])
@pytest.mark.parametrize("case", [c for c in CASES if c[0] in ("3x3s1", "11x11s4_c3", "3x3s2")], ids=_ids)
def test_workspace_canary(case, math):
    """I6: no kernel writes outside the declared workspace."""
    name, conv_type, algo = case
    shape = SHAPES[name]
    d = mu.desc(*shape, math)
    x, w, dy = _inputs(shape, "normal")
    _, intact = run_gpu(d, conv_type, [(algo, shape[0] - 1), (algo, 1)], x, w, dy, canary=True)
    assert intact


def test_errors_before_launch():
    import paper_conf_cluster_oyamabhm18_b200.torch_api as T
    from gpu_util import handle
    shape = (2, 16, 8, 8, 16, 3, 3, 1, 1)
    d = mu.desc(*shape, mu.MATH_F32)
    x = torch.zeros(2, 8, 8, 16, device="cuda")
    w = torch.zeros(16, 3, 3, 16, device="cuda")
    with pytest.raises(mu.MucuError) as e:  # parts do not sum to N
        T.conv_forward(handle(), d, [(0, 1)], x, w)
    assert e.value.status == 1
    with pytest.raises(mu.MucuError) as e:  # I2C needs workspace
        T.conv_forward(handle(), d, [(1, 2)], x, w)
    assert e.value.status == 3
    d5 = mu.desc(2, 16, 8, 8, 16, 5, 5, 2, 1, mu.MATH_F32)
    w5 = torch.zeros(16, 5, 5, 16, device="cuda")
    ws = torch.zeros(1 << 20, dtype=torch.uint8, device="cuda")
    with pytest.raises(mu.MucuError) as e:  # Winograd on 5x5
        T.conv_forward(handle(), d5, [(2, 2)], x, w5, workspace=ws)
    assert e.value.status == 2


@pytest.mark.parametrize("math", [mu.MATH_F32, mu.MATH_BF16], ids=["f32", "bf16"])
def test_benchmark_dp_execute_end_to_end(math):
    """WR steps 1-3 on the GPU: benchmark every (algo, b), DP, then
    execute the plan -- the result matches the oracle."""
    import paper_conf_cluster_oyamabhm18_b200.torch_api as T
    from gpu_util import handle
    shape = (8, 64, 13, 13, 64, 3, 3, 1, 1)
    d = mu.desc(*shape, math)
    h = handle()
    h.set_policy(mu.POLICY_ALL)
    limit = 2 << 20
    for conv_type in (mu.FWD, mu.BWD_DATA, mu.BWD_FILTER):
        t, wsz = T.benchmark(h, d, conv_type, limit)
        assert (t[mu.IMPLICIT_GEMM, 1:] > 0).all()        # IG always fits (zero workspace)
        assert (wsz[t >= 0] <= limit).all()
        total, plan = mu.plan_wr(8, t, wsz, limit)
        assert sum(b for _, b in plan) == 8
        x, w, dy = _inputs(shape, "int", seed=17)
        ref = oracle_ref(shape, conv_type, x, w, dy)
        if math == mu.MATH_BF16 and conv_type != mu.BWD_FILTER:
            ref = torch.from_numpy(ref).to(torch.bfloat16).double().numpy()
        got, _ = run_gpu(d, conv_type, plan, x, w, dy)
        assert np.array_equal(got, ref)
    h.set_policy(mu.POLICY_POW2)


def test_cp_async_gather_producers_still_exact():
    """The cp.async gather producers (used when TMA im2col does not apply) are
    re-run on the vector-path shapes with TMA im2col disabled."""
    import os
    import subprocess
    import sys
    env = dict(os.environ, MUCU_TMA_IM2COL="0")
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", os.path.abspath(__file__), "-k",
                        "(c64 or c128) and not cp_async"], env=env, capture_output=True, text=True)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]


@pytest.mark.parametrize("math", [mu.MATH_F32, mu.MATH_TF32, mu.MATH_BF16], ids=["f32", "tf32", "bf16"])
@pytest.mark.parametrize("name", ["11x11s4_c3", "7x7s2_c3", "5x5s2_c2_k32", "4x4s3_c3_p0", "11x11s4_c3_ragged"])
def test_small_c_dgrad_alpha_beta_exact(name, math):
    """Zero-workspace BackwardData of C <= 4 layers (phase sub-filters, FFMA):
    integer data exact, alpha / beta, micro-batched plan."""
    shape = SHAPES[name]
    d = mu.desc(*shape, math)
    x, w, dy = _inputs(shape, "int", seed=19)
    n, c, h, wd, k, r, s, pad, st = shape
    out0 = np.random.default_rng(3).integers(-2, 3, size=(n, h, wd, c)).astype(np.float32)
    ref = oracle_ref(shape, mu.BWD_DATA, x, w, dy, alpha=2.0, beta=-1.0, out0=out0)
    if math == mu.MATH_BF16:
        ref = torch.from_numpy(ref).to(torch.bfloat16).double().numpy()
    got, _ = run_gpu(d, mu.BWD_DATA, [(mu.IMPLICIT_GEMM, n - 1), (mu.IMPLICIT_GEMM, 1)], x, w, dy, alpha=2.0,
                     beta=-1.0, out0=out0)
    assert np.array_equal(got, ref)
