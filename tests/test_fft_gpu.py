"""GPU parity of the FFT and FFT_TILING algorithms (kernels_fft.cu)
against the fp64 oracle, through the C ABI.

The frequency-domain algorithms compute the same convolution with a
different rounding: an F x F DFT adds ~log2(F^2) roundings per value, so they are
never bit-exact (no integer-exact case, unlike the GEMM algorithms) but stay within
the F32 tolerance of the other F32 algorithms, max|d| / ||ref||_inf <= 1e-5.
I1 holds bitwise (each plane and each output is computed independently of b),
I2 within tolerance.  Shapes: stride 1 (the only eligible stride), single and
multiple tiles with ragged edges, pad 0 / same / larger than R - 1.
"""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_cluster_oyamabhm18_b200 as mu
from paper_conf_cluster_oyamabhm18_b200 import torch_api as T
from synthetic import conv_inputs, network

pytestmark = pytest.mark.gpu

from gpu_util import handle, normwise_err, oracle_ref, run_gpu  # noqa: E402

TOL = 1e-5

# n, c, h, w, k, r, s, pad, stride
SHAPES = {
    "5x5_alexnet_conv2": (2, 64, 27, 27, 48, 5, 5, 2, 1),   # FFT F = 32, FFT_TILING 1 tile
    "3x3_alexnet_conv3": (3, 32, 13, 13, 40, 3, 3, 1, 1),   # FFT F = 16
    "3x3_multi_tile": (2, 16, 40, 37, 24, 3, 3, 1, 1),      # FFT ineligible (F = 64); 2 x 2 tiles
    "5x5_p0_ragged": (2, 8, 36, 30, 16, 5, 5, 0, 1),        # tiles 28 x 26: 2 x 1, ragged
    "7x7_p3": (2, 4, 20, 20, 8, 7, 7, 3, 1),
    "3x3_p0": (2, 12, 12, 14, 20, 3, 3, 0, 1),              # DGRAD F needs H + R - 1
    "3x3_p2": (2, 32, 7, 7, 32, 3, 3, 2, 1),                # pad > R - 1
    "1x1": (3, 24, 10, 9, 40, 1, 1, 0, 1),
    "odd_channels": (2, 3, 11, 11, 5, 3, 3, 1, 1),
    "big_tiles": (1, 8, 70, 66, 8, 11, 11, 5, 1),            # FFT_TILING 22 x 22 tiles: 4 x 3
}


def _eligible(shape, conv_type, algo):
    n, c, h, w, k, r, s, pad, st = shape
    if st != 1:
        return False
    p, q = h + 2 * pad - r + 1, w + 2 * pad - s + 1
    eh, ew = (h, w) if conv_type == mu.BWD_DATA else (p, q)
    if algo == mu.FFT:
        f = 8
        while f < max(eh + r - 1, ew + s - 1):
            f *= 2
        return f <= 32
    return r <= 16 and s <= 16


CASES = [(name, t, a) for name in SHAPES for t in (mu.FWD, mu.BWD_DATA, mu.BWD_FILTER)
         for a in (mu.FFT, mu.FFT_TILING) if _eligible(SHAPES[name], t, a)]


def _ids(c):
    return f"{c[0]}-{mu.TYPE_NAMES[c[1]]}-{mu.ALGO_NAMES[c[2]]}"


def _inputs(shape, kind="normal", seed=3):
    return conv_inputs(*shape, seed=seed, kind=kind)


@pytest.mark.parametrize("case", CASES, ids=_ids)
def test_fft_parity_random(case):
    name, conv_type, algo = case
    shape = SHAPES[name]
    d = mu.desc(*shape, mu.MATH_F32)
    x, w, dy = _inputs(shape)
    ref = oracle_ref(shape, conv_type, x, w, dy)
    got, _ = run_gpu(d, conv_type, [(algo, shape[0])], x, w, dy)
    assert got.shape == ref.shape
    assert normwise_err(got, ref) <= TOL


@pytest.mark.parametrize("case", CASES, ids=_ids)
def test_fft_parity_integer_inputs(case):
    """Integer-valued data: not bit-exact in the frequency domain, within tolerance."""
    name, conv_type, algo = case
    shape = SHAPES[name]
    d = mu.desc(*shape, mu.MATH_F32)
    x, w, dy = _inputs(shape, "int", seed=5)
    ref = oracle_ref(shape, conv_type, x, w, dy)
    got, _ = run_gpu(d, conv_type, [(algo, shape[0])], x, w, dy)
    assert normwise_err(got, ref) <= TOL


@pytest.mark.parametrize("case", [c for c in CASES if c[1] != mu.BWD_FILTER], ids=_ids)
def test_fft_micro_batch_bit_identity(case):
    """I1: micro-batched FWD / DGRAD bitwise equal to the same algorithm at full N."""
    name, conv_type, algo = case
    shape = list(SHAPES[name])
    shape[0] = 5
    shape = tuple(shape)
    d = mu.desc(*shape, mu.MATH_F32)
    x, w, dy = _inputs(shape, seed=9)
    full, _ = run_gpu(d, conv_type, [(algo, 5)], x, w, dy)
    split, _ = run_gpu(d, conv_type, [(algo, 3), (algo, 1), (algo, 1)], x, w, dy)
    assert np.array_equal(full, split)


@pytest.mark.parametrize("name", ["5x5_alexnet_conv2", "3x3_multi_tile", "3x3_alexnet_conv3"])
def test_fft_wgrad_accumulates_over_micro_batches(name):
    """I2: dW summed over micro-batches of mixed algorithms = full-batch dW."""
    shape = list(SHAPES[name])
    shape[0] = 4
    shape = tuple(shape)
    d = mu.desc(*shape, mu.MATH_F32)
    x, w, dy = _inputs(shape, seed=11)
    ref = oracle_ref(shape, mu.BWD_FILTER, x, None, dy)
    first = mu.FFT if _eligible(shape, mu.BWD_FILTER, mu.FFT) else mu.FFT_TILING
    plan = [(first, 2), (mu.FFT_TILING, 1), (mu.IMPLICIT_GEMM, 1)]
    got, _ = run_gpu(d, mu.BWD_FILTER, plan, x, w, dy)
    assert normwise_err(got, ref) <= TOL


@pytest.mark.parametrize("name", ["5x5_alexnet_conv2", "3x3_multi_tile"])
def test_fft_wgrad_spectrum_runs(name):
    """Consecutive FFT / FFT_TILING BackwardFilter micro-batches accumulate dW in the
    frequency domain and transform it back once per run: runs of
    different lengths and micro-batch sizes, broken by other algorithms, with
    alpha / beta (the run's first micro-batch carries the user's beta)."""
    shape = list(SHAPES[name])
    shape[0] = 6
    shape = tuple(shape)
    d = mu.desc(*shape, mu.MATH_F32)
    x, w, dy = _inputs(shape, seed=13)
    algo = mu.FFT if _eligible(shape, mu.BWD_FILTER, mu.FFT) else mu.FFT_TILING
    out0 = np.random.default_rng(5).standard_normal(oracle_ref(shape, mu.BWD_FILTER, x, None, dy).shape)
    ref = oracle_ref(shape, mu.BWD_FILTER, x, None, dy, alpha=1.5, beta=-0.5, out0=out0)
    for plan in ([(algo, 3), (algo, 2), (algo, 1)],
                 [(algo, 2), (mu.IMPLICIT_GEMM, 1), (algo, 1), (algo, 2)],
                 [(mu.IMPLICIT_GEMM, 1), (algo, 4), (mu.FFT_TILING, 1)],
                 [(algo, 1)] * 6):
        got, _ = run_gpu(d, mu.BWD_FILTER, plan, x, w, dy, alpha=1.5, beta=-0.5, out0=out0.astype(np.float32))
        assert normwise_err(got, ref) <= TOL, plan


@pytest.mark.parametrize("conv_type", [mu.FWD, mu.BWD_DATA, mu.BWD_FILTER], ids=["fwd", "dgrad", "wgrad"])
def test_fft_alpha_beta_mixed_plan(conv_type):
    """out = alpha*op + beta*out with FFT, FFT_TILING, Winograd and IG micro-batches."""
    shape = (4, 32, 9, 9, 48, 3, 3, 1, 1)
    d = mu.desc(*shape, mu.MATH_F32)
    x, w, dy = _inputs(shape, seed=13)
    plan = [(mu.FFT, 1), (mu.WINOGRAD, 1), (mu.FFT_TILING, 1), (mu.IMPLICIT_GEMM, 1)]
    n, c, h, wd, k, r, s, pad, st = shape
    p, q = mu.output_dims(d)
    out_shape = {mu.FWD: (n, p, q, k), mu.BWD_DATA: (n, h, wd, c), mu.BWD_FILTER: (k, r, s, c)}[conv_type]
    out0 = np.random.default_rng(1).standard_normal(out_shape).astype(np.float32)
    ref = oracle_ref(shape, conv_type, x, w, dy, alpha=2.0, beta=-1.0, out0=out0)
    got, _ = run_gpu(d, conv_type, plan, x, w, dy, alpha=2.0, beta=-1.0, out0=out0)
    assert normwise_err(got, ref) <= TOL


@pytest.mark.parametrize("case", [c for c in CASES if c[0] in ("3x3_multi_tile", "5x5_alexnet_conv2")], ids=_ids)
def test_fft_workspace_canary(case):
    """I6: no FFT kernel writes outside the declared workspace."""
    name, conv_type, algo = case
    shape = SHAPES[name]
    d = mu.desc(*shape, mu.MATH_F32)
    x, w, dy = _inputs(shape)
    _, intact = run_gpu(d, conv_type, [(algo, shape[0] - 1), (algo, 1)], x, w, dy, canary=True)
    assert intact


def test_fft_ineligible_configurations():
    """UNSUPPORTED before any launch: tensor-core maths, stride > 1, FFT above F = 32."""
    x = torch.zeros(2, 8, 8, 16, device="cuda")
    w = torch.zeros(16, 3, 3, 16, device="cuda")
    ws = torch.zeros(1 << 24, dtype=torch.uint8, device="cuda")
    for math in (mu.MATH_TF32, mu.MATH_BF16):
        d = mu.desc(2, 16, 8, 8, 16, 3, 3, 1, 1, math)
        xx, ww = (x, w) if math == mu.MATH_TF32 else (x.bfloat16(), w.bfloat16())
        for algo in (mu.FFT, mu.FFT_TILING):
            with pytest.raises(mu.MucuError) as e:
                T.conv_forward(handle(), d, [(algo, 2)], xx, ww, workspace=ws)
            assert e.value.status == 2
    d = mu.desc(2, 16, 8, 8, 16, 3, 3, 1, 2, mu.MATH_F32)
    with pytest.raises(mu.MucuError) as e:
        T.conv_forward(handle(), d, [(mu.FFT, 2)], x, w, workspace=ws)
    assert e.value.status == 2
    d = mu.desc(1, 16, 40, 40, 16, 3, 3, 1, 1, mu.MATH_F32)
    with pytest.raises(mu.MucuError):
        mu.workspace_size(d, mu.FWD, mu.FFT, 1)
    assert mu.workspace_size(d, mu.FWD, mu.FFT_TILING, 1) > 0


@pytest.mark.parametrize("algo", [mu.FFT, mu.FFT_TILING], ids=["FFT", "FFTT"])
def test_fft_alexnet_full_size_sampled(algo):
    """AlexNet conv2-5 at N = 256, F32, micro-batches of 32 (the paper's FFT at b = 32),
    FWD / DGRAD / WGRAD checked on oracle-computed samples (tolerance relative to the
    oracle's sampled magnitudes)."""
    rng = np.random.default_rng(0)
    n = 256
    for layer in [l for l in network("alexnet") if l.stride == 1]:
        shape = (n, layer.c, layer.h, layer.w, layer.k, layer.r, layer.s, layer.pad, 1)
        d = mu.desc(*shape, mu.MATH_F32)
        x, w, dy = conv_inputs(*shape, seed=7)
        plan = [(algo, 32)] * 8
        for conv_type, fn in ((mu.FWD, "fwd"), (mu.BWD_DATA, "dgrad"), (mu.BWD_FILTER, "wgrad")):
            got, _ = run_gpu(d, conv_type, plan, x, w, dy)
            assert np.isfinite(got).all()
            idxs = [tuple(int(rng.integers(0, s)) for s in got.shape) for _ in range(16)]
            refs = []
            for idx in idxs:
                if fn == "fwd":
                    refs.append(oracle.forward_at(x, w, layer.pad, 1, idx))
                elif fn == "dgrad":
                    refs.append(oracle.backward_data_at(dy, w, layer.h, layer.w, layer.pad, 1, idx))
                else:
                    refs.append(oracle.backward_filter_at(x, dy, layer.r, layer.s, layer.pad, 1, idx))
            scale = max(abs(r) for r in refs)
            for idx, ref in zip(idxs, refs):
                assert abs(float(got[idx]) - ref) <= TOL * scale, (layer.name, fn, idx, float(got[idx]), ref)
