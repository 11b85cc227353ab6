"""GPU parity of the alternative tilings the default heuristics pick only at
full size (or not at all), forced on the small parity shapes:

* MUCU_FORCE_MT=4 / 2: 512- / 256-row tiles (four / two interleaved TMEM
  accumulators; chosen by default for narrow N when there is at least one
  such tile per SM -- never at parity-test sizes);
* MUCU_HALO=1: the halo producer for stride-1 FWD / DGRAD (opt-in).

Integer-valued inputs make every tensor-core path exact (sums < 2^24), so the
check is bit-exact against the fp64 oracle (BF16 outputs: RNE of the oracle).
"""
import numpy as np
import pytest
import torch

import paper_conf_cluster_oyamabhm18_b200 as mu
from synthetic import conv_inputs

pytestmark = pytest.mark.gpu

from gpu_util import oracle_ref, run_gpu  # noqa: E402

SHAPES = {
    "3x3s1_c64": (2, 64, 12, 12, 64, 3, 3, 1, 1),
    "3x3s1_c128": (2, 128, 10, 10, 192, 3, 3, 1, 1),
    "5x5s1": (2, 64, 11, 11, 48, 5, 5, 2, 1),
    "3x3s1_p2": (2, 32, 7, 7, 32, 3, 3, 2, 1),
    "3x3s2_c64": (2, 64, 15, 15, 128, 3, 3, 1, 2),
    "3x3s2_even": (2, 64, 14, 14, 64, 3, 3, 1, 2),      # strided DGRAD: the 4 phases in one launch
    "1x1s2_c128": (2, 128, 14, 12, 64, 1, 1, 0, 2),     # strided DGRAD: 3 tapless phases zeroed
    "1x1s1": (3, 64, 10, 10, 96, 1, 1, 0, 1),
    "7x7s2_c3": (2, 3, 23, 23, 64, 7, 7, 3, 2),
    "big_k": (1, 128, 6, 6, 256, 3, 3, 1, 1),
}
# per_atom_boxes: the one-box-per-atom TMA loads the multi-dimensional boxes replaced (§6.1)
NO_BOXES = {"MUCU_B_BOX": "0", "MUCU_A_BOX": "0", "MUCU_WIN_BOX": "0", "MUCU_A_MERGE": "0"}
ENVS = {"mt4": {"MUCU_FORCE_MT": "4"}, "mt2": {"MUCU_FORCE_MT": "2"}, "halo": {"MUCU_HALO": "1"},
        "per_phase": {"MUCU_MERGE_PHASES": "0"}, "per_atom_boxes": NO_BOXES}
CASES = [(s, t, a) for s in SHAPES for t in (mu.FWD, mu.BWD_DATA)
         for a in (mu.IMPLICIT_GEMM, mu.IM2COL_GEMM)]


@pytest.mark.parametrize("env", list(ENVS))
@pytest.mark.parametrize("math", [mu.MATH_TF32, mu.MATH_BF16], ids=["tf32", "bf16"])
@pytest.mark.parametrize("case", CASES, ids=lambda c: f"{c[0]}-{mu.TYPE_NAMES[c[1]]}-{mu.ALGO_NAMES[c[2]]}")
def test_forced_tiling_exact(case, math, env, monkeypatch):
    for k, v in ENVS[env].items():
        monkeypatch.setenv(k, v)
    name, conv_type, algo = case
    shape = SHAPES[name]
    d = mu.desc(*shape, math)
    x, w, dy = conv_inputs(*shape, seed=21, kind="int")
    ref = oracle_ref(shape, conv_type, x, w, dy)
    if math == mu.MATH_BF16:
        ref = torch.from_numpy(ref).to(torch.bfloat16).double().numpy()
    got, _ = run_gpu(d, conv_type, [(algo, shape[0])], x, w, dy)
    assert np.array_equal(got, ref)


# BackwardFilter through the per-atom TMA loads and multi-k-block stages
@pytest.mark.parametrize("env", ["per_atom_boxes", "km2"])
@pytest.mark.parametrize("math", [mu.MATH_TF32, mu.MATH_BF16], ids=["tf32", "bf16"])
@pytest.mark.parametrize("name", ["3x3s1_c64", "3x3s1_c128", "1x1s1", "1x1s2_c128", "7x7s2_c3", "big_k"])
def test_wgrad_alternative_loads_exact(name, math, env, monkeypatch):
    envs = NO_BOXES if env == "per_atom_boxes" else {"MUCU_DENSE_KM": "4", "MUCU_WIN_KM1": "0"}
    for k, v in envs.items():
        monkeypatch.setenv(k, v)
    shape = SHAPES[name]
    d = mu.desc(*shape, math)
    x, w, dy = conv_inputs(*shape, seed=29, kind="int")
    ref = oracle_ref(shape, mu.BWD_FILTER, x, w, dy)
    for algo in (mu.IMPLICIT_GEMM, mu.IM2COL_GEMM):
        got, _ = run_gpu(d, mu.BWD_FILTER, [(algo, shape[0])], x, w, dy)
        assert np.array_equal(got, ref), (name, algo)


# Cluster split-K BackwardFilter (DSMEM reduction, ordered split groups): every
# cluster size and a multi-group chain, forced on mid-size shapes with enough
# k-blocks; integer data -> exact, random data -> bitwise reproducible.
SPLITK_SHAPES = {
    "3x3_c64": (16, 64, 28, 28, 64, 3, 3, 1, 1),
    "3x3_k192": (8, 128, 14, 14, 192, 3, 3, 1, 1),
    "1x1_k512": (16, 256, 14, 14, 512, 1, 1, 0, 1),
    "11x11s4_c3": (8, 3, 99, 99, 64, 11, 11, 2, 4),
    "7x7s2_c3": (8, 3, 64, 64, 64, 7, 7, 3, 2),
}
SPLITK_ENVS = {"cl2": {"MUCU_FORCE_CL": "2"}, "cl4": {"MUCU_FORCE_CL": "4"}, "cl8": {"MUCU_FORCE_CL": "8"},
               "cl16": {"MUCU_FORCE_CL": "16"}, "cl2x3": {"MUCU_FORCE_CL": "2", "MUCU_FORCE_G": "3"},
               "cl4x2": {"MUCU_FORCE_CL": "4", "MUCU_FORCE_G": "2"}}


@pytest.mark.parametrize("env", list(SPLITK_ENVS))
@pytest.mark.parametrize("math", [mu.MATH_TF32, mu.MATH_BF16], ids=["tf32", "bf16"])
@pytest.mark.parametrize("name", list(SPLITK_SHAPES))
def test_cluster_splitk_wgrad_exact(name, math, env, monkeypatch):
    for k, v in SPLITK_ENVS[env].items():
        monkeypatch.setenv(k, v)
    shape = SPLITK_SHAPES[name]
    d = mu.desc(*shape, math)
    x, w, dy = conv_inputs(*shape, seed=31, kind="int", lo=-1, hi=1)
    algos = [mu.IMPLICIT_GEMM, mu.IM2COL_GEMM] + ([mu.WINOGRAD] if shape[5] == 3 and shape[8] == 1 else [])
    out0 = np.random.default_rng(5).integers(-2, 3, size=(shape[4], shape[5], shape[6], shape[1])).astype(np.float32)
    for algo in algos:
        ref = oracle_ref(shape, mu.BWD_FILTER, x, w, dy)
        got, _ = run_gpu(d, mu.BWD_FILTER, [(algo, shape[0])], x, w, dy)
        assert np.array_equal(got, ref), (name, algo)
        # beta applied exactly once (split group 0), alpha on every partial
        ref = oracle_ref(shape, mu.BWD_FILTER, x, w, dy, alpha=2.0, beta=-1.0, out0=out0)
        got, _ = run_gpu(d, mu.BWD_FILTER, [(algo, shape[0])], x, w, dy, alpha=2.0, beta=-1.0, out0=out0)
        assert np.array_equal(got, ref), (name, algo, "alpha/beta")
    xr, wr, dyr = conv_inputs(*shape, seed=32, kind="normal")
    for algo in algos:
        a1, _ = run_gpu(d, mu.BWD_FILTER, [(algo, shape[0])], xr, wr, dyr)
        a2, _ = run_gpu(d, mu.BWD_FILTER, [(algo, shape[0])], xr, wr, dyr)
        assert np.array_equal(a1, a2), (name, algo, "reproducible")


@pytest.mark.parametrize("math", [mu.MATH_TF32, mu.MATH_BF16], ids=["tf32", "bf16"])
@pytest.mark.parametrize("name", list(SPLITK_SHAPES))
def test_nondeterministic_wgrad_exact(name, math):
    """mucu_set_deterministic(0): split partials added with L2 atomics after a
    beta prescale -- exact on integer data (any order), alpha / beta applied once."""
    from gpu_util import handle
    h = handle()
    h.set_deterministic(False)
    try:
        shape = SPLITK_SHAPES[name]
        d = mu.desc(*shape, math)
        x, w, dy = conv_inputs(*shape, seed=33, kind="int", lo=-1, hi=1)
        out0 = np.random.default_rng(6).integers(-2, 3, size=(shape[4], shape[5], shape[6], shape[1])).astype(np.float32)
        algos = [mu.IMPLICIT_GEMM, mu.IM2COL_GEMM] + ([mu.WINOGRAD] if shape[5] == 3 and shape[8] == 1 else [])
        for algo in algos:
            ref = oracle_ref(shape, mu.BWD_FILTER, x, w, dy, alpha=2.0, beta=-1.0, out0=out0)
            got, _ = run_gpu(d, mu.BWD_FILTER, [(algo, shape[0])], x, w, dy, alpha=2.0, beta=-1.0, out0=out0)
            assert np.array_equal(got, ref), (name, algo)
    finally:
        h.set_deterministic(True)
