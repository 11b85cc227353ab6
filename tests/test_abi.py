"""The C-ABI library loads on a CPU-only host and exports every function
include/mucudnn.h declares; host-only entry points behave as documented.
No compute (GPU) calls here."""
import ctypes
import os
import re

import pytest

import paper_conf_cluster_oyamabhm18_b200 as mu
from paper_conf_cluster_oyamabhm18_b200 import _lib

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "mucudnn.h")


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(mucu_[a-z_0-9]+)\s*\(", src)))


def test_header_declares_the_boundary():
    fns = declared_functions()
    for name in ["mucu_create", "mucu_benchmark", "mucu_plan_wr", "mucu_pareto_front", "mucu_solve_wd",
                 "mucu_conv_forward", "mucu_conv_backward_data", "mucu_conv_backward_filter",
                 "mucu_network_plan", "mucu_workspace_size"]:
        assert name in fns


def test_library_exports_every_declared_symbol():
    lib = ctypes.CDLL(_lib._LIB_PATH)
    missing = [f for f in declared_functions() if not hasattr(lib, f)]
    assert not missing, missing


def test_status_strings_and_version():
    assert mu.version() == 100
    for i, name in enumerate(_lib.STATUS):
        assert _lib.status_string(i) == name


def test_output_dims_and_invalid_descriptor():
    assert mu.output_dims(mu.desc(8, 64, 27, 27, 192, 5, 5, 2, 1)) == (27, 27)
    assert mu.output_dims(mu.desc(1, 3, 224, 224, 64, 11, 11, 2, 4)) == (55, 55)
    assert mu.output_dims(mu.desc(1, 3, 224, 224, 64, 7, 7, 3, 2)) == (112, 112)
    with pytest.raises(mu.MucuError) as e:
        mu.output_dims(mu.desc(1, 3, 2, 2, 4, 5, 5, 0, 1))
    assert e.value.status == 1


# Closed-form workspace sizes (header comment of mucu_workspace_size).
def test_workspace_im2col_alexnet_conv2_cfg1():
    d = mu.desc(8, 64, 27, 27, 192, 5, 5, 2, 1, mu.MATH_F32)
    assert mu.workspace_size(d, mu.FWD, mu.IMPLICIT_GEMM, 8) == 0
    assert mu.workspace_size(d, mu.FWD, mu.IM2COL_GEMM, 1) == 4_665_600   # 729 * 1600 * 4
    assert mu.workspace_size(d, mu.FWD, mu.IM2COL_GEMM, 2) == 9_331_200   # > 8 MiB: b = 1 only
    with pytest.raises(mu.MucuError) as e:
        mu.workspace_size(d, mu.FWD, mu.WINOGRAD, 1)                       # 5x5: ineligible
    assert e.value.status == 2


def test_workspace_winograd_alexnet_conv3():
    d = mu.desc(256, 192, 13, 13, 384, 3, 3, 1, 1, mu.MATH_F32)
    U = 16 * 384 * 192 * 4
    per_sample = 16 * 49 * 192 * 4 + 16 * 49 * 384 * 4                    # V + M = 1,806,336
    assert per_sample == 1_806_336
    assert mu.workspace_size(d, mu.FWD, mu.WINOGRAD, 1) == U + per_sample
    assert mu.workspace_size(d, mu.FWD, mu.WINOGRAD, 10) == U + 10 * per_sample
    # WGRAD F(3x3,2x2): V + D at Tp = align256(b*T) tile rows, M fp32 (header closed form)
    for b in (1, 10):
        Tp = -(-b * 49 // 256) * 256
        assert mu.workspace_size(d, mu.BWD_FILTER, mu.WINOGRAD, b) == 16 * Tp * (192 + 384) * 4 + 16 * 384 * 192 * 4
    d5 = mu.desc(2, 40, 9, 9, 24, 3, 3, 1, 1, mu.MATH_BF16)                 # pitches 64 / 64 (128 B)
    assert mu.workspace_size(d5, mu.BWD_FILTER, mu.WINOGRAD, 2) == 16 * 256 * (64 + 64) * 2 + 16 * 64 * 64 * 4


def test_workspace_bf16_resnet_and_pointwise():
    d = mu.desc(256, 64, 56, 56, 64, 3, 3, 1, 1, mu.MATH_BF16)
    assert mu.workspace_size(d, mu.FWD, mu.IM2COL_GEMM, 1) == 3_612_672   # 3136 * 576 * 2
    # WG bf16: V bf16 + M fp32 per sample = 4,816,896 (SURVEY ResNet-18 layer1 row)
    U = 16 * 64 * 64 * 2
    assert mu.workspace_size(d, mu.FWD, mu.WINOGRAD, 1) - U == 4_816_896
    p = mu.desc(256, 256, 56, 56, 64, 1, 1, 0, 1, mu.MATH_BF16)
    for t in (mu.FWD, mu.BWD_DATA):
        assert mu.workspace_size(p, t, mu.IM2COL_GEMM, 256) == 0          # im2col(x) == x
    # BackwardFilter: no im2col, but ceil(148 / (1 x 2 dW tiles)) = 74 partial dW slots of
    # K x R*S*C fp32 (deterministic split-K over all SMs)
    assert mu.workspace_size(p, mu.BWD_FILTER, mu.IM2COL_GEMM, 256) == 74 * 64 * 256 * 4
    pf = mu.desc(256, 256, 56, 56, 64, 1, 1, 0, 1, mu.MATH_F32)
    assert mu.workspace_size(pf, mu.BWD_FILTER, mu.IM2COL_GEMM, 256) == 0  # F32 SIMT: ordered chain
    ds = mu.desc(256, 256, 56, 56, 512, 1, 1, 0, 2, mu.MATH_BF16)
    assert mu.workspace_size(ds, mu.FWD, mu.IM2COL_GEMM, 1) == 401_408    # 784 * 256 * 2


def test_workspace_unaligned_filter_row():
    d = mu.desc(4, 3, 224, 224, 64, 7, 7, 3, 2, mu.MATH_F32)               # RSC = 147
    kp = 148                                                               # ceil to 4 floats
    col = 112 * 112 * kp * 4
    filt = -(-64 * kp * 4 // 256) * 256
    assert mu.workspace_size(d, mu.FWD, mu.IM2COL_GEMM, 1) == filt + -(-col // 256) * 256


def test_workspace_small_c_tensor_core():
    # C*elt < 16 B on tensor cores, stride 1: I2C FWD/WGRAD keep x with channels padded to 16 B
    d = mu.desc(4, 3, 224, 224, 64, 7, 7, 3, 1, mu.MATH_BF16)
    assert mu.workspace_size(d, mu.FWD, mu.IM2COL_GEMM, 2) == 2 * 224 * 224 * 16
    # WGRAD: 147 taps would pad to 256 staged rows (> 1/4 padding): the channel-padded x as FWD
    assert mu.workspace_size(d, mu.BWD_FILTER, mu.IM2COL_GEMM, 1) == 224 * 224 * 16
    assert mu.workspace_size(d, mu.BWD_FILTER, mu.IM2COL_GEMM, 4) == 4 * 224 * 224 * 16


def test_workspace_space_to_depth():
    # AlexNet conv1 on tensor cores (TF32, stride 4).  FWD: 2 x 2 output super-pixels over
    # 8 x 8 input ones (u = 2, f = 8): Dr = (4*1 + 11 - 1) // 8 + 1 = 2, Cs = 8*8*3 = 192 (a
    # multiple of the TF32 atom 32), Pu = 28, 29 x 29 input super-pixels, filter 4K x 4 x 192.
    d = mu.desc(4, 3, 224, 224, 64, 11, 11, 2, 4, mu.MATH_TF32)
    a256 = lambda v: -(-v // 256) * 256  # noqa: E731
    xs = 29 * 29 * 192 * 4
    assert mu.workspace_size(d, mu.FWD, mu.IM2COL_GEMM, 2) == a256(4 * 64 * 4 * 192 * 4) + a256(2 * xs)
    # WGRAD: staged-row kernel, 148 partial dW tiles of 384 (363 taps) x 64 fp32
    assert mu.workspace_size(d, mu.BWD_FILTER, mu.IM2COL_GEMM, 3) == a256(148 * 384 * 64 * 4)
    # DGRAD: dx super-pixels of f = 8 (u = 2; 8*8*3 = 192 <= 256 columns), Dr = 10 // 4 + 2 = 4
    assert mu.workspace_size(d, mu.BWD_DATA, mu.IM2COL_GEMM, 4) == a256(192 * 16 * 64 * 4)
    # ResNet conv1 BF16 (stride 2): FWD u = 2, f = 4: Dr = (2*1 + 7 - 1) // 4 + 1 = 3, Cs = 48 -> 64,
    # 56 x 56 output super-pixels, 58 x 58 input super-pixels, filter 4K x 9 x 64.
    d = mu.desc(2, 3, 224, 224, 64, 7, 7, 3, 2, mu.MATH_BF16)
    assert mu.workspace_size(d, mu.FWD, mu.IM2COL_GEMM, 2) == a256(4 * 64 * 9 * 64 * 2) + a256(2 * 58 * 58 * 64 * 2)
    # WGRAD: 147 taps -> 256 staged rows is > 1/4 padding: window form (64-B atoms, tpa = 8,
    # na = 1), Wp = max(2*(Q-1) + 8, W + 3) rounded up to 4 = 232
    # + 148 deterministic split-K partial tiles of M = 7 rows x 32 (one 64-B atom) x K fp32
    assert mu.workspace_size(d, mu.BWD_FILTER, mu.IM2COL_GEMM, 2) == a256(2 * 224 * 232 * 4 * 2) + \
        a256(148 * 224 * 64 * 4)
    # window form when the x row (W*C*elt) is not a multiple of 16 B: 64-B atoms (one 8-tap atom
    # per filter row), tpa = 8, na = 1, Wp = max(2*(Q-1) + 8, W + 3) rounded up to 4
    d = mu.desc(2, 3, 223, 223, 64, 7, 7, 3, 2, mu.MATH_BF16)  # W*C = 669: no chunking
    q = (223 + 6 - 7) // 2 + 1
    wp = -(-max(2 * (q - 1) + 8, 223 + 3) // 4) * 4
    assert mu.workspace_size(d, mu.BWD_FILTER, mu.IM2COL_GEMM, 2) == a256(2 * 223 * wp * 4 * 2) + \
        a256(148 * 224 * 64 * 4)
    # DGRAD: f = 4 (4*4*3 = 48 columns), Dr = 6 // 2 + 2 = 5: filter 48 x 25*64
    assert mu.workspace_size(d, mu.BWD_DATA, mu.IM2COL_GEMM, 2) == a256(48 * 25 * 64 * 2)
    # stride 3, BF16: 3*8 B is not a multiple of 16 -> WGRAD keeps the space-to-depth image
    # (u = 1, f = 3, Dr = ceil(4/3) = 2, Cs = 27 -> 64, (P + 1) x (Q + 1) super-pixels)
    d = mu.desc(1, 3, 20, 22, 64, 4, 4, 0, 3, mu.MATH_BF16)
    assert mu.workspace_size(d, mu.BWD_FILTER, mu.IM2COL_GEMM, 1) == a256(1 * 7 * 8 * 64 * 2)
    # stride 1 keeps the channel-padded image (16 B per pixel)
    d = mu.desc(2, 3, 32, 32, 64, 3, 3, 1, 1, mu.MATH_BF16)
    assert mu.workspace_size(d, mu.FWD, mu.IM2COL_GEMM, 2) == 2 * 32 * 32 * 16


def test_workspace_i2c_wgrad_slots():
    """I2C BackwardFilter of atom-aligned layers: im2col by TMA in shared memory, the
    workspace is only the partial dW slots (include/mucudnn.h closed form)."""
    d = mu.desc(256, 64, 27, 27, 192, 5, 5, 2, 1, mu.MATH_TF32)       # AlexNet conv2
    ps = -(-148 // (1 * -(-1600 // 256)))                              # 148 / (1 * 7) -> 22
    for b in (1, 64, 256):                                             # b-independent
        assert mu.workspace_size(d, mu.BWD_FILTER, mu.IM2COL_GEMM, b) == ps * 192 * 1600 * 4
    d = mu.desc(256, 512, 7, 7, 512, 3, 3, 1, 1, mu.MATH_BF16)        # ResNet layer4 3x3
    ps = -(-148 // (2 * 18))                                           # -> 5
    assert mu.workspace_size(d, mu.BWD_FILTER, mu.IM2COL_GEMM, 32) == ps * 512 * 4608 * 4
    # F32 keeps the explicit im2col matrix (SIMT path), no slots
    d = mu.desc(8, 64, 27, 27, 192, 5, 5, 2, 1, mu.MATH_F32)
    assert mu.workspace_size(d, mu.BWD_FILTER, mu.IM2COL_GEMM, 1) == 729 * 1600 * 4


# NEXT-3 entry points: argument validation happens on the host before any device work.
def _reduce_call(target):
    d = mu.desc(2, 8, 6, 6, 8, 3, 3, 1, 1, mu.MATH_F32)
    plan = (_lib.MicroConfig * 1)(_lib.MicroConfig(mu.IMPLICIT_GEMM, 2))
    return _lib.lib.mucu_conv_backward_filter_reduce(None, ctypes.byref(d), plan, 1, 1.0, ctypes.c_void_p(256),
                                                     ctypes.c_void_p(512), 0.0, ctypes.c_void_p(1024),
                                                     ctypes.byref(target) if target is not None else None,
                                                     None, 0, None)


def test_reduce_target_validation():
    ok_ptrs = [4096, 8192]
    assert _reduce_call(None) == 1                                        # no target
    assert _reduce_call(_lib.reduce_target([])) == 1                      # count 0
    assert _reduce_call(_lib.reduce_target([4096] * 8)) == 1              # valid target, NULL handle
    t = _lib.reduce_target([4096] * 8)
    t.count = 9
    assert _reduce_call(t) == 1                                           # count > MUCU_MAX_REDUCE_RANKS
    assert _reduce_call(_lib.reduce_target(ok_ptrs, multicast=True)) == 1  # multicast needs count 1
    assert _reduce_call(_lib.reduce_target([4096 + 4])) == 6              # MISALIGNED
    assert _reduce_call(_lib.reduce_target([0])) == 6                     # NULL destination


def test_peer_barrier_validation_and_multicast_probe():
    bad = _lib.reduce_target([])
    assert _lib.lib.mucu_peer_barrier(ctypes.byref(bad), ctypes.c_void_p(4096), 1, None) == 1
    assert _lib.lib.mucu_peer_barrier(ctypes.byref(_lib.reduce_target([4096, 8192], multicast=True)),
                                      ctypes.c_void_p(4096), 1, None) == 1
    assert _lib.lib.mucu_peer_barrier(ctypes.byref(_lib.reduce_target([4098])), ctypes.c_void_p(4096), 1,
                                      None) == 6
    # host query: no CUDA device here -> "not supported", not an error
    assert _lib.nvls_supported(0) is False
    h = ctypes.c_void_p()
    assert _lib.lib.mucu_nvls_create(0, 0, 1024, ctypes.byref(h)) == 1     # ranks < 1
    assert _lib.lib.mucu_nvls_import(0, 1, 1024, -1, ctypes.byref(h)) == 1  # fd < 0
    assert _lib.lib.mucu_nvls_barrier(None, None) == 1
    assert _lib.lib.mucu_nvls_destroy(None) == 0
