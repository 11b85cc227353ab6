"""ctypes binding of libmucudnn.so (include/mucudnn.h) -- argument marshalling only.

Every function here has the C ABI's name without the ``mucu_`` prefix and does
nothing but convert Python / numpy arguments to C types and raise on a non-OK
status.  All computation happens in the native library (planner) or in its
sm_100a kernels (convolutions).  There is no CPU fallback: if the shared
library is missing the import fails loudly.
"""
from __future__ import annotations

import ctypes
import os
from typing import List, Optional, Sequence, Tuple

import numpy as np

_LIB_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "lib", "libmucudnn.so")

FWD, BWD_DATA, BWD_FILTER = 0, 1, 2
IMPLICIT_GEMM, IM2COL_GEMM, WINOGRAD, FFT, FFT_TILING = 0, 1, 2, 3, 4
NUM_ALGOS = 5
MATH_F32, MATH_TF32, MATH_BF16 = 0, 1, 2
POLICY_ALL, POLICY_POW2, POLICY_UNDIVIDED = 0, 1, 2
ALGO_NAMES = {IMPLICIT_GEMM: "IG", IM2COL_GEMM: "I2C", WINOGRAD: "WG", FFT: "FFT", FFT_TILING: "FFTT"}
TYPE_NAMES = {FWD: "FWD", BWD_DATA: "DGRAD", BWD_FILTER: "WGRAD"}
MATH_NAMES = {MATH_F32: "f32", MATH_TF32: "tf32", MATH_BF16: "bf16"}

OK = 0
STATUS = ["MUCU_OK", "MUCU_ERR_INVALID_VALUE", "MUCU_ERR_UNSUPPORTED", "MUCU_ERR_INSUFFICIENT_WORKSPACE",
          "MUCU_ERR_INFEASIBLE", "MUCU_ERR_CAPACITY", "MUCU_ERR_MISALIGNED", "MUCU_ERR_CUDA", "MUCU_ERR_INTERNAL"]


class MucuError(RuntimeError):
    def __init__(self, status: int, msg: str):
        self.status = status
        super().__init__(f"{STATUS[status] if 0 <= status < len(STATUS) else status}: {msg}")


class ConvDesc(ctypes.Structure):
    _fields_ = [(f, ctypes.c_int32) for f in ("n", "c", "h", "w", "k", "r", "s", "pad", "stride", "math")]

    def __repr__(self):
        return "ConvDesc(" + ", ".join(f"{f}={getattr(self, f)}" for f, _ in self._fields_) + ")"


MAX_REDUCE_RANKS = 8


class ReduceTarget(ctypes.Structure):
    """mucu_reduce_target_t: one multicast address, or one buffer per rank (NEXT-3)."""
    _fields_ = [("multicast", ctypes.c_int32), ("count", ctypes.c_int32),
                ("dst", ctypes.c_void_p * MAX_REDUCE_RANKS)]


def reduce_target(ptrs: Sequence[int], multicast: bool = False) -> ReduceTarget:
    t = ReduceTarget()
    t.multicast = 1 if multicast else 0
    t.count = len(ptrs)
    for i, p in enumerate(ptrs):
        t.dst[i] = p
    return t


class MicroConfig(ctypes.Structure):
    _fields_ = [("algo", ctypes.c_int32), ("micro_n", ctypes.c_int32)]


def desc(n, c, h, w, k, r, s, pad, stride, math=MATH_F32) -> ConvDesc:
    return ConvDesc(n, c, h, w, k, r, s, pad, stride, math)


def _load():
    if not os.path.exists(_LIB_PATH):
        raise ImportError(f"{_LIB_PATH} not built: run `python -c 'import __graft_entry__ as g; g.build()'`")
    lib = ctypes.CDLL(_LIB_PATH)
    P = ctypes.POINTER
    i32, i64, u64, f32, vp = ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64, ctypes.c_float, ctypes.c_void_p
    D, MC = P(ConvDesc), P(MicroConfig)
    sig = {
        "mucu_status_string": (ctypes.c_char_p, [ctypes.c_int]),
        "mucu_last_error": (ctypes.c_char_p, [vp]),
        "mucu_version": (i32, []),
        "mucu_launch_count": (u64, []),
        "mucu_create": (ctypes.c_int, [P(vp), ctypes.c_int]),
        "mucu_destroy": (ctypes.c_int, [vp]),
        "mucu_set_policy": (ctypes.c_int, [vp, ctypes.c_int]),
        "mucu_set_bench_params": (ctypes.c_int, [vp, i32, i32]),
        "mucu_set_deterministic": (ctypes.c_int, [vp, i32]),
        "mucu_output_dims": (ctypes.c_int, [D, P(i32), P(i32)]),
        "mucu_workspace_size": (ctypes.c_int, [D, ctypes.c_int, ctypes.c_int, i32, P(u64)]),
        "mucu_plan_wr": (ctypes.c_int, [i32, P(i64), P(u64), u64, MC, i32, P(i32), P(i64)]),
        "mucu_pareto_front": (ctypes.c_int, [i32, P(i64), P(u64), u64, P(i64), P(u64), i32, P(i32), MC, P(i32)]),
        "mucu_solve_wd": (ctypes.c_int, [i32, P(i32), P(i64), P(u64), u64, P(i32), P(u64), P(i64)]),
        "mucu_benchmark_scratch_size": (ctypes.c_int, [D, ctypes.c_int, u64, P(u64)]),
        "mucu_benchmark": (ctypes.c_int, [vp, D, ctypes.c_int, u64, vp, u64, vp, P(i64), P(u64)]),
        "mucu_plan_layer": (ctypes.c_int, [vp, D, ctypes.c_int, u64, vp, u64, vp, MC, i32, P(i32), P(i64)]),
        "mucu_conv_forward": (ctypes.c_int, [vp, D, MC, i32, f32, vp, vp, f32, vp, vp, u64, vp]),
        "mucu_conv_backward_data": (ctypes.c_int, [vp, D, MC, i32, f32, vp, vp, f32, vp, vp, u64, vp]),
        "mucu_conv_backward_filter": (ctypes.c_int, [vp, D, MC, i32, f32, vp, vp, f32, vp, vp, u64, vp]),
        "mucu_conv_backward_filter_reduce": (ctypes.c_int, [vp, D, MC, i32, f32, vp, vp, f32, vp, P(ReduceTarget), vp,
                                                             u64, vp]),
        "mucu_peer_barrier": (ctypes.c_int, [P(ReduceTarget), vp, ctypes.c_uint32, vp]),
        "mucu_nvls_supported": (ctypes.c_int, [ctypes.c_int, P(i32)]),
        "mucu_nvls_create": (ctypes.c_int, [ctypes.c_int, i32, u64, P(vp)]),
        "mucu_nvls_export": (ctypes.c_int, [vp, P(i32)]),
        "mucu_nvls_import": (ctypes.c_int, [ctypes.c_int, i32, u64, i32, P(vp)]),
        "mucu_nvls_bind": (ctypes.c_int, [vp, P(vp), P(vp)]),
        "mucu_nvls_barrier": (ctypes.c_int, [vp, vp]),
        "mucu_nvls_destroy": (ctypes.c_int, [vp]),
        "mucu_network_create": (ctypes.c_int, [P(vp)]),
        "mucu_network_destroy": (ctypes.c_int, [vp]),
        "mucu_network_add": (ctypes.c_int, [vp, D, ctypes.c_int, P(i32)]),
        "mucu_network_plan": (ctypes.c_int, [vp, vp, u64, vp, u64, vp]),
        "mucu_network_plan_from_tables": (ctypes.c_int, [vp, u64, P(i64), P(u64)]),
        "mucu_network_get": (ctypes.c_int, [vp, i32, MC, i32, P(i32), P(u64), P(u64), P(i64)]),
    }
    for name, (res, args) in sig.items():
        fn = getattr(lib, name)
        fn.restype = res
        fn.argtypes = args
    return lib


lib = _load()


def _check(status: int):
    if status != OK:
        raise MucuError(status, lib.mucu_last_error(None).decode())


def _i64(a):
    a = np.ascontiguousarray(a, dtype=np.int64)
    return a, a.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))


def _u64(a):
    a = np.ascontiguousarray(a, dtype=np.uint64)
    return a, a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64))


def _full_tables(time_ns, ws):
    """Timing tables with fewer than NUM_ALGOS algorithm rows get the missing rows as
    'not measured' (time -1, workspace 0)."""
    t = np.asarray(time_ns, dtype=np.int64)
    w = np.asarray(ws, dtype=np.uint64)
    if t.shape[0] < NUM_ALGOS:
        pad = NUM_ALGOS - t.shape[0]
        t = np.concatenate([t, np.full((pad, t.shape[1]), -1, np.int64)])
        w = np.concatenate([w, np.zeros((pad, w.shape[1]), np.uint64)])
    return t, w


def version() -> int:
    return lib.mucu_version()


def launch_count() -> int:
    return int(lib.mucu_launch_count())


def status_string(s: int) -> str:
    return lib.mucu_status_string(s).decode()


def output_dims(d: ConvDesc) -> Tuple[int, int]:
    p, q = ctypes.c_int32(), ctypes.c_int32()
    _check(lib.mucu_output_dims(ctypes.byref(d), ctypes.byref(p), ctypes.byref(q)))
    return p.value, q.value


def workspace_size(d: ConvDesc, conv_type: int, algo: int, micro_n: int) -> int:
    b = ctypes.c_uint64()
    _check(lib.mucu_workspace_size(ctypes.byref(d), conv_type, algo, micro_n, ctypes.byref(b)))
    return b.value


def plan_wr(n: int, time_ns, ws, ws_limit: int) -> Tuple[int, List[Tuple[int, int]]]:
    """WR DP.  time_ns, ws: [NUM_ALGOS][n+1] (fewer rows: the rest unmeasured).
    Returns (total_ns, [(algo, b), ...])."""
    time_ns, ws = _full_tables(time_ns, ws)
    t, tp = _i64(time_ns)
    w, wp = _u64(ws)
    assert t.shape == (NUM_ALGOS, n + 1) and w.shape == t.shape
    out = (MicroConfig * n)()
    cnt, tot = ctypes.c_int32(), ctypes.c_int64()
    _check(lib.mucu_plan_wr(n, tp, wp, int(ws_limit), out, n, ctypes.byref(cnt), ctypes.byref(tot)))
    return tot.value, [(out[i].algo, out[i].micro_n) for i in range(cnt.value)]


def pareto_front(n: int, time_ns, ws, ws_cap: int = (1 << 64) - 1):
    """WD desirable set.  Returns [(T, M, [(algo, b), ...]), ...] sorted by M."""
    time_ns, ws = _full_tables(time_ns, ws)
    t, tp = _i64(time_ns)
    w, wp = _u64(ws)
    ln = ctypes.c_int32()
    st = lib.mucu_pareto_front(n, tp, wp, int(ws_cap), None, None, 0, ctypes.byref(ln), None, None)
    if st not in (OK, 5):
        _check(st)
    L = ln.value
    ft = np.zeros(L, np.int64)
    fm = np.zeros(L, np.uint64)
    plans = (MicroConfig * (L * n))()
    plen = np.zeros(L, np.int32)
    _check(lib.mucu_pareto_front(n, tp, wp, int(ws_cap), ft.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                 fm.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)), L, ctypes.byref(ln), plans,
                                 plen.ctypes.data_as(ctypes.POINTER(ctypes.c_int32))))
    res = []
    for i in range(L):
        res.append((int(ft[i]), int(fm[i]), [(plans[i * n + j].algo, plans[i * n + j].micro_n) for j in range(plen[i])]))
    return res


def solve_wd(fronts: Sequence[Sequence[Tuple[int, int]]], total_limit: int):
    """WD MCKP (Eq. (1)-(4)).  fronts[k] = [(t, m), ...].  Returns (total_ns, choice list, offsets)."""
    K = len(fronts)
    flen = np.array([len(f) for f in fronts], np.int32)
    t = np.array([int(x[0]) for f in fronts for x in f], np.int64)
    m = np.array([int(x[1]) for f in fronts for x in f], np.uint64)
    choice = np.zeros(K, np.int32)
    off = np.zeros(K, np.uint64)
    tot = ctypes.c_int64()
    _check(lib.mucu_solve_wd(K, flen.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)),
                             t.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                             m.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)), int(total_limit),
                             choice.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)),
                             off.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64)), ctypes.byref(tot)))
    return tot.value, [int(c) for c in choice], [int(o) for o in off]


def benchmark_scratch_size(d: ConvDesc, conv_type: int, ws_limit: int) -> int:
    b = ctypes.c_uint64()
    _check(lib.mucu_benchmark_scratch_size(ctypes.byref(d), conv_type, int(ws_limit), ctypes.byref(b)))
    return b.value


def _plan_array(plan: Sequence[Tuple[int, int]]):
    arr = (MicroConfig * len(plan))()
    for i, (a, b) in enumerate(plan):
        arr[i].algo, arr[i].micro_n = int(a), int(b)
    return arr


class Handle:
    """One library handle per device (mucu_create / mucu_destroy)."""

    def __init__(self, device: int = 0):
        h = ctypes.c_void_p()
        _check(lib.mucu_create(ctypes.byref(h), device))
        self._h = h

    def close(self):
        if self._h is not None and self._h.value:
            lib.mucu_destroy(self._h)
        self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    @property
    def ptr(self):
        return self._h

    def set_policy(self, policy: int):
        _check(lib.mucu_set_policy(self._h, policy))

    def set_deterministic(self, deterministic: bool):
        """BackwardFilter split-K reduction: fixed order (default) or L2 atomics."""
        _check(lib.mucu_set_deterministic(self._h, 1 if deterministic else 0))

    def set_bench_params(self, warmup: int, reps: int):
        _check(lib.mucu_set_bench_params(self._h, warmup, reps))

    def benchmark(self, d: ConvDesc, conv_type: int, ws_limit: int, scratch_ptr: int, scratch_bytes: int,
                  stream: int):
        n = d.n
        t = np.zeros((NUM_ALGOS, n + 1), np.int64)
        w = np.zeros((NUM_ALGOS, n + 1), np.uint64)
        _check(lib.mucu_benchmark(self._h, ctypes.byref(d), conv_type, int(ws_limit), ctypes.c_void_p(scratch_ptr),
                                  int(scratch_bytes), ctypes.c_void_p(stream),
                                  t.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                  w.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64))))
        return t, w

    def plan_layer(self, d: ConvDesc, conv_type: int, ws_limit: int, scratch_ptr: int, scratch_bytes: int,
                   stream: int):
        out = (MicroConfig * d.n)()
        cnt, tot = ctypes.c_int32(), ctypes.c_int64()
        _check(lib.mucu_plan_layer(self._h, ctypes.byref(d), conv_type, int(ws_limit), ctypes.c_void_p(scratch_ptr),
                                   int(scratch_bytes), ctypes.c_void_p(stream), out, d.n, ctypes.byref(cnt),
                                   ctypes.byref(tot)))
        return tot.value, [(out[i].algo, out[i].micro_n) for i in range(cnt.value)]

    def _conv(self, fn, d, plan, alpha, p0, p1, beta, pout, ws_ptr, ws_bytes, stream):
        arr = _plan_array(plan)
        _check(fn(self._h, ctypes.byref(d), arr, len(plan), float(alpha), ctypes.c_void_p(p0), ctypes.c_void_p(p1),
                  float(beta), ctypes.c_void_p(pout), ctypes.c_void_p(ws_ptr or 0), int(ws_bytes),
                  ctypes.c_void_p(stream)))

    def conv_forward(self, d, plan, alpha, x, w, beta, y, ws_ptr, ws_bytes, stream):
        self._conv(lib.mucu_conv_forward, d, plan, alpha, x, w, beta, y, ws_ptr, ws_bytes, stream)

    def conv_backward_data(self, d, plan, alpha, dy, w, beta, dx, ws_ptr, ws_bytes, stream):
        self._conv(lib.mucu_conv_backward_data, d, plan, alpha, dy, w, beta, dx, ws_ptr, ws_bytes, stream)

    def conv_backward_filter(self, d, plan, alpha, x, dy, beta, dw, ws_ptr, ws_bytes, stream):
        self._conv(lib.mucu_conv_backward_filter, d, plan, alpha, x, dy, beta, dw, ws_ptr, ws_bytes, stream)

    def conv_backward_filter_reduce(self, d, plan, alpha, x, dy, beta, dw, target: ReduceTarget, ws_ptr, ws_bytes,
                                    stream):
        arr = _plan_array(plan)
        _check(lib.mucu_conv_backward_filter_reduce(
            self._h, ctypes.byref(d), arr, len(plan), float(alpha), ctypes.c_void_p(x), ctypes.c_void_p(dy),
            float(beta), ctypes.c_void_p(dw), ctypes.byref(target), ctypes.c_void_p(ws_ptr or 0), int(ws_bytes),
            ctypes.c_void_p(stream)))


def peer_barrier(flags: ReduceTarget, own: int, target: int, stream: int = 0):
    _check(lib.mucu_peer_barrier(ctypes.byref(flags), ctypes.c_void_p(own), int(target), ctypes.c_void_p(stream)))


def nvls_supported(device: int = 0) -> bool:
    v = ctypes.c_int32()
    _check(lib.mucu_nvls_supported(device, ctypes.byref(v)))
    return bool(v.value)


class Nvls:
    """One rank's NVLink multicast buffer (NEXT-3; include/mucudnn.h).  Rank 0 creates
    (``fd=None``) and exports an fd for the peers; the others import it."""

    def __init__(self, device: int, ranks: int, nbytes: int, fd: Optional[int] = None):
        h = ctypes.c_void_p()
        if fd is None:
            _check(lib.mucu_nvls_create(device, ranks, int(nbytes), ctypes.byref(h)))
        else:
            _check(lib.mucu_nvls_import(device, ranks, int(nbytes), int(fd), ctypes.byref(h)))
        self._h = h
        self.local = self.multicast = None

    def export(self) -> int:
        fd = ctypes.c_int32()
        _check(lib.mucu_nvls_export(self._h, ctypes.byref(fd)))
        return fd.value

    def bind(self) -> Tuple[int, int]:
        loc, mc = ctypes.c_void_p(), ctypes.c_void_p()
        _check(lib.mucu_nvls_bind(self._h, ctypes.byref(loc), ctypes.byref(mc)))
        self.local, self.multicast = loc.value, mc.value
        return self.local, self.multicast

    def barrier(self, stream: int = 0):
        _check(lib.mucu_nvls_barrier(self._h, ctypes.c_void_p(stream)))

    def close(self):
        if self._h is not None and self._h.value:
            lib.mucu_nvls_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Network:
    """WD kernel list: add kernels, plan once, query plans/segments."""

    def __init__(self):
        h = ctypes.c_void_p()
        _check(lib.mucu_network_create(ctypes.byref(h)))
        self._h = h
        self.descs: List[Tuple[ConvDesc, int]] = []

    def __del__(self):
        try:
            if self._h is not None and self._h.value:
                lib.mucu_network_destroy(self._h)
        except Exception:
            pass

    def add(self, d: ConvDesc, conv_type: int) -> int:
        kid = ctypes.c_int32()
        _check(lib.mucu_network_add(self._h, ctypes.byref(d), conv_type, ctypes.byref(kid)))
        self.descs.append((d, conv_type))
        return kid.value

    def plan(self, handle: Handle, total_limit: int, scratch_ptr: int, scratch_bytes: int, stream: int):
        _check(lib.mucu_network_plan(self._h, handle.ptr, int(total_limit), ctypes.c_void_p(scratch_ptr),
                                     int(scratch_bytes), ctypes.c_void_p(stream)))

    def plan_from_tables(self, total_limit: int, tables):
        tables = [_full_tables(tt, ww) for tt, ww in tables]
        t = np.concatenate([tt.ravel() for tt, _ in tables])
        w = np.concatenate([ww.ravel() for _, ww in tables])
        _check(lib.mucu_network_plan_from_tables(self._h, int(total_limit),
                                                 t.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                                 w.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64))))

    def get(self, kernel_id: int):
        n = self.descs[kernel_id][0].n
        out = (MicroConfig * n)()
        cnt = ctypes.c_int32()
        off, nb, t = ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_int64()
        _check(lib.mucu_network_get(self._h, kernel_id, out, n, ctypes.byref(cnt), ctypes.byref(off),
                                    ctypes.byref(nb), ctypes.byref(t)))
        return [(out[i].algo, out[i].micro_n) for i in range(cnt.value)], off.value, nb.value, t.value
