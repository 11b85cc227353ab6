"""Network-level planning and execution of conv layers (Sec. III/III-A).

ConvNet owns, for a list of conv layers at mini-batch N:
* device tensors (x, w, dy inputs; y, dx, dw outputs) -- NHWC / KRSC,
* one plan per kernel (layer x {FWD, DGRAD, WGRAD}) from
  - WR: per-kernel benchmark + DP under a per-layer workspace limit,
    one workspace per kernel (Fig. 4, "one workspace per layer"), or
  - WD: one network workspace, per-kernel desirable sets + the
    exact MCKP, each kernel a segment of it (Fig. 14),
  - "undivided": the fastest single algorithm at micro-batch N that
    fits the same limit -- the comparison baseline of BASELINE.json,
* `iteration()`: forward of every layer in order, then BackwardData and
  BackwardFilter in reverse order (the conv part of a training iteration,
  P:L198), each call executing its plan through the C ABI.

In data-parallel runs each BackwardFilter output is handed to `grad_hook`
(e.g. an asynchronous NCCL allreduce, see distributed.py) right after its last
micro-batch, so communication overlaps the remaining backward layers.
"""
from __future__ import annotations

from dataclasses import dataclass, field
from typing import Callable, Dict, List, Optional, Sequence, Tuple

import numpy as np
import torch

from . import _lib as L
from . import torch_api as T

TYPES = (L.FWD, L.BWD_DATA, L.BWD_FILTER)


@dataclass
class Kernel:
    layer: int
    conv_type: int
    desc: L.ConvDesc
    plan: List[Tuple[int, int]] = field(default_factory=list)
    table: Optional[Tuple[np.ndarray, np.ndarray]] = None
    est_ns: int = 0
    ws_bytes: int = 0
    ws_offset: int = 0


def layer_flops(layer, n: int) -> int:
    """Direct-convolution FLOPs of one direction, 2 N K C R S P Q."""
    return 2 * n * layer.k * layer.c * layer.r * layer.s * layer.p * layer.q


def fft_tiling(layer, conv_type: int, algo: int):
    """(F, tiles per image) of FFT / FFT_TILING (kernels_fft.cu fft_geom)."""
    eh, ew = (layer.h, layer.w) if conv_type == L.BWD_DATA else (layer.p, layer.q)
    if algo == L.FFT:
        f = 8
        while f < max(eh + layer.r - 1, ew + layer.s - 1):
            f *= 2
        return f, 1
    th, tw = min(eh, 33 - layer.r), min(ew, 33 - layer.s)
    return 32, -(-eh // th) * -(-ew // tw)


def algorithmic_flops(layer, conv_type: int, plan) -> int:
    """Tensor/FMA work the chosen algorithms actually perform:
    IG / I2C: 2 b K C R S P Q; Winograd F(2x2,3x3): 16 GEMMs of 2 (b T) K C;
    FFT / FFT_TILING: F (F/2 + 1) complex GEMMs of 8 (b tiles) K C (transforms excluded)."""
    f = 0
    for algo, b in plan:
        if algo in (L.FFT, L.FFT_TILING):
            F, tiles = fft_tiling(layer, conv_type, algo)
            f += 8 * F * (F // 2 + 1) * b * tiles * layer.k * layer.c
        elif algo == L.WINOGRAD:
            oh, ow = (layer.h, layer.w) if conv_type == L.BWD_DATA else (layer.p, layer.q)
            t = ((oh + 1) // 2) * ((ow + 1) // 2)
            f += 2 * 16 * b * t * layer.k * layer.c
        else:
            f += layer_flops(layer, b)
    return f


def algorithmic_bytes(layer, conv_type: int, n: int, elt: int) -> int:
    """HBM bytes the convolution must move once (SURVEY 8(d) "IG: x + w + y"):
    the operands and the result, no workspace; dW is fp32 (written once, beta = 0)."""
    x = n * layer.h * layer.w * layer.c * elt
    y = n * layer.p * layer.q * layer.k * elt
    w = layer.k * layer.r * layer.s * layer.c * elt
    if conv_type == L.BWD_FILTER:
        return x + y + layer.k * layer.r * layer.s * layer.c * 4
    return x + y + w


def shard_benchmark(costs: Dict[str, int], world: int) -> List[List[str]]:
    """Assign benchmark jobs to ranks: longest-processing-time first onto the
    least-loaded rank (ties -> lower rank), deterministic on every rank."""
    shards: List[List[str]] = [[] for _ in range(world)]
    load = [0] * world
    for dk in sorted(costs, key=lambda d: (-costs[d], d)):
        r = min(range(world), key=lambda i: (load[i], i))
        shards[r].append(dk)
        load[r] += costs[dk]
    return shards


class ConvNet:
    def __init__(self, handle: L.Handle, layers: Sequence, n: int, math: int, device: str = "cuda",
                 types: Sequence[int] = TYPES):
        """types: the convolution operations to plan and run per layer (all three for
        a training iteration; e.g. (FWD,) for BASELINE config 1)."""
        self.h = handle
        self.types = tuple(types)
        self.layers = list(layers)
        self.n = n
        self.math = math
        self.device = device
        self.dtype = torch.bfloat16 if math == L.MATH_BF16 else torch.float32
        self.descs = [L.desc(n, l.c, l.h, l.w, l.k, l.r, l.s, l.pad, l.stride, math) for l in self.layers]
        self.kernels: Dict[Tuple[int, int], Kernel] = {
            (i, t): Kernel(i, t, d) for i, d in enumerate(self.descs) for t in self.types}
        self.tensors: List[Dict[str, torch.Tensor]] = []
        self.workspaces: Dict[Tuple[int, int], Optional[torch.Tensor]] = {}
        self.net_ws: Optional[torch.Tensor] = None
        self.nvls = None  # distributed.FusedGradReduce over dw_flat (NEXT-3), set by the caller

    # ----------------------------------------------------------- memory --
    def allocate(self, seed: int = 0, kind: str = "normal", generator=None):
        """Seeded synthetic tensors on the device (values do not affect timing)."""
        from synthetic import torch_conv_inputs  # workload generator (no method arithmetic)
        self.tensors = []
        # all filter gradients are views of one flat fp32 buffer, zeroed once per
        # iteration (the framework's zero_grad); BackwardFilter then accumulates with
        # beta = 1, so no per-layer beta = 0 pre-scale launch is needed
        shapes = [T.shapes(d)[1] for d in self.descs]
        sizes = [int(np.prod(s_)) for s_ in shapes]
        offs = [0]
        for n_ in sizes:
            offs.append(offs[-1] + (n_ + 63) // 64 * 64)  # 256-B aligned views
        self.dw_flat = torch.zeros(max(offs[-1], 1), dtype=torch.float32, device=self.device)
        for i, (l, d) in enumerate(zip(self.layers, self.descs)):
            x, w, dy = torch_conv_inputs(l, self.n, seed=1000 * seed + i, device=self.device, dtype=self.dtype,
                                         kind=kind)
            xs, ws_, ys = T.shapes(d)
            self.tensors.append(dict(
                x=x, w=w, dy=dy,
                y=torch.empty(ys, dtype=self.dtype, device=self.device),
                dx=torch.empty(xs, dtype=self.dtype, device=self.device),
                dw=self.dw_flat[offs[i]:offs[i] + sizes[i]].view(ws_)))

    # ---------------------------------------------------------- planning --
    def benchmark_all(self, ws_limit: int, progress: Optional[Callable] = None, group=None):
        """P:L88 step 1 for every kernel.  Identical kernels (same descriptor and
        type) are benchmarked once (P:L159 cache).  In a data-parallel job the
        unique kernels are sharded over the ranks (largest first onto the least
        loaded rank) and the tables all-gathered: homogeneous GPUs give the same
        tables, so the pass takes ~1/world of the time (SURVEY 8(f)
        NEXT-2)."""
        import torch.distributed as dist
        world = dist.get_world_size(group) if dist.is_available() and dist.is_initialized() else 1
        rank = dist.get_rank(group) if world > 1 else 0
        uniq: Dict[str, List[Tuple[int, int]]] = {}
        for key, k in self.kernels.items():
            uniq.setdefault(self._db_key(k, ws_limit, "bench"), []).append(key)
        costs = {dk: layer_flops(self.layers[keys[0][0]], self.n) for dk, keys in uniq.items()}
        mine = shard_benchmark(costs, world)[rank]
        local = {}
        scratch = None
        for dk in mine:
            k = self.kernels[uniq[dk][0]]
            need = L.benchmark_scratch_size(k.desc, k.conv_type, ws_limit)
            if scratch is None or scratch.numel() < need:
                scratch = None
                torch.cuda.empty_cache()
                scratch = T.make_scratch(k.desc, k.conv_type, ws_limit)
            local[dk] = self.h.benchmark(k.desc, k.conv_type, ws_limit, scratch.data_ptr(), scratch.numel(),
                                         T._stream())
            if progress:
                progress(uniq[dk][0])
        del scratch
        if torch.cuda.is_available():
            torch.cuda.empty_cache()
        tables = local
        if world > 1:
            parts = [None] * world
            dist.all_gather_object(parts, local, group=group)
            tables = {dk: tb for part in parts for dk, tb in part.items()}
        for dk, keys in uniq.items():
            for key in keys:
                self.kernels[key].table = tables[dk]

    # File-based benchmark DB ("caches ... the benchmark results into ...
    # optional file-based database", enabling offline benchmarking and sharing
    # among homogeneous GPUs).  Keyed by descriptor, conv type and limit.
    @staticmethod
    def _db_key(k: Kernel, ws_limit: int, policy: str) -> str:
        d = k.desc
        return (f"{d.n},{d.c},{d.h},{d.w},{d.k},{d.r},{d.s},{d.pad},{d.stride},{d.math}|{k.conv_type}|"
                f"{ws_limit}|{policy}")

    def save_tables(self, path: str, ws_limit: int, policy: str):
        arrs = {}
        for k in self.kernels.values():
            key = self._db_key(k, ws_limit, policy)
            arrs[key + "|t"], arrs[key + "|w"] = k.table
        np.savez(path, **arrs)

    def load_tables(self, path: str, ws_limit: int, policy: str) -> bool:
        """Fill every kernel's table from the DB; False if any entry is missing."""
        db = np.load(path)
        for k in self.kernels.values():
            key = self._db_key(k, ws_limit, policy)
            if key + "|t" not in db:
                return False
            k.table = (db[key + "|t"], db[key + "|w"])
        return True

    def plan_wr(self, ws_limit: int):
        """WR: per-kernel DP on its timing table; one workspace per kernel."""
        for k in self.kernels.values():
            t, w = k.table
            k.est_ns, k.plan = L.plan_wr(self.n, t, w, ws_limit)
            k.ws_bytes = T.plan_workspace(k.desc, k.conv_type, k.plan)
        self._alloc_workspaces()

    def plan_undivided(self, ws_limit: int):
        """Best single algorithm at micro-batch N within the limit: the
        C planner (mucu_plan_wr) on the table restricted to b = N, i.e. exactly
        what the `undivided` batch-size policy benchmarks."""
        n = self.n
        for k in self.kernels.values():
            t, w = k.table
            tu = np.full_like(t, -1)
            tu[:, n] = t[:, n]
            k.est_ns, k.plan = L.plan_wr(n, tu, w, ws_limit)
            k.ws_bytes = T.plan_workspace(k.desc, k.conv_type, k.plan)
        self._alloc_workspaces()

    def plan_wd(self, total_limit: int):
        """WD: desirable sets + exact MCKP over all kernels, one
        network workspace carved into 256-B aligned segments (reading G18)."""
        import time
        net = L.Network()
        order = list(self.kernels.keys())
        for key in order:
            net.add(self.kernels[key].desc, key[1])
        tables = [self.kernels[key].table for key in order]
        t0 = time.perf_counter()
        net.plan_from_tables(total_limit, tables)  # fronts (set-valued DP) + MCKP, in the C library
        self.wd_stats = {"kernels": len(order), "plan_ms": round((time.perf_counter() - t0) * 1e3, 3),
                         "total_limit_mib": round(total_limit / 2 ** 20, 3)}
        # ILP size (562 binary variables for ResNet-50): one 0-1 variable per
        # desirable configuration of every kernel; the exact MCKP is timed alone
        fronts = [L.pareto_front(self.n, t, w, total_limit) for t, w in tables]
        self.wd_stats["ilp_variables"] = int(sum(len(f) for f in fronts))
        t1 = time.perf_counter()
        L.solve_wd([[(int(T), int(M)) for T, M, _ in f] for f in fronts], total_limit)
        self.wd_stats["ilp_solve_ms"] = round((time.perf_counter() - t1) * 1e3, 3)
        for kid, key in enumerate(order):
            k = self.kernels[key]
            k.plan, k.ws_offset, k.ws_bytes, k.est_ns = net.get(kid)
        total = max((k.ws_offset + k.ws_bytes for k in self.kernels.values()), default=0)
        self.net_ws = torch.empty(max(total, 256), dtype=torch.uint8, device=self.device)
        self.workspaces = {key: (self.net_ws[k.ws_offset:k.ws_offset + k.ws_bytes] if k.ws_bytes else None)
                           for key, k in self.kernels.items()}

    def _alloc_workspaces(self):
        self.net_ws = None
        self.workspaces = {}
        for key, k in self.kernels.items():
            self.workspaces[key] = torch.empty(k.ws_bytes, dtype=torch.uint8, device=self.device) if k.ws_bytes else None

    def total_workspace(self) -> int:
        if self.net_ws is not None:
            return self.net_ws.numel()
        return sum(k.ws_bytes for k in self.kernels.values())

    # --------------------------------------------------------- execution --
    def run_kernel(self, i: int, conv_type: int):
        k = self.kernels[(i, conv_type)]
        t = self.tensors[i]
        ws = self.workspaces.get((i, conv_type))
        if conv_type == L.FWD:
            T.conv_forward(self.h, k.desc, k.plan, t["x"], t["w"], t["y"], workspace=ws)
        elif conv_type == L.BWD_DATA:
            T.conv_backward_data(self.h, k.desc, k.plan, t["dy"], t["w"], t["dx"], workspace=ws)
        elif self.nvls is not None:  # NEXT-3: the cross-rank sum fused into the epilogue
            T.conv_backward_filter_reduce(self.h, k.desc, k.plan, t["x"], t["dy"], t["dw"],
                                          self.nvls.target(t["dw"].data_ptr() - self.dw_flat.data_ptr()),
                                          beta=1.0, workspace=ws)
        else:  # dw was zeroed at the start of the backward pass (zero_grad): accumulate
            T.conv_backward_filter(self.h, k.desc, k.plan, t["x"], t["dy"], t["dw"], beta=1.0, workspace=ws)

    def iteration(self, on_op: Optional[Callable] = None, grad_hook: Optional[Callable] = None,
                  skip_conv1_dgrad: bool = False, concurrent: bool = False):
        """FWD of all layers, then DGRAD + WGRAD in reverse order.  on_op(i, type,
        'begin'|'end') lets a caller record CUDA events around each call.

        concurrent=True runs each layer's BackwardFilter on a side stream next to
        its BackwardData (both only need the layer's dy, i.e. the previous
        BackwardData): the two persistent kernels fill each other's partial last
        waves.  Each kernel keeps its own workspace (WR) or segment (WD), so the
        overlap is memory-safe; results are unchanged."""
        if concurrent:
            return self._iteration_concurrent(grad_hook, skip_conv1_dgrad, on_op)
        order = [(i, L.FWD) for i in range(len(self.layers))]
        for i in reversed(range(len(self.layers))):
            if not (skip_conv1_dgrad and i == 0):
                order.append((i, L.BWD_DATA))
            order.append((i, L.BWD_FILTER))
        order = [o for o in order if o in self.kernels]
        zeroed = False
        for i, t in order:
            if t != L.FWD and not zeroed:
                self.dw_flat.zero_()  # zero_grad, once per iteration, before the first backward call
                if self.nvls is not None:
                    self.nvls.begin()
                zeroed = True
            if on_op:
                on_op(i, t, "begin")
            self.run_kernel(i, t)
            if on_op:
                on_op(i, t, "end")
            if t == L.BWD_FILTER and grad_hook is not None:
                grad_hook(i, self.tensors[i]["dw"])
        if self.nvls is not None and zeroed:
            self.nvls.end()

    def _iteration_concurrent(self, grad_hook, skip_conv1_dgrad, on_op=None):
        """on_op(i, type, 'begin'|'end') runs on the host around each call with the
        call's stream current (for stream-ordered hooks; not for event timing)."""
        main = torch.cuda.current_stream()
        if getattr(self, "_side", None) is None:
            self._side = torch.cuda.Stream()
            self._dy_ready = [torch.cuda.Event() for _ in self.layers]
        side = self._side
        hook = on_op or (lambda *a: None)

        def run(i, t):
            if (i, t) not in self.kernels:
                return
            hook(i, t, "begin")
            self.run_kernel(i, t)
            hook(i, t, "end")
        for i in range(len(self.layers)):
            run(i, L.FWD)
        self.dw_flat.zero_()  # zero_grad, once per iteration, before the first backward call
        if self.nvls is not None:
            self.nvls.begin()
        for i in reversed(range(len(self.layers))):
            if i == len(self.layers) - 1:
                hook(i, L.BWD_DATA, "first")  # stream-ordered setup before any backward call
            # dy of layer i: produced by the previous BackwardData on the main stream
            self._dy_ready[i].record(main)
            if not (skip_conv1_dgrad and i == 0):
                run(i, L.BWD_DATA)
            side.wait_event(self._dy_ready[i])
            with torch.cuda.stream(side):
                run(i, L.BWD_FILTER)
                if grad_hook is not None:
                    grad_hook(i, self.tensors[i]["dw"])
        main.wait_stream(side)
        if self.nvls is not None:
            self.nvls.end()

    def flops_per_iteration(self, skip_conv1_dgrad: bool = False) -> int:
        f = sum(layer_flops(self.layers[i], self.n) for (i, t) in self.kernels)
        return f - (layer_flops(self.layers[0], self.n) if skip_conv1_dgrad and (0, L.BWD_DATA) in self.kernels else 0)

    def summary(self):
        rows = []
        for (i, t), k in sorted(self.kernels.items()):
            rows.append(dict(layer=self.layers[i].name, type=L.TYPE_NAMES[t],
                             plan=[(L.ALGO_NAMES[a], b) for a, b in k.plan], est_us=k.est_ns / 1e3,
                             ws_MiB=round(k.ws_bytes / 2 ** 20, 3)))
        return rows
