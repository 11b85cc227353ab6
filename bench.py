"""bench.py -- conv fwd+bwd ms/iter of micro-batched plans vs the best undivided
algorithm at the same workspace (BASELINE.json metric), on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--config alexnet|resnet18|resnet50] [--math tf32|bf16|f32]
                    [--policy pow2|all|undivided] [--ws-mib 64] [--wd-mib T] [--batch 256]
                    [--layers conv2] [--types fwd,dgrad,wgrad] [--global-batch G]

BASELINE.json configs as bench lines:
  cfg1  --config alexnet --layers conv2 --types fwd --batch 8 --math f32 --ws-mib 8 --policy all
  cfg2  (default: TF32) / --math f32
  cfg3  --config resnet18 --math bf16 --wd-mib 480
  cfg4  --config resnet50 --math bf16 [--wd-mib 10176]
  cfg5  --config resnet50 --math bf16 --global-batch 2048 --gpus N   (strong scaling, 2048/N per GPU)
With --gpus N > 1 and no torchrun environment, bench.py re-launches itself
under torch.distributed.run with N ranks (one per GPU, NCCL, 127.0.0.1).

Default (N=1): BASELINE.json configs[1] -- AlexNet's 5 conv layers, forward +
backward (15 kernels; --no-input-grad drops the first layer's BackwardData as
Caffe's `time` command does), N=256 per GPU, fp32 storage with TF32 tensor cores,
WR policy with a 64 MiB per-kernel workspace limit, `powerOfTwo` batch policy.
A step = one pass of the whole hot path: for every kernel the planned
sequence of micro-batches through the C ABI.  Synthetic seeded NHWC data.

Timing: W untimed warm-ups, then K steps; before every step a 512 MiB buffer
is overwritten (L2 flush, outside the timed events); each step is bracketed
by CUDA events on the launching stream; barrier + synchronize around the
region; value = max over ranks of the mean step time.
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "conv fwd+bwd ms/iter at fixed workspace vs best undivided algo; TC util vs peak"
MATHS = {"f32": 0, "tf32": 1, "bf16": 2}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="alexnet", choices=["alexnet", "resnet18", "resnet50"])
    ap.add_argument("--math", default="tf32", choices=list(MATHS))
    ap.add_argument("--policy", default="pow2", choices=["pow2", "all", "undivided"])
    ap.add_argument("--ws-mib", type=float, default=64.0, help="WR per-kernel workspace limit (MiB)")
    ap.add_argument("--wd-mib", type=float, default=0.0, help="use WD with this total workspace (MiB)")
    ap.add_argument("--batch", type=int, default=256, help="mini-batch per GPU")
    ap.add_argument("--global-batch", type=int, default=0,
                    help="global mini-batch sharded over the ranks (strong scaling, cfg5); overrides --batch")
    ap.add_argument("--layers", default="", help="comma-separated layer names to run (default: all conv layers)")
    ap.add_argument("--types", default="fwd,dgrad,wgrad", help="conv operations per layer (fwd,dgrad,wgrad)")
    ap.add_argument("--no-input-grad", dest="input_grad", action="store_false",
                    help="skip the first layer's BackwardData (the data layer needs no gradient, as in "
                         "Caffe's `time` command, P:L198); the default times all 3 kernels per layer (SURVEY 8(d) cfg2)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-concurrent-wgrad", dest="concurrent_wgrad", action="store_false",
                    help="run each BackwardFilter after its BackwardData on one stream")
    ap.add_argument("--cpu-sample", type=int, default=0, help="oracle sample (images per kernel); 0 = auto")
    ap.add_argument("--nondeterministic", action="store_true",
                    help="BackwardFilter split-K partials added with L2 atomics (mucu_set_deterministic(0)); "
                         "default: fixed-order reduction, bitwise reproducible dW")
    ap.add_argument("--grad-reduce", default="nccl", choices=["nccl", "nvls", "p2p"],
                    help="cross-rank dW sum: async NCCL allreduce per layer, or fused into the BackwardFilter "
                         "epilogue (NEXT-3): multimem.red to an NVLink multicast buffer (nvls) or red.global.add "
                         "to every rank's buffer over NVLink P2P (p2p); both also run at one GPU")
    ap.add_argument("--oracle-probe", type=int, default=0, help=argparse.SUPPRESS)  # internal: time N oracle images
    ap.add_argument("--json-out", default="")
    ap.add_argument("--tables-in", default="", help="benchmark DB (.npz) to plan from instead of benchmarking")
    ap.add_argument("--tables-out", default="", help="write the benchmark DB (.npz) after the benchmark pass")
    return ap.parse_args()


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d, "measured"
    return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0, "sm_max_mhz": 1965.0}, "fallback"


class ClockSampler:
    """Samples SM clock and throttle reasons (NVML) during the timed region."""
    NAMES = {0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
             0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
             0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting"}

    def __init__(self, index):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.hd = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.hd, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:
            pass

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.hd, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.hd)
                for bit, name in self.NAMES.items():
                    if r & bit and bit != 0x1:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.02)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        if self.ok:
            self._stop.set()
            self.t.join()

    def result(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons)}
        return {"sm_mhz": float(np.median(self.samples)), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ---------------------------------------------------------------- workload --
TYPE_KEYS = {"fwd": 0, "dgrad": 1, "wgrad": 2}


def select(args):
    """(layers, kernels): the conv layers of --config (restricted by --layers) and
    the (layer index, conv type) pairs one step runs, in iteration order."""
    from synthetic import network
    layers = network(args.config)
    if args.layers:
        names = [n.strip() for n in args.layers.split(",") if n.strip()]
        missing = [n for n in names if n not in {l.name for l in layers}]
        if missing:
            raise SystemExit(f"unknown layer(s) {missing} in {args.config}")
        layers = [l for l in layers if l.name in names]
    types = sorted({TYPE_KEYS[t.strip()] for t in args.types.split(",") if t.strip()})
    kernels = [(i, 0) for i in range(len(layers)) if 0 in types]
    for i in reversed(range(len(layers))):
        if 1 in types and not (i == 0 and not args.input_grad):
            kernels.append((i, 1))
        if 2 in types:
            kernels.append((i, 2))
    return layers, types, kernels


def workload_name(args, layers, types, kernels):
    tnames = "+".join(["fwd", "dgrad", "wgrad"][t] for t in types)
    what = "fwd+bwd" if types == [0, 1, 2] else tnames
    scope = "conv layers" if not args.layers else ",".join(l.name for l in layers)
    return f"{args.config} {scope} {what} ({len(kernels)} kernel{'s' if len(kernels) != 1 else ''})"


# --------------------------------------------------------------- oracle arm --
def oracle_sample_time(layers, kernels, n_sample, threads=None):
    """Time the fp64 oracle (oracle/, unchanged) on n_sample images of every
    kernel of the step; returns seconds."""
    import oracle
    from synthetic import conv_inputs
    if threads:
        os.environ["OMP_NUM_THREADS"] = str(threads)
    oracle.build()
    tot = 0.0
    for i, l in enumerate(layers):
        ts = [t for (j, t) in kernels if j == i]
        if not ts:
            continue
        x, w, dy = conv_inputs(n_sample, l.c, l.h, l.w, l.k, l.r, l.s, l.pad, l.stride, seed=i)
        x, w, dy = x.astype(np.float64), w.astype(np.float64), dy.astype(np.float64)
        t0 = time.perf_counter()
        if 0 in ts:
            oracle.conv_forward(x, w, l.pad, l.stride)
        if 1 in ts:
            oracle.conv_backward_data(dy, w, l.h, l.w, l.pad, l.stride)
        if 2 in ts:
            oracle.conv_backward_filter(x, dy, l.r, l.s, l.pad, l.stride)
        tot += time.perf_counter() - t0
    return tot


def single_thread_ms(batch):
    """The oracle on ONE host thread: one image of every kernel of the
    step in a child process with OMP_NUM_THREADS=1, scaled to N = batch."""
    import subprocess
    cmd = [sys.executable, os.path.abspath(__file__), "--oracle-probe", "1"] + \
        [a for a in sys.argv[1:] if not a.startswith("--json-out")]
    try:
        r = subprocess.run(cmd, env=dict(os.environ, OMP_NUM_THREADS="1"), capture_output=True, text=True,
                           timeout=600)
        secs = float(r.stdout.strip().splitlines()[-1])
    except Exception:  # noqa: BLE001 -- a reported extra, never fatal
        return None
    return round(secs * 1e3 * batch, 3)


def cpu_baseline(layers, kernels, batch, n_sample):
    cores = os.cpu_count()
    secs = oracle_sample_time(layers, kernels, n_sample)
    ms_per_iter = secs * 1e3 * batch / n_sample
    exact = n_sample == batch
    return {"value": round(ms_per_iter, 3), "unit": "ms/iter", "cores": cores, "kind": "oracle",
            "single_thread_value": single_thread_ms(batch),
            "sample": f"{n_sample} image(s) per kernel, all {len(kernels)} timed kernels, fp64 7-loop oracle "
                      f"(OpenMP, {cores} threads), {secs:.2f} s measured"
                      + ("" if exact else f", x{batch // n_sample} extrapolated to N={batch} (work is linear in N, P:L50)")
                      + "; single_thread_value: 1 image per kernel on one thread, scaled"}


def auto_sample(layers, kernels, batch):
    """Pick the oracle sample so one measurement takes ~10-20 s on this host
    (one probe image through every kernel, then scale)."""
    per_img = oracle_sample_time(layers, kernels, 1)
    n = int(max(1, min(batch, 20.0 / max(per_img, 1e-6))))
    while batch % n:
        n -= 1
    return n


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    layers, types, kernels = select(args)
    world = int(os.environ.get("WORLD_SIZE", str(args.gpus)))
    batch = args.global_batch // world if args.global_batch else args.batch
    n_sample = args.cpu_sample or auto_sample(layers, kernels, batch)
    for _ in range(args.warmup):
        pass  # the oracle has no warm-up state; W is accepted for the contract
    times = [oracle_sample_time(layers, kernels, n_sample) for _ in range(args.steps)]
    ms = float(np.mean(times)) * 1e3 * batch / n_sample
    cb = {"value": round(ms, 3), "unit": "ms/iter", "cores": os.cpu_count(), "kind": "oracle",
          "sample": f"{n_sample} image(s) per kernel per step, x{batch // n_sample} extrapolated to N={batch}"}
    line = {"impl": "reference", "metric": METRIC, "value": round(ms, 3), "unit": "ms/iter", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 3), "higher_is_better": False,
            "scaling": "strong" if args.global_batch else "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": workload_name(args, layers, types, kernels),
                       "batch_per_gpu": batch, "math": "fp64 oracle",
                       "first_layer_backward_data": bool(args.input_grad)},
            "cpu_baseline": cb,
            "e2e": {"value": round(ms, 3), "unit": "ms/iter", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def respawn(args):
    """--gpus N > 1 outside torchrun: re-launch this script under
    torch.distributed.run with N ranks (one per GPU) and return its exit code."""
    import socket
    import subprocess
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def measure_tf32_peak(torch, dev):
    """Dense TF32 tensor-core peak on this GPU (cuBLAS fp32 matmul with TF32
    allowed, 8192^3, best of 10, CUDA events): the TF32 roofline denominator."""
    n = 8192
    a = torch.randn(n, n, device=dev)
    b = torch.randn(n, n, device=dev)
    prev = torch.backends.cuda.matmul.allow_tf32
    torch.backends.cuda.matmul.allow_tf32 = True
    try:
        for _ in range(3):
            torch.matmul(a, b)
        best = 1e30
        for _ in range(10):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            torch.matmul(a, b)
            e1.record()
            e1.synchronize()
            best = min(best, e0.elapsed_time(e1))
    finally:
        torch.backends.cuda.matmul.allow_tf32 = prev
    del a, b
    return 2.0 * n ** 3 / (best * 1e-3) / 1e12


# ------------------------------------------------------------------ our arm --
class _NoReduce:
    """grad_hook stand-in when the reduction is fused into the kernels (--grad-reduce nvls)."""

    def __call__(self, layer, dw):
        pass

    def wait(self):
        pass


def main():
    args = parse()
    if args.oracle_probe:
        layers, types, kernels = select(args)
        print(oracle_sample_time(layers, kernels, args.oracle_probe), flush=True)
        return
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(respawn(args))
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist

    import paper_conf_cluster_oyamabhm18_b200 as mu
    from paper_conf_cluster_oyamabhm18_b200.distributed import GradAllreduce, init_from_env, max_over_ranks
    from paper_conf_cluster_oyamabhm18_b200.network import ConvNet, algorithmic_bytes, algorithmic_flops

    distributed = init_from_env("nccl")
    rank = dist.get_rank() if distributed else 0
    world = dist.get_world_size() if distributed else 1
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    peaks, peaks_src = load_peaks()

    layers, types, kernels = select(args)
    if args.global_batch:
        if args.global_batch % world:
            raise SystemExit(f"--global-batch {args.global_batch} not divisible by {world} ranks")
        args.batch = args.global_batch // world
    math = MATHS[args.math]
    h = mu.Handle(local)
    h.set_policy({"pow2": mu.POLICY_POW2, "all": mu.POLICY_ALL, "undivided": mu.POLICY_UNDIVIDED}[args.policy])
    h.set_deterministic(not args.nondeterministic)
    ws_limit = int(args.ws_mib * 2 ** 20)
    net = ConvNet(h, layers, args.batch, math, device=dev, types=types)
    net.allocate(seed=rank)
    skip_c1 = not args.input_grad

    # ---- planning: benchmark pass + DP / ILP ----
    t0 = time.perf_counter()
    plan_limit = int(args.wd_mib * 2 ** 20) if args.wd_mib > 0 else ws_limit
    if not (args.tables_in and os.path.exists(args.tables_in) and net.load_tables(args.tables_in, plan_limit, args.policy)):
        net.benchmark_all(plan_limit)
        if args.tables_out and rank == 0:
            net.save_tables(args.tables_out, plan_limit, args.policy)
    bench_s = time.perf_counter() - t0
    flush = torch.empty(512 * 2 ** 20, dtype=torch.uint8, device=dev)
    grad_ar = GradAllreduce()
    if args.grad_reduce != "nccl":
        # NEXT-3: the dW sum is fused into BackwardFilter (the final dw writer adds every
        # value to all ranks' sum buffers); no per-layer collective call remains
        from paper_conf_cluster_oyamabhm18_b200.distributed import FusedGradReduce
        net.nvls = FusedGradReduce(net.dw_flat.numel(), local, kind=args.grad_reduce)
        grad_ar = _NoReduce()
    stream = torch.cuda.current_stream()

    # BackwardFilter of each layer on a side stream next to its BackwardData
    # (network.iteration concurrent=True); the evented per-op pass is sequential.
    conc = args.concurrent_wgrad

    host_ms = []  # host enqueue time of the steps of the last timed() call

    def timed(nsteps, nwarm, record_ops=False):
        ops = {}
        for _ in range(nwarm):
            net.iteration(grad_hook=grad_ar, skip_conv1_dgrad=skip_c1, concurrent=conc and not record_ops)
            grad_ar.wait()
        torch.cuda.synchronize()
        if distributed:
            dist.barrier()
        torch.cuda.synchronize()
        step_ms = []
        host_ms.clear()
        launches0 = mu._lib.launch_count()
        for _ in range(nsteps):
            flush.zero_()  # L2 flush (outside the timed events)
            ev = []

            def on_op(i, t, what):
                if record_ops:
                    e = torch.cuda.Event(enable_timing=True)
                    e.record(stream)
                    ev.append((i, t, what, e))
            s0 = torch.cuda.Event(enable_timing=True)
            s1 = torch.cuda.Event(enable_timing=True)
            s0.record(stream)
            h0 = time.perf_counter()
            net.iteration(on_op=on_op, grad_hook=grad_ar, skip_conv1_dgrad=skip_c1,
                          concurrent=conc and not record_ops)
            grad_ar.wait()
            host_ms.append((time.perf_counter() - h0) * 1e3)  # host time to enqueue the step
            s1.record(stream)
            s1.synchronize()
            step_ms.append(s0.elapsed_time(s1))
            if record_ops:
                begins = {}
                for i, t, what, e in ev:
                    if what == "begin":
                        begins[(i, t)] = e
                    else:
                        ops.setdefault((i, t), []).append(begins[(i, t)].elapsed_time(e))
        launches = mu._lib.launch_count() - launches0
        torch.cuda.synchronize()
        if distributed:
            dist.barrier()
        return float(np.mean(step_ms)), ops, launches

    # Baseline: best undivided algorithm at the same per-kernel limit,
    # timed as a whole step and per kernel; both max-reduced over the ranks.
    und_ms, und_ops = None, {}
    if args.wd_mib <= 0:
        net.plan_undivided(ws_limit)
        und_ms, _, _ = timed(max(3, args.steps // 2), args.warmup)
        und_ms = max_over_ranks(und_ms)
        _, und_ops, _ = timed(3, 1, record_ops=True)
    if args.wd_mib > 0:
        net.plan_wd(int(args.wd_mib * 2 ** 20))
    elif args.policy == "undivided":
        pass
    else:
        net.plan_wr(ws_limit)
    if os.environ.get("MUCU_PROFILE"):
        # ncu --profile-from-start off: capture exactly the timed steps, then stop.
        timed(0, args.warmup)
        torch.cuda.profiler.start()
        timed(args.steps, 0)
        torch.cuda.profiler.stop()
        print(json.dumps({"profiled_steps": args.steps, "plans": {f"{layers[i].name}/{mu.TYPE_NAMES[t]}": k.plan
                                                                  for (i, t), k in sorted(net.kernels.items())}}))
        return
    # The step is timed without per-op events: an event record between two calls
    # serialises them (no programmatic-launch overlap) and cost ~9 % of the
    # ResNet-50 step.  Per-op times come from a second, separately timed pass
    # with events around every call.
    with ClockSampler(local) as clk:
        ms, _, launches = timed(args.steps, args.warmup)
    host_enqueue_ms = float(np.mean(host_ms)) if host_ms else None
    ms_max = max_over_ranks(ms)
    ms_ops, ops, _ = timed(max(3, args.steps // 2), 1, record_ops=True)

    # ---- end to end through the public API with host buffers ----
    # The input pipeline of a training loop: step k+1's inputs (x of the first
    # layer, dy of the last) are uploaded from pinned host memory (double-buffered,
    # upload stream) while step k computes; each layer's dW is read back to the
    # host (download stream) as soon as its BackwardFilter is done (forward-only
    # workloads read back the last layer's y).  Every timed step performs its own
    # h2d_bytes / d2h_bytes of copies; the first step's upload is not hidden.
    has_bwd = any(t != 0 for t in types)
    up_names = [(0, "x")] + ([(len(layers) - 1, "dy")] if has_bwd else [])
    hosts = {key: net.tensors[key[0]][key[1]].detach().cpu().pin_memory() for key in up_names}
    bufs = {key: [net.tensors[key[0]][key[1]], torch.empty_like(net.tensors[key[0]][key[1]])] for key in up_names}
    dw_host = [torch.empty_like(t["dw"], device="cpu").pin_memory() for t in net.tensors] if 2 in types else []
    y_host = None if has_bwd else torch.empty_like(net.tensors[-1]["y"], device="cpu").pin_memory()
    up_stream, down_stream = torch.cuda.Stream(), torch.cuda.Stream()
    ready = [torch.cuda.Event(), torch.cuda.Event()]
    done = [torch.cuda.Event(), torch.cuda.Event()]

    def upload(k):
        j = k % 2
        if k >= 2:
            up_stream.wait_event(done[j])  # step k-2 has finished with these buffers
        with torch.cuda.stream(up_stream):
            for key in up_names:
                bufs[key][j].copy_(hosts[key], non_blocking=True)
            ready[j].record(up_stream)

    def e2e_op(i, t, what):
        if what == "end" and t == mu.BWD_FILTER and not distributed:  # N > 1: after the dW allreduce
            down_stream.wait_stream(torch.cuda.current_stream())  # the BackwardFilter's stream
            with torch.cuda.stream(down_stream):
                dw_host[i].copy_(net.tensors[i]["dw"], non_blocking=True)

    def e2e_run(nsteps):
        s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        s0.record(stream)
        upload(0)
        for k in range(nsteps):
            if k + 1 < nsteps:
                upload(k + 1)  # prefetch the next step's inputs while this one computes
            j = k % 2
            stream.wait_event(ready[j])
            for key in up_names:
                net.tensors[key[0]][key[1]] = bufs[key][j]
            net.iteration(on_op=e2e_op, grad_hook=grad_ar, skip_conv1_dgrad=skip_c1, concurrent=conc)
            grad_ar.wait()
            if distributed and dw_host:
                down_stream.wait_stream(stream)
                with torch.cuda.stream(down_stream):
                    for t, hbuf in zip(net.tensors, dw_host):
                        hbuf.copy_(t["dw"], non_blocking=True)
            if y_host is not None:
                down_stream.wait_stream(stream)
                with torch.cuda.stream(down_stream):
                    y_host.copy_(net.tensors[-1]["y"], non_blocking=True)
            stream.wait_stream(down_stream)  # the step's results are on the host
            done[j].record(stream)
        s1.record(stream)
        s1.synchronize()
        return s0.elapsed_time(s1) / nsteps

    e2e_run(2)  # warm-up
    torch.cuda.synchronize()
    if distributed:
        dist.barrier()
    e2e_ms = e2e_run(max(5, args.steps))
    for key in up_names:
        net.tensors[key[0]][key[1]] = bufs[key][0]
    e2e_ms = max_over_ranks(e2e_ms)
    h2d_bytes = sum(t.numel() * t.element_size() for t in hosts.values())
    d2h_bytes = sum(b.numel() * 4 for b in dw_host) + (y_host.numel() * y_host.element_size() if y_host is not None else 0)

    # ---- dominant kernel roofline ----
    op_ms = {k: float(np.median(v)) for k, v in ops.items()}  # median: robust to a one-step hiccup
    op_ms_max = {k: max_over_ranks(v) for k, v in sorted(op_ms.items())}
    und_op_ms = {k: max_over_ranks(float(np.median(v))) for k, v in sorted(und_ops.items())}
    dom = max(op_ms, key=op_ms.get)
    li, lt = dom
    kern = net.kernels[dom]
    bf16_peak = peaks.get("bf16_tflops", 1590.0)
    hbm_peak = peaks.get("hbm_gbs", 6650.0)
    elt = 2 if math == mu.MATH_BF16 else 4
    tf32_measured = None
    if math == mu.MATH_BF16:
        tpeak, tbound = bf16_peak, "tensor"
        peak_note = f"bf16 dense {peaks_src} (burst, MEASURED_PEAKS.json)"
    elif math == mu.MATH_TF32:
        tf32_measured = measure_tf32_peak(torch, dev)
        tpeak, tbound = tf32_measured, "tensor"
        peak_note = "tf32 dense measured in this run: cuBLAS fp32 matmul 8192^3 with TF32 allowed, best of 10"
    else:
        sm_mhz = peaks.get("sm_max_mhz", 1965.0)
        tpeak, tbound = 148 * 128 * 2 * sm_mhz * 1e6 / 1e12, "alu"
        peak_note = "fp32 FFMA: 148 SM x 128 lanes x 2 flop x max SM clock (DESIGN.md)"

    def floor_ms(i, t, plan):
        """Roofline floor of one op: max(F / compute peak, B / HBM peak)."""
        f = algorithmic_flops(layers[i], t, plan)
        b = algorithmic_bytes(layers[i], t, args.batch, elt)
        return max(f / (tpeak * 1e12), b / (hbm_peak * 1e9)) * 1e3, f, b

    # The dominant op is bounded by whichever of its compute / byte floors is
    # larger; achieved = that algorithmic work / the op's mean CUDA-event time.
    _, alg_flops, alg_bytes = floor_ms(li, lt, kern.plan)
    if alg_bytes / (hbm_peak * 1e9) > alg_flops / (tpeak * 1e12):
        bound, punit, peak = "hbm", "GB/s", hbm_peak
        achieved = alg_bytes / (op_ms[dom] * 1e-3) / 1e9
        peak_note = f"HBM copy bandwidth, {peaks_src} (MEASURED_PEAKS.json hbm_gbs)"
    else:
        bound, punit, peak = tbound, "TFLOP/s", tpeak
        achieved = alg_flops / (op_ms[dom] * 1e-3) / 1e12
    step_floor = sum(floor_ms(i, t, k.plan)[0] for (i, t), k in net.kernels.items() if (i, t) in op_ms)
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tp):
        try:
            tj = json.load(open(tp))
            traffic = tj.get(f"{args.config}/{args.math}/{layers[li].name}/{mu.TYPE_NAMES[lt]}")
        except Exception:
            traffic = None

    conv_flops = net.flops_per_iteration(skip_conv1_dgrad=skip_c1)
    total_ws = net.total_workspace()
    kname = lambda i, t: f"{layers[i].name}/{mu.TYPE_NAMES[t]}"  # noqa: E731
    if rank == 0:
        cb = None
        if not args.no_cpu_baseline and world == 1:
            n_sample = args.cpu_sample or auto_sample(layers, kernels, args.batch)
            cb = cpu_baseline(layers, kernels, args.batch, n_sample)
        line = {
            "metric": METRIC, "value": round(ms_max, 4), "unit": "ms/iter", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms_max, 4), "higher_is_better": False,
            "scaling": "strong" if args.global_batch else "weak", "vs_baseline": None, "dtype": args.math,
            "data": "synthetic",
            "config": {"workload": workload_name(args, layers, types, kernels),
                       "batch_per_gpu": args.batch, "global_batch": args.batch * world,
                       "policy": ("WD" if args.wd_mib > 0 else "WR"),
                       "ws_limit_mib": (args.wd_mib if args.wd_mib > 0 else args.ws_mib),
                       "batch_size_policy": args.policy, "parallelism": f"dp{world}",
                       "l2": "512 MiB buffer overwritten before every timed step",
                       "first_layer_backward_data": bool(args.input_grad),
                       "backward_streams": 2 if args.concurrent_wgrad else 1,
                       "grad_reduce": ({"nvls": "fused into the BackwardFilter epilogue: multimem.red to an NVLS "
                                                "buffer, 2 device barriers per step",
                                        "p2p": "fused into the BackwardFilter epilogue: red.global.add to every "
                                               "rank's buffer over NVLink P2P, 2 device barriers per step"}
                                       .get(args.grad_reduce) or
                                       ("async NCCL allreduce per layer" if world > 1 else "none (1 GPU)")),
                       "wgrad_reduction": ("split-K with fp32 L2 atomics (non-deterministic)" if args.nondeterministic
                                           else "ordered split-K (deterministic)")},
            "images_per_s": round(args.batch * world / (ms_max * 1e-3), 1),
            "conv_tflops_direct": round(conv_flops * world / (ms_max * 1e-3) / 1e12, 2),
            "ms_per_step_with_op_events": round(ms_ops, 4),
            "host_enqueue_ms_per_step": round(host_enqueue_ms, 4) if host_enqueue_ms is not None else None,
            "undivided_ms_per_step": round(und_ms, 4) if und_ms is not None else None,
            "speedup_vs_undivided": round(und_ms / ms_max, 4) if und_ms is not None else None,
            "speedup_by_kernel": {kname(i, t): round(und_op_ms[(i, t)] / v, 3)
                                  for (i, t), v in op_ms_max.items() if (i, t) in und_op_ms},
            "undivided_per_kernel_ms": {kname(i, t): round(v, 4) for (i, t), v in und_op_ms.items()},
            "workspace_total_mib": round(total_ws / 2 ** 20, 2),
            "wd_ilp": getattr(net, "wd_stats", None),
            "plan_time_s": round(bench_s, 2),
            "roofline": {"bound": bound, "achieved": round(achieved, 2), "peak": round(peak, 1), "unit": punit,
                         "frac": round(achieved / peak, 4), "traffic": traffic,
                         "kernel": f"{layers[li].name} {mu.TYPE_NAMES[lt]} plan="
                                   f"{[(mu.ALGO_NAMES[a], b) for a, b in kern.plan]}",
                         "algorithmic_flops": alg_flops, "algorithmic_bytes": alg_bytes,
                         "avg_ms": round(op_ms[dom], 4),
                         "share_of_step": round(op_ms[dom] / ms_ops, 4), "peak_source": peak_note,
                         "tf32_peak_measured_tflops": round(tf32_measured, 1) if tf32_measured else None,
                         "step_floor_ms": round(step_floor, 4), "step_frac": round(step_floor / ms_max, 4)},
            "cpu_baseline": cb,
            "e2e": {"value": round(e2e_ms, 4), "unit": "ms/iter", "h2d_bytes_per_step": int(h2d_bytes),
                    "d2h_bytes_per_step": int(d2h_bytes)},
            "gpu_launches": int(launches),
            "clocks": clk.result(),
            "per_kernel_ms": {kname(i, t): round(v, 4) for (i, t), v in op_ms_max.items()},
            "plans": {kname(i, t): [(mu.ALGO_NAMES[a], b) for a, b in k.plan]
                      for (i, t), k in sorted(net.kernels.items())},
        }
        if args.json_out:
            with open(args.json_out, "w") as f:
                json.dump(line, f, indent=1)
        print(json.dumps(line), flush=True)
    if distributed:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
