"""bench.py -- conv fwd+bwd ms/iter of micro-batched plans vs the best undivided
algorithm at the same workspace (BASELINE.json metric), on B200.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
                    [--config alexnet|resnet18|resnet50] [--math tf32|bf16|f32]
                    [--policy pow2|all|undivided] [--ws-mib 64] [--wd-mib T] [--batch 256]

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
    ap.add_argument("--no-input-grad", dest="input_grad", action="store_false",
                    help="skip the first layer's BackwardData (the data layer needs no gradient, as in "
                         "Caffe's `time` command, P:L198); the default times all 3 kernels per layer (SURVEY 8(d) cfg2)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-concurrent-wgrad", dest="concurrent_wgrad", action="store_false",
                    help="run each BackwardFilter after its BackwardData on one stream")
    ap.add_argument("--cpu-sample", type=int, default=0, help="oracle sample (images per kernel); 0 = auto")
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


# --------------------------------------------------------------- oracle arm --
def oracle_sample_time(layers, n_sample, threads=None, input_grad=True):
    """Time the fp64 oracle (oracle/, unchanged) on n_sample images of every
    kernel of the iteration (the first layer's BackwardData only if
    input_grad); returns seconds."""
    import oracle
    from synthetic import conv_inputs
    if threads:
        os.environ["OMP_NUM_THREADS"] = str(threads)
    oracle.build()
    tot = 0.0
    for i, l in enumerate(layers):
        x, w, dy = conv_inputs(n_sample, l.c, l.h, l.w, l.k, l.r, l.s, l.pad, l.stride, seed=i)
        x, w, dy = x.astype(np.float64), w.astype(np.float64), dy.astype(np.float64)
        t0 = time.perf_counter()
        oracle.conv_forward(x, w, l.pad, l.stride)
        if i > 0 or input_grad:
            oracle.conv_backward_data(dy, w, l.h, l.w, l.pad, l.stride)
        oracle.conv_backward_filter(x, dy, l.r, l.s, l.pad, l.stride)
        tot += time.perf_counter() - t0
    return tot


def n_kernels(layers, input_grad):
    return 3 * len(layers) - (0 if input_grad else 1)


def cpu_baseline(layers, batch, n_sample, input_grad=True):
    cores = os.cpu_count()
    secs = oracle_sample_time(layers, n_sample, input_grad=input_grad)
    ms_per_iter = secs * 1e3 * batch / n_sample
    return {"value": round(ms_per_iter, 3), "unit": "ms/iter", "cores": cores, "kind": "oracle",
            "sample": f"{n_sample} image(s) per kernel, all {n_kernels(layers, input_grad)} timed kernels, fp64 7-loop oracle, "
                      f"{secs:.2f} s measured, x{batch // n_sample} extrapolated to N={batch} (work is linear in N, P:L50)"}


def auto_sample(layers, batch, input_grad=True):
    """Pick the oracle sample so one measurement takes ~10-20 s on this host
    (one probe image through every kernel, then scale)."""
    per_img = oracle_sample_time(layers, 1, input_grad=input_grad)
    n = int(max(1, min(batch, 20.0 / max(per_img, 1e-6))))  # powers of two below: ~10-20 s
    while batch % n:
        n -= 1
    return n


def run_reference(args):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    from synthetic import network
    layers = network(args.config)
    n_sample = args.cpu_sample or auto_sample(layers, args.batch, args.input_grad)
    for _ in range(args.warmup):
        pass  # the oracle has no warm-up state; W is accepted for the contract
    times = [oracle_sample_time(layers, n_sample, input_grad=args.input_grad) for _ in range(args.steps)]
    ms = float(np.mean(times)) * 1e3 * args.batch / n_sample
    cb = {"value": round(ms, 3), "unit": "ms/iter", "cores": os.cpu_count(), "kind": "oracle",
          "sample": f"{n_sample} image(s) per kernel per step, x{args.batch // n_sample} extrapolated to N={args.batch}"}
    line = {"impl": "reference", "metric": METRIC, "value": round(ms, 3), "unit": "ms/iter", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 3), "higher_is_better": False,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"{args.config} conv layers fwd+bwd ({n_kernels(layers, args.input_grad)} kernels)",
                       "batch_per_gpu": args.batch, "math": "fp64 oracle",
                       "first_layer_backward_data": bool(args.input_grad)},
            "cpu_baseline": cb,
            "e2e": {"value": round(ms, 3), "unit": "ms/iter", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ our arm --
def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist

    import paper_conf_cluster_oyamabhm18_b200 as mu
    from paper_conf_cluster_oyamabhm18_b200.distributed import GradAllreduce, init_from_env, max_over_ranks
    from paper_conf_cluster_oyamabhm18_b200.network import ConvNet, algorithmic_bytes, algorithmic_flops, layer_flops
    from synthetic import network

    distributed = init_from_env("nccl")
    rank = dist.get_rank() if distributed else 0
    world = dist.get_world_size() if distributed else 1
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    peaks, peaks_src = load_peaks()

    layers = network(args.config)
    math = MATHS[args.math]
    h = mu.Handle(local)
    h.set_policy({"pow2": mu.POLICY_POW2, "all": mu.POLICY_ALL, "undivided": mu.POLICY_UNDIVIDED}[args.policy])
    ws_limit = int(args.ws_mib * 2 ** 20)
    net = ConvNet(h, layers, args.batch, math, device=dev)
    net.allocate(seed=rank)

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
    stream = torch.cuda.current_stream()

    # BackwardFilter of each layer on a side stream next to its BackwardData
    # (network.iteration concurrent=True); the evented per-op pass is sequential.
    conc = args.concurrent_wgrad

    def timed(nsteps, nwarm, record_ops=False):
        ops = {}
        for _ in range(nwarm):
            net.iteration(grad_hook=grad_ar, skip_conv1_dgrad=not args.input_grad, concurrent=conc and not record_ops)
            grad_ar.wait()
        torch.cuda.synchronize()
        if distributed:
            dist.barrier()
        torch.cuda.synchronize()
        step_ms = []
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
            net.iteration(on_op=on_op, grad_hook=grad_ar, skip_conv1_dgrad=not args.input_grad,
                          concurrent=conc and not record_ops)
            grad_ar.wait()
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

    results = {}
    # Baseline: best undivided algorithm at the same per-kernel limit.
    if args.wd_mib <= 0:
        net.plan_undivided(ws_limit)
        und_ms, _, _ = timed(max(3, args.steps // 2), args.warmup)
        results["undivided"] = und_ms
        und_plans = {k: list(v.plan) for k, v in net.kernels.items()}
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
    # ResNet-50 step (tools/graph_probe.py).  Per-op times come from a second,
    # separately timed pass with events around every call.
    with ClockSampler(local) as clk:
        ms, _, launches = timed(args.steps, args.warmup)
    ms_max = max_over_ranks(ms)
    ms_ops, ops, _ = timed(max(3, args.steps // 2), 1, record_ops=True)

    # ---- end to end through the public API with host buffers ----
    x_host = net.tensors[0]["x"].detach().cpu().pin_memory()
    dy_host = net.tensors[-1]["dy"].detach().cpu().pin_memory()
    dw_host = [torch.empty_like(t["dw"], device="cpu").pin_memory() for t in net.tensors]

    # The input pipeline of a training loop: step k+1's x and dy are uploaded from
    # pinned host memory (double-buffered, on an upload stream) while step k
    # computes, and each layer's dW is read back to the host (download stream)
    # as soon as its BackwardFilter is done.  Every timed step performs its own
    # h2d_bytes / d2h_bytes of copies; the first step's upload is not hidden.
    up_stream, down_stream = torch.cuda.Stream(), torch.cuda.Stream()
    x_bufs = [net.tensors[0]["x"], torch.empty_like(net.tensors[0]["x"])]
    dy_bufs = [net.tensors[-1]["dy"], torch.empty_like(net.tensors[-1]["dy"])]
    ready = [torch.cuda.Event(), torch.cuda.Event()]
    done = [torch.cuda.Event(), torch.cuda.Event()]

    def upload(k):
        j = k % 2
        if k >= 2:
            up_stream.wait_event(done[j])  # step k-2 has finished with these buffers
        with torch.cuda.stream(up_stream):
            x_bufs[j].copy_(x_host, non_blocking=True)
            dy_bufs[j].copy_(dy_host, non_blocking=True)
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
            net.tensors[0]["x"], net.tensors[-1]["dy"] = x_bufs[j], dy_bufs[j]
            net.iteration(on_op=e2e_op, grad_hook=grad_ar, skip_conv1_dgrad=not args.input_grad,
                          concurrent=conc)
            grad_ar.wait()
            if distributed:
                down_stream.wait_stream(stream)
                with torch.cuda.stream(down_stream):
                    for t, hbuf in zip(net.tensors, dw_host):
                        hbuf.copy_(t["dw"], non_blocking=True)
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
    net.tensors[0]["x"], net.tensors[-1]["dy"] = x_bufs[0], dy_bufs[0]
    e2e_ms = max_over_ranks(e2e_ms)
    h2d_bytes = x_host.numel() * x_host.element_size() + dy_host.numel() * dy_host.element_size()
    d2h_bytes = sum(b.numel() * 4 for b in dw_host)

    # ---- dominant kernel roofline ----
    op_ms = {k: float(np.median(v)) for k, v in ops.items()}  # median: robust to a one-step hiccup
    dom = max(op_ms, key=op_ms.get)
    li, lt = dom
    kern = net.kernels[dom]
    bf16_peak = peaks.get("bf16_tflops", 1590.0)
    hbm_peak = peaks.get("hbm_gbs", 6650.0)
    elt = 2 if math == mu.MATH_BF16 else 4
    if math == mu.MATH_BF16:
        tpeak, tbound = bf16_peak, "tensor"
        peak_note = f"bf16 dense {peaks_src} (burst)"
    elif math == mu.MATH_TF32:
        tpeak, tbound = bf16_peak * 0.5, "tensor"
        peak_note = f"tf32 = {peaks_src} bf16 burst x nominal tf32/bf16 ratio 1.125/2.25"
    else:
        sm_mhz = peaks.get("sm_max_mhz", 1965.0)
        tpeak, tbound = 148 * 128 * 2 * sm_mhz * 1e6 / 1e12, "alu"
        peak_note = "fp32 FFMA: 148 SM x 128 lanes x 2 flop x max SM clock"

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

    conv_flops = net.flops_per_iteration(skip_conv1_dgrad=not args.input_grad)
    total_ws = net.total_workspace()
    if rank == 0:
        cb = None
        if not args.no_cpu_baseline and world == 1:
            n_sample = args.cpu_sample or auto_sample(layers, args.batch, args.input_grad)
            cb = cpu_baseline(layers, args.batch, n_sample, args.input_grad)
        line = {
            "metric": METRIC, "value": round(ms_max, 4), "unit": "ms/iter", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms_max, 4), "higher_is_better": False,
            "scaling": "weak", "vs_baseline": None, "dtype": args.math, "data": "synthetic",
            "config": {"workload": f"{args.config} conv layers fwd+bwd ({n_kernels(layers, args.input_grad)} kernels)",
                       "batch_per_gpu": args.batch, "global_batch": args.batch * world,
                       "policy": ("WD" if args.wd_mib > 0 else "WR"),
                       "ws_limit_mib": (args.wd_mib if args.wd_mib > 0 else args.ws_mib),
                       "batch_size_policy": args.policy, "parallelism": f"dp{world}",
                       "l2": "512 MiB buffer overwritten before every timed step",
                       "first_layer_backward_data": bool(args.input_grad),
                       "backward_streams": 2 if args.concurrent_wgrad else 1},
            "images_per_s": round(args.batch * world / (ms_max * 1e-3), 1),
            "conv_tflops_direct": round(conv_flops / (ms_max * 1e-3) / 1e12, 2),
            "ms_per_step_with_op_events": round(ms_ops, 4),
            "undivided_ms_per_step": round(results["undivided"], 4) if "undivided" in results else None,
            "speedup_vs_undivided": round(results["undivided"] / ms, 4) if "undivided" in results else None,
            "workspace_total_mib": round(total_ws / 2 ** 20, 2),
            "plan_time_s": round(bench_s, 2),
            "roofline": {"bound": bound, "achieved": round(achieved, 2), "peak": round(peak, 1), "unit": punit,
                         "frac": round(achieved / peak, 4), "traffic": traffic,
                         "kernel": f"{layers[li].name} {mu.TYPE_NAMES[lt]} plan="
                                   f"{[(mu.ALGO_NAMES[a], b) for a, b in kern.plan]}",
                         "algorithmic_flops": alg_flops, "algorithmic_bytes": alg_bytes,
                         "avg_ms": round(op_ms[dom], 4),
                         "share_of_step": round(op_ms[dom] / ms_ops, 4), "peak_source": peak_note,
                         "step_floor_ms": round(step_floor, 4), "step_frac": round(step_floor / ms, 4)},
            "cpu_baseline": cb,
            "e2e": {"value": round(e2e_ms, 4), "unit": "ms/iter", "h2d_bytes_per_step": int(h2d_bytes),
                    "d2h_bytes_per_step": int(d2h_bytes)},
            "gpu_launches": int(launches),
            "clocks": clk.result(),
            "per_kernel_ms": {f"{layers[i].name}/{mu.TYPE_NAMES[t]}": round(v, 4) for (i, t), v in sorted(op_ms.items())},
            "plans": {f"{layers[i].name}/{mu.TYPE_NAMES[t]}": [(mu.ALGO_NAMES[a], b) for a, b in k.plan]
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
