"""Time one (layer, conv type, algorithm, micro-batch) call with CUDA events.

    python tools/time_one.py --config alexnet --layer conv2 --type WGRAD --algo IG --b 256 --math tf32
Prints ms per call and achieved direct-conv TFLOP/s; several --layer/--type
pairs may be given as layer:type:algo:b specs via --specs."""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_cluster_oyamabhm18_b200 as mu  # noqa: E402
from paper_conf_cluster_oyamabhm18_b200 import torch_api as T  # noqa: E402
from synthetic import network, torch_conv_inputs  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="alexnet")
ap.add_argument("--math", default="tf32")
ap.add_argument("--n", type=int, default=256)
ap.add_argument("--specs", nargs="+", default=["conv2:WGRAD:IG:256"])
ap.add_argument("--reps", type=int, default=10)
a = ap.parse_args()
math = {"f32": 0, "tf32": 1, "bf16": 2}[a.math]
dt = torch.bfloat16 if math == 2 else torch.float32
h = mu.Handle(0)
layers = {l.name: l for l in network(a.config)}
for spec in a.specs:
    name, ty, al, b = spec.split(":")
    layer = layers[name]
    ctype = {"FWD": 0, "DGRAD": 1, "WGRAD": 2}[ty]
    algo = {"IG": 0, "I2C": 1, "WG": 2, "FFT": 3, "FFTT": 4}[al]
    b = int(b)
    d = mu.desc(a.n, layer.c, layer.h, layer.w, layer.k, layer.r, layer.s, layer.pad, layer.stride, math)
    x, w, dy = torch_conv_inputs(layer, a.n, 0, "cuda", dt)
    plan = [(algo, b)] * (a.n // b)
    ws = torch.empty(max(T.plan_workspace(d, ctype, plan), 256), dtype=torch.uint8, device="cuda")
    args = {0: (x, w), 1: (dy, w), 2: (x, dy)}[ctype]
    for _ in range(3):
        T.run(h, d, ctype, plan, *args, workspace=ws)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(a.reps):
        T.run(h, d, ctype, plan, *args, workspace=ws)
    e1.record()
    e1.synchronize()
    ms = e0.elapsed_time(e1) / a.reps
    fl = layer.flops(a.n)
    print(f"{spec:28s} {ms:8.4f} ms  {fl / ms / 1e9:8.1f} TFLOP/s(direct)", flush=True)
