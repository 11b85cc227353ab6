"""Run one (layer, conv type, plan) call under cudaProfilerStart/Stop so that
`ncu --profile-from-start off` captures exactly its kernels.

    python tools/profile_one.py --config alexnet --layer conv2 --type FWD --algo IG --b 256 --math tf32
"""
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
ap.add_argument("--layer", default="conv2")
ap.add_argument("--type", default="FWD", choices=["FWD", "DGRAD", "WGRAD"])
ap.add_argument("--algo", default="IG", choices=["IG", "I2C", "WG", "FFT", "FFTT"])
ap.add_argument("--b", type=int, default=256)
ap.add_argument("--n", type=int, default=256)
ap.add_argument("--math", default="tf32", choices=["f32", "tf32", "bf16"])
ap.add_argument("--reps", type=int, default=1)
a = ap.parse_args()

layer = [l for l in network(a.config) if l.name == a.layer][0]
math = {"f32": 0, "tf32": 1, "bf16": 2}[a.math]
ctype = {"FWD": 0, "DGRAD": 1, "WGRAD": 2}[a.type]
algo = {"IG": 0, "I2C": 1, "WG": 2, "FFT": 3, "FFTT": 4}[a.algo]
h = mu.Handle(0)
d = mu.desc(a.n, layer.c, layer.h, layer.w, layer.k, layer.r, layer.s, layer.pad, layer.stride, math)
dt = torch.bfloat16 if math == 2 else torch.float32
x, w, dy = torch_conv_inputs(layer, a.n, 0, "cuda", dt)
plan = [(algo, a.b)] * (a.n // a.b)
ws_bytes = T.plan_workspace(d, ctype, plan)
ws = torch.empty(max(ws_bytes, 256), dtype=torch.uint8, device="cuda")
args = {0: (x, w), 1: (dy, w), 2: (x, dy)}[ctype]
for _ in range(3):
    T.run(h, d, ctype, plan, *args, workspace=ws)
torch.cuda.synchronize()
torch.cuda.profiler.start()
for _ in range(a.reps):
    T.run(h, d, ctype, plan, *args, workspace=ws)
torch.cuda.synchronize()
torch.cuda.profiler.stop()
print("profiled", a)
