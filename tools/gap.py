"""Per-kernel gap to the roofline floor from a bench JSON line (analysis aid).

    python tools/gap.py gpurun_out/r01c/bench_resnet50_bf16.json [--top 30]

floor(kernel) = max(F / peak, bytes / BW), F = 2 N K C R S P Q, bytes = the
operands the op must touch once (x + w + y, dW fp32).  Sorted by ms - floor.
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from synthetic.networks import alexnet, resnet18, resnet50  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("json")
ap.add_argument("--top", type=int, default=30)
a = ap.parse_args()
d = json.load(open(a.json))
cfg = d["config"]["workload"].split()[0].lower()
net = {"alexnet": alexnet, "resnet18": resnet18, "resnet-18": resnet18, "resnet50": resnet50,
       "resnet-50": resnet50}[cfg.replace(",", "")]()
n = d["config"]["batch_per_gpu"]
elt = 2 if d["dtype"] == "bf16" else 4
_mp = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")
_pk = json.load(open(_mp)) if os.path.exists(_mp) else {}
_bf16 = _pk.get("bf16_tflops", 1614.0) * 1e12
peak = _bf16 if d["dtype"] == "bf16" else (_bf16 / 2 if d["dtype"] == "tf32" else 74e12)
bw = _pk.get("hbm_gbs", 6500.0) * 1e9
rows = []
for L in net:
    for t in ("FWD", "DGRAD", "WGRAD"):
        key = f"{L.name}/{t}"
        if key not in d["per_kernel_ms"]:
            continue
        ms = d["per_kernel_ms"][key]
        F = L.flops(n)
        xb = n * L.h * L.w * L.c * elt
        yb = n * L.p * L.q * L.k * elt
        wb = L.k * L.r * L.s * L.c * (4 if t == "WGRAD" else elt)
        floor = max(F / peak, (xb + yb + wb) / bw) * 1e3
        rows.append((ms - floor, key, ms, floor, F / (ms * 1e-3) / 1e12, d.get("plans", {}).get(key)))
rows.sort(reverse=True)
tot = sum(r[2] for r in rows)
fl = sum(r[3] for r in rows)
print(f"total {tot:.3f} ms  floor {fl:.3f} ms  ({fl / tot:.1%})")
for g, k, ms, f, tf, pl in rows[:a.top]:
    print(f"{k:28s} {ms:7.4f} floor {f:7.4f} gap {g:7.4f}  {tf:6.0f} TF/s  {pl}")
