"""Copy the judged summaries of one gpu_round.sh output directory into profiles/.

    python tools/make_profiles.py gpurun_out/r01c r01
Writes profiles/<round>_launches_alexnet_tf32.{csv,txt} (the ncu launch list of
`bench.py` = per-kernel share of the step), profiles/<round>_dominant_full.txt
(curated `ncu --set full` metrics + top stall lines of the dominant kernel),
profiles/<round>_bench_*.json (the bench lines) and profiles/traffic.json."""
import glob
import json
import os
import shutil
import subprocess
import sys

src, rnd = sys.argv[1], sys.argv[2]
root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
dst = os.path.join(root, "profiles")
os.makedirs(dst, exist_ok=True)
tools = os.path.join(root, "tools")


def run(*args):
    return subprocess.run([sys.executable, *args], capture_output=True, text=True).stdout


lc = os.path.join(src, "launches_alexnet_tf32.csv")
if os.path.exists(lc):
    shutil.copy(lc, os.path.join(dst, f"{rnd}_launches_alexnet_tf32.csv"))
    with open(os.path.join(dst, f"{rnd}_launches_alexnet_tf32.txt"), "w") as f:
        f.write("# ncu --metrics gpu__time_duration.sum --clock-control none, 2 timed steps of\n"
                "# `MUCU_PROFILE=1 python bench.py --steps 2 --warmup 3` (AlexNet TF32, default config).\n"
                "# Cold-cache, serialised per-launch times: compare SHARES with bench.py per_kernel_ms.\n")
        f.write(run(os.path.join(tools, "ncu_summary.py"), "launches", lc))
rep = os.path.join(src, "dominant_full.ncu-rep")
if os.path.exists(rep):
    status = open(os.path.join(src, "status")).read() if os.path.exists(os.path.join(src, "status")) else ""
    dom = [l for l in status.splitlines() if l.startswith("dominant")]
    with open(os.path.join(dst, f"{rnd}_dominant_full.txt"), "w") as f:
        f.write("# ncu --set full --clock-control none --import-source on, first tc_conv_gemm launch of the\n"
                f"# dominant op of the AlexNet TF32 bench step ({dom[0] if dom else '?'})\n")
        f.write(run(os.path.join(tools, "ncu_summary.py"), "full", rep))
        f.write("\n\n# warp-stall samples by source line\n")
        f.write(run(os.path.join(tools, "ncu_lines.py"), rep, "15"))
for b in glob.glob(os.path.join(src, "bench_*.json")):
    shutil.copy(b, os.path.join(dst, f"{rnd}_{os.path.basename(b)}"))
for t in sorted(glob.glob(os.path.join(src, "ops", "*.txt"))):
    shutil.copy(t, os.path.join(dst, f"{rnd}_ops_{os.path.basename(t)}"))
for extra in ("status", "tests.log", "gpu.txt"):
    if os.path.exists(os.path.join(src, extra)):
        shutil.copy(os.path.join(src, extra), os.path.join(dst, f"{rnd}_{extra.replace('.log', '')}.txt"))
tj = os.path.join(src, "traffic.json")
if os.path.exists(tj):
    shutil.copy(tj, os.path.join(dst, "traffic.json"))
print(sorted(os.listdir(dst)))
