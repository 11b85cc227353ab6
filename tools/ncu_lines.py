"""Warp-stall samples per CUDA source line of an ncu report (cuda,sass view).

    python tools/ncu_lines.py REPORT.ncu-rep [top]"""
import csv
import io
import subprocess
import sys
from collections import defaultdict

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 20
txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
agg = defaultdict(float)
srcs = {}
fname = "?"
header = None
for row in csv.reader(io.StringIO(txt)):
    if not row:
        continue
    if row[0] == "File Path":
        fname = row[1].split("/")[-1]
        continue
    if row[0] == "Line No":
        header = row
        continue
    if header is None or len(row) < 5 or not row[0].isdigit():
        continue
    try:
        v = float(row[4] or 0)
    except ValueError:
        continue
    key = (fname, int(row[0]))
    agg[key] += v
    srcs.setdefault(key, row[1].strip()[:100])
tot = sum(agg.values()) or 1
for key, v in sorted(agg.items(), key=lambda kv: -kv[1])[:top]:
    print(f"{v / tot * 100:5.1f}%  {key[0]}:{key[1]}  {srcs[key]}")
