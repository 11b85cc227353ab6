"""Per-kernel summary of an ncu report with several launches (tools/prof_ops.sh).

    python tools/ncu_ops.py REP.ncu-rep [top_stall_lines [kernel_regex]]
"""
import csv, io, subprocess, sys

rep = sys.argv[1]
KEYS = [("gpu__time_duration.sum", "us", 1e-3), ("dram__bytes_read.sum", "MB", 1e-6), ("dram__bytes_write.sum", "MB", 1e-6),
                ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed", "%tc", 1),
        ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "%lts", 1),
        ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "%dram", 1),
        ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "%sm", 1),
        ("sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active", "%fma", 1),
        ("smsp__issue_active.avg.pct_of_peak_sustained_active", "%issue", 1),
        ("launch__grid_size", "grid", 1), ("launch__registers_per_thread", "regs", 1)]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rr = list(csv.reader(io.StringIO(raw)))
hdr, units = rr[0], rr[1]
for row in rr[2:]:
    d = dict(zip(hdr, row))
    name = d.get("Kernel Name", "?")[:70]
    out = []
    for k, lab, sc in KEYS:
        if k not in d:
            continue
        v = float(d[k].replace(",", "") or 0)
        u = units[hdr.index(k)]
        if lab in ("us",) and u == "nsecond":
            v = v * 1e-3
        elif lab in ("us",) and u == "usecond":
            pass
        elif lab == "MB":
            v = v * {"byte": 1e-6, "Kbyte": 1e-3, "Mbyte": 1, "Gbyte": 1e3}.get(u, 1e-6)
        out.append(f"{lab}={v:.1f}")
    print(f"{name:70s} " + " ".join(out))
if len(sys.argv) > 2:
    import os
    # stall samples per CUDA line of the first launch matching kernel_regex (default tc_conv) (tools/ncu_lines.py logic)
    from collections import defaultdict
    txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                          "-k", "regex:" + (sys.argv[3] if len(sys.argv) > 3 else "tc_conv"), "-c", "1"], capture_output=True, text=True).stdout
    agg, srcs, fname, header = defaultdict(float), {}, "?", None
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
        agg[(fname, int(row[0]))] += v
        srcs.setdefault((fname, int(row[0])), row[1].strip()[:100])
    tot = sum(agg.values()) or 1
    for key, v in sorted(agg.items(), key=lambda kv: -kv[1])[:int(sys.argv[2])]:
        print(f"{v / tot * 100:5.1f}%  {key[0]}:{key[1]}  {srcs[key]}")
