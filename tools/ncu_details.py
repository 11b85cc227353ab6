"""Print key 'details' metrics and the top stall SASS lines of an ncu report."""
import csv, io, subprocess, sys
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(out)))
h = r[0]
for row in r[1:]:
    d = dict(zip(h, row))
    n = d.get('Metric Name', '')
    if any(k in n for k in ['Duration', 'Throughput', 'Hit Rate', 'Achieved Occupancy', 'Eligible', 'Warp Cycles Per Issued', 'Issue Slots']):
        print(f"{n} = {d.get('Metric Value')} {d.get('Metric Unit')}")
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rr = list(csv.reader(io.StringIO(raw)))
if len(rr) > 2:
    d = dict(zip(rr[0], rr[2]))
    for k in rr[0]:
        if k in ("dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum") or ("pipe_tensor" in k and "pct_of_peak_sustained_elapsed" in k and k.endswith("avg.pct_of_peak_sustained_elapsed")):
            print(f"{k} = {d[k]} {rr[1][rr[0].index(k)]}")
if len(sys.argv) > 2:
    src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(src)))
    hh = rows[1]
    data = [dict(zip(hh, x)) for x in rows[2:]]
    col = 'Warp Stall Sampling (All Samples)'
    tot = sum(float(x[col] or 0) for x in data) or 1
    for x in sorted(data, key=lambda x: -float(x[col] or 0))[:int(sys.argv[2])]:
        print(f"{float(x[col]) / tot * 100:5.1f}%  {x['Source'][:80]}  ex={x['Instructions Executed']}")
