"""Markdown table of a measurement round's bench lines (DESIGN.md section 10 / README):
    python tools/state_table.py profiles r02c"""
import glob
import json
import os
import sys

d, rnd = sys.argv[1], sys.argv[2]
print("| config | ms/iter | best undivided | speedup | e2e | dominant op (bound, frac) | step_frac | clocks |")
print("|---|---|---|---|---|---|---|---|")
for f in sorted(glob.glob(os.path.join(d, f"{rnd}_bench_*.json"))):
    j = json.load(open(f))
    r = j.get("roofline") or {}
    c = j.get("config", {})
    name = os.path.basename(f)[len(rnd) + 7:-5]
    und = j.get("undivided_ms_per_step")
    sp = j.get("speedup_vs_undivided")
    e2e = (j.get("e2e") or {}).get("value")
    clk = j.get("clocks") or {}
    kern = (r.get("kernel") or "").split(" plan")[0]
    print(f"| {name} ({c.get('policy')} {c.get('ws_limit_mib')} MiB) | {j['value']:.3f} | "
          f"{und if und is not None else '–'} | {str(sp) + '×' if sp else '–'} | {e2e if e2e else '–'} | "
          f"{kern} ({r.get('bound')}, {r.get('frac')}) | {r.get('step_frac')} | "
          f"{clk.get('sm_mhz')} MHz {','.join(clk.get('reasons') or []) or 'ok'} |")
