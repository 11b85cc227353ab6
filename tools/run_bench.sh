timeout -s KILL 600 python -m pytest tests -q -m gpu -x 2>&1 | tail -2
timeout -s KILL 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --tables-in gpurun_out/tables_alexnet_tf32.npz --json-out gpurun_out/bench.json > gpurun_out/b.log 2>&1
python - <<'PY'
import json; d=json.load(open("gpurun_out/bench.json")); print("ms", d["value"], "undiv", d["undivided_ms_per_step"], "frac", d["roofline"]["frac"], d["roofline"]["kernel"][:40])
print(d["per_kernel_ms"])
PY
