#!/bin/bash
set -u
timeout 900 python -m pytest tests -q -m gpu -x 2>&1 | tail -1
for c in "alexnet tf32" "alexnet bf16" "resnet18 bf16" "resnet50 bf16"; do set -- $c; timeout 300 python bench.py --config $1 --math $2 --no-cpu-baseline --tables-in scratch/tables_$1_$2.npz 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['workload'], d['value'], d['undivided_ms_per_step'], d['e2e']['value'], d['gpu_launches'], d['roofline']['frac'], d['clocks']['reasons'])"; done
