#!/bin/bash
set -u
timeout 900 python -m pytest tests -q -m gpu -x 2>&1 | tail -1
for c in "resnet50 bf16" "resnet18 bf16"; do set -- $c; timeout 300 python bench.py --config $1 --math $2 --no-cpu-baseline --tables-in scratch/tables_$1_$2.npz 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['workload'], d['value'], d['e2e']['value'], d['roofline']['frac'], d['roofline']['step_frac'], d['clocks']['reasons'])"; done
