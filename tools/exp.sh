#!/bin/bash
set -u
timeout 900 python -m pytest tests -q -m gpu -x 2>&1 | tail -2
for rep in 1 2; do for pdl in 0 1; do
  for cfg in "resnet50 bf16" "alexnet tf32"; do set -- $cfg
  MUCU_PDL=$pdl timeout 300 python bench.py --config $1 --math $2 --no-cpu-baseline --tables-in scratch/tables_$1_$2.npz --steps 20 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.readlines()[-1]); print('PDL=$pdl $1 $2', d['value'], d['e2e']['value'], d['roofline']['step_frac'], d['clocks']['reasons'])"
  done
done; done
