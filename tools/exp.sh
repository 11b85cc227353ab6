#!/bin/bash
for c in "resnet50 bf16" "alexnet tf32" "resnet18 bf16" "alexnet bf16"; do set -- $c; echo "== $1 $2"
timeout 300 python tools/graph_probe.py --config $1 --math $2 --tables scratch/tables_$1_$2.npz 2>&1 | tail -6
done
