#!/bin/bash
set -u
source tools/specs.sh
for env in "MUCU_SPLIT_WAVES=0" "MUCU_SPLIT_WAVES=1" "MUCU_SPLIT_E=8" "MUCU_SPLIT_E=32" "MUCU_SPLIT_E=16 MUCU_KM=1"; do echo "== $env"
env $env timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs $SP_resnet50
env $env timeout 120 python tools/time_one.py --config alexnet --math tf32 --specs $SP_alexnet
done
