#!/bin/bash
set -u
source tools/specs.sh
for env in "MUCU_A_BOX=0" "MUCU_A_BOX=1" "MUCU_A_BOX=0" "MUCU_A_BOX=1"; do echo "== $env"
env $env timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs $SP_resnet50
env $env timeout 120 python tools/time_one.py --config alexnet --math bf16 --specs $SP_alexnet
done
