#!/bin/bash
set -u
timeout 900 python -m pytest tests -q -m gpu -x 2>&1 | tail -1
for env in "MUCU_WIN_KM1=0" "MUCU_WIN_KM1=1"; do echo "== $env"
env $env timeout 60 python tools/time_one.py --config resnet50 --math bf16 --specs conv1:WGRAD:I2C:128
env $env timeout 60 python tools/time_one.py --config alexnet --math bf16 --specs conv1:WGRAD:I2C:128
done
