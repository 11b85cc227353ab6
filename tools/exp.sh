#!/bin/bash
set -u
timeout 900 python -m pytest tests -q -m gpu -x 2>&1 | tail -1
SP="layer1.0.conv2:FWD:IG:256 layer1.0.conv2:DGRAD:IG:256 layer2.1.conv2:FWD:IG:256 layer2.0.conv2:DGRAD:IG:256 conv1:DGRAD:I2C:256 conv1:FWD:I2C:128 layer1.0.conv1:FWD:IG:256"
for env in "MUCU_A_MERGE=0" "MUCU_A_MERGE=1" "MUCU_A_MERGE=0" "MUCU_A_MERGE=1"; do echo "== $env"
env $env timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs $SP
env $env timeout 120 python tools/time_one.py --config alexnet --math tf32 --specs conv2:DGRAD:IG:256 conv3:DGRAD:IG:256 conv1:DGRAD:I2C:256 conv1:FWD:I2C:64
done
