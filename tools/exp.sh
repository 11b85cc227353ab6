#!/bin/bash
set -u
timeout 900 python -m pytest tests -q -m gpu -x 2>&1 | tail -1
SP="layer1.0.conv3:FWD:I2C:256 layer1.1.conv1:FWD:I2C:256 layer2.0.conv3:FWD:I2C:256 layer3.0.conv3:FWD:I2C:256 layer1.1.conv1:DGRAD:I2C:256 layer1.0.conv3:DGRAD:I2C:256 layer2.1.conv1:DGRAD:I2C:256 layer3.2.conv1:DGRAD:I2C:256"
for env in "MUCU_A_MERGE=0" "MUCU_A_MERGE=1" "MUCU_A_MERGE=0" "MUCU_A_MERGE=1"; do echo "== $env"
env $env timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs $SP
done
