#!/bin/bash
set -u
timeout 900 python -m pytest tests -q -m gpu -x 2>&1 | tail -1
source tools/specs.sh
SPP="layer1.0.conv1:WGRAD:I2C:256 layer2.0.conv3:WGRAD:I2C:256 layer2.1.conv1:WGRAD:I2C:256 layer3.0.conv3:WGRAD:I2C:256 layer3.1.conv1:WGRAD:I2C:256 layer4.0.conv3:WGRAD:I2C:256 layer4.1.conv1:WGRAD:I2C:256 layer1.1.conv1:DGRAD:I2C:256 layer2.1.conv1:DGRAD:I2C:256 layer3.1.conv1:DGRAD:I2C:256 layer4.1.conv1:DGRAD:I2C:256 layer4.2.conv3:DGRAD:I2C:256"
for env in "MUCU_B_BOX=0" "MUCU_B_BOX=1"; do echo "== $env"
env $env timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs $SPP
done
