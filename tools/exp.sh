#!/bin/bash
set -u
timeout 900 python -m pytest tests -q -m gpu -x 2>&1 | tail -2
timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs layer1.0.conv2:FWD:IG:256 layer1.0.conv2:DGRAD:IG:256 layer1.0.conv2:WGRAD:IG:256 layer3.1.conv2:FWD:IG:256 conv1:WGRAD:I2C:128 conv1:FWD:I2C:128 conv1:DGRAD:I2C:256 layer4.1.conv1:WGRAD:I2C:256
timeout 120 python tools/time_one.py --config alexnet --math tf32 --specs conv1:WGRAD:I2C:64 conv2:DGRAD:IG:256 conv2:WGRAD:IG:256 conv2:FWD:IG:256
for c in "resnet50 bf16" "alexnet tf32" "resnet18 bf16" "alexnet bf16"; do set -- $c; timeout 300 python bench.py --config $1 --math $2 --no-cpu-baseline --tables-in scratch/tables_$1_$2.npz 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print(d['config']['workload'], d['value'], d['undivided_ms_per_step'], d['e2e']['value'], d['roofline']['frac'], d['roofline']['step_frac'], d['clocks']['reasons'])"; done
