#!/bin/bash
set -u
timeout 900 python -m pytest tests/test_conv_gpu.py tests/test_tilings_gpu.py -q -x -k "c3 or c2 or 7x7" 2>&1 | tail -2
for v in 0 1; do echo "== EXACT_N=$v"
MUCU_D2S_EXACT_N=$v timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs conv1:DGRAD:I2C:256
MUCU_D2S_EXACT_N=$v timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs conv1:DGRAD:I2C:256
done
