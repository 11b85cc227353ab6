#!/bin/bash
set -u
timeout 900 python -m pytest tests/test_conv_gpu.py tests/test_tilings_gpu.py -q -x -k "c3 or c2 or 7x7" 2>&1 | tail -2
for v in 0 1; do echo "== WIN_BOX=$v"
MUCU_WIN_BOX=$v timeout 120 python tools/time_one.py --config alexnet --math tf32 --specs conv1:WGRAD:I2C:64
MUCU_WIN_BOX=$v timeout 120 python tools/time_one.py --config alexnet --math bf16 --specs conv1:WGRAD:I2C:128
MUCU_WIN_BOX=$v timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs conv1:WGRAD:I2C:128
done
