#!/bin/bash
set -u
timeout 900 python -m pytest tests/test_conv_gpu.py tests/test_tilings_gpu.py -q -x -k "s2 or 1x1" 2>&1 | tail -2
timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs layer2.0.downsample:DGRAD:IG:256 layer3.0.downsample:DGRAD:IG:256 layer4.0.downsample:DGRAD:IG:256
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off \
  python tools/profile_one.py --config resnet50 --math bf16 --layer layer3.0.downsample --type DGRAD --algo IG --b 256 --n 256 2>&1 | grep -E "zero_tapless|tc_conv|duration"
