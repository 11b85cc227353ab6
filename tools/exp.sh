#!/bin/bash
set -u
timeout 900 python -m pytest tests/test_conv_gpu.py tests/test_tilings_gpu.py -q -x -k "c3 or c2 or 7x7" 2>&1 | tail -2
for spec in "alexnet tf32 64 FWD" "alexnet tf32 64 WGRAD" "resnet50 bf16 128 FWD" "resnet50 bf16 128 WGRAD"; do set -- $spec
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off \
  python tools/profile_one.py --config $1 --math $2 --layer conv1 --type $4 --algo I2C --b $3 --n $3 2>&1 | grep -E "s2d_input|win_pad|duration"
done
