#!/bin/bash
# RGB-layer BackwardFilter: staged-row (AlexNet conv1) and window (ResNet conv1) kernels.
OUT=${1:-gpurun_out/c1}; mkdir -p $OUT
for math in tf32 bf16; do
  echo "== alexnet $math" >> $OUT/c1.txt
  timeout 120 python tools/time_one.py --math $math --specs conv1:WGRAD:I2C:256 conv1:WGRAD:IG:256 conv1:FWD:IG:256 >> $OUT/c1.txt 2>&1
done
for v in "" "MUCU_FORCE_CL=2" "MUCU_FORCE_CL=4" "MUCU_FORCE_CL=8" "MUCU_DETERMINISTIC=0"; do
  echo "== resnet50 bf16 [$v]" >> $OUT/c1.txt
  env $v MUCU_LOG_TILING=1 timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs conv1:WGRAD:I2C:128 conv1:WGRAD:IG:256 >> $OUT/c1.txt 2>&1
done
