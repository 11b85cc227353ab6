#!/bin/bash
# ResNet-50 BF16 deterministic BackwardFilter: cluster size / group count sweep vs the
# non-deterministic (L2 atomic) reduction.
OUT=${1:-gpurun_out/exp_r50}; mkdir -p $OUT
SPECS="layer1.0.conv2:WGRAD:IG:256 layer2.1.conv2:WGRAD:IG:256 layer3.1.conv2:WGRAD:IG:256 layer2.0.downsample:WGRAD:IG:256"
for v in "" "MUCU_DETERMINISTIC=0" "MUCU_FORCE_CL=2" "MUCU_FORCE_CL=4" "MUCU_FORCE_CL=8" "MUCU_FORCE_CL=16" "MUCU_FORCE_CL=2 MUCU_FORCE_G=1" "MUCU_FORCE_CL=4 MUCU_FORCE_G=1" "MUCU_FORCE_CL=8 MUCU_FORCE_G=1" "MUCU_FORCE_CL=16 MUCU_FORCE_G=1"; do
  echo "== bf16 [$v]" >> $OUT/r50.txt
  env $v MUCU_LOG_TILING=1 timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs $SPECS >> $OUT/r50.txt 2>&1
done
