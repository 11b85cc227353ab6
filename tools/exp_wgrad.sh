#!/bin/bash
# WGRAD tiling experiment (AlexNet conv2-5, TF32 and BF16): default vs knob variants.
OUT=${1:-gpurun_out/exp}; mkdir -p $OUT
SPECS="conv2:WGRAD:IG:256 conv3:WGRAD:IG:256 conv4:WGRAD:IG:256 conv5:WGRAD:IG:256 conv2:FWD:IG:256 conv2:DGRAD:IG:256"
for math in tf32 bf16; do
  for v in "" "MUCU_FORCE_BN=256" "MUCU_KM=1" "MUCU_FORCE_BN=256 MUCU_KM=1" "MUCU_M64=0" "MUCU_FORCE_CL=4" "MUCU_FORCE_CL=8" "MUCU_MT2=0"; do
    echo "== $math [$v]" >> $OUT/wgrad.txt
    env $v MUCU_LOG_TILING=1 timeout 120 python tools/time_one.py --math $math --specs $SPECS >> $OUT/wgrad.txt 2>&1
  done
done
