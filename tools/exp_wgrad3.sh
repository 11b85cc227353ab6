#!/bin/bash
# BackwardFilter pipeline shapes for AlexNet conv2 / conv3 / conv5 (TF32): tile height x
# width x k-blocks per stage.
OUT=${1:-gpurun_out/exp3}; mkdir -p $OUT
for v in "" "MUCU_MT2=0 MUCU_FORCE_BN=128" "MUCU_MT2=0 MUCU_FORCE_BN=128 MUCU_KM=1" "MUCU_MT2=0 MUCU_FORCE_BN=64 MUCU_KM=4" "MUCU_MT2=0 MUCU_FORCE_BN=64" "MUCU_MT2=0 MUCU_FORCE_BN=192"; do
  echo "== tf32 [$v]" >> $OUT/wgrad3.txt
  env $v MUCU_LOG_TILING=1 timeout 120 python tools/time_one.py --math tf32 --specs conv2:WGRAD:IG:256 conv3:WGRAD:IG:256 conv5:WGRAD:IG:256 >> $OUT/wgrad3.txt 2>&1
done
