#!/bin/bash
# WGRAD pipeline experiment: conv2 / conv5 TF32 with tile / stage knobs.
OUT=${1:-gpurun_out/exp2}; mkdir -p $OUT
SPECS="conv2:WGRAD:IG:256 conv5:WGRAD:IG:256"
for v in "" "MUCU_FORCE_BN=64" "MUCU_FORCE_BN=96" "MUCU_FORCE_BN=64 MUCU_KM=4" "MUCU_FORCE_BN=32 MUCU_KM=4" "MUCU_KM=1 MUCU_MAX_STAGES=2" "MUCU_KM=1 MUCU_MAX_STAGES=3" "MUCU_FORCE_BN=64 MUCU_MAX_STAGES=2" "MUCU_FORCE_BN=64 MUCU_MAX_STAGES=3" "MUCU_FORCE_BN=64 MUCU_FORCE_CL=4" "MUCU_M64=0 MUCU_FORCE_BN=64"; do
  echo "== tf32 [$v]" >> $OUT/wgrad2.txt
  env $v MUCU_LOG_TILING=1 timeout 120 python tools/time_one.py --math tf32 --specs $SPECS >> $OUT/wgrad2.txt 2>&1
done
