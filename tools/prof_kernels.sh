#!/bin/bash
# ncu --set full of the first tc_conv_gemm launch of each spec:
#   tools/prof_kernels.sh OUTDIR config:math:layer:TYPE:ALGO:b ...
OUT=$1; shift
mkdir -p $OUT
for spec in "$@"; do
  IFS=: read cfg math layer typ algo b <<< "$spec"
  timeout -s KILL 600 ncu --set full --clock-control none --import-source on --profile-from-start off \
    -k regex:tc_conv_gemm -c 1 -o $OUT/${cfg}_${math}_${layer}_${typ}_${algo}_${b} -f \
    python tools/profile_one.py --config $cfg --math $math --layer $layer --type $typ --algo $algo --b $b --n $b \
    > $OUT/${cfg}_${math}_${layer}_${typ}_${algo}_${b}.log 2>&1
  echo "$spec rc=$?"
done
