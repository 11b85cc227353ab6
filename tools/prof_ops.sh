#!/bin/bash
# ncu --set full of every kernel of one call of each op (aux kernels included),
# summarised on the box (reports are large):
#   tools/prof_ops.sh OUTDIR config:math:layer:TYPE:ALGO:b[:n] ...   (KEEP=1 keeps the .ncu-rep)
OUT=$1; shift
mkdir -p $OUT
for spec in "$@"; do
  IFS=: read cfg math layer typ algo b n <<< "$spec"
  n=${n:-$b}
  name=${cfg}_${math}_${layer}_${typ}_${algo}_${b}_${n}
  timeout -s KILL 600 ncu --set full --clock-control none --import-source on --profile-from-start off \
    -c 8 -o $OUT/$name -f \
    python tools/profile_one.py --config $cfg --math $math --layer $layer --type $typ --algo $algo --b $b --n $n \
    > $OUT/$name.log 2>&1
  echo "$spec rc=$?"
  python tools/ncu_ops.py $OUT/$name.ncu-rep 25 "${KREGEX:-tc_conv|simt}" > $OUT/$name.txt 2>&1
  [ "${KEEP:-0}" = 1 ] || rm -f $OUT/$name.ncu-rep
done
