#!/bin/bash
# Batch-size policies: undivided / powerOfTwo / all on AlexNet at
# WR 64 MiB, F32 (the paper's precision) and TF32: ms/iter and benchmark-pass time.
OUT=${1:-gpurun_out/pol}; mkdir -p $OUT
for math in f32 tf32; do
  for pol in undivided pow2 all; do
    timeout -s KILL 1500 python bench.py --math $math --policy $pol --steps 5 --no-cpu-baseline \
      --json-out $OUT/bench_alexnet_${math}_${pol}.json > $OUT/${math}_${pol}.log 2>&1
    echo "$math $pol rc=$?" >> $OUT/status
  done
done
