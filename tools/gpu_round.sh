#!/bin/bash
# Round measurement on a B200 box (run via gpurun from the repo root):
#   tests, smoke, benches, the ncu launch list of the default bench step and a
#   full-set capture of its dominant kernel.  Every step has its own timeout.
# usage: tools/gpu_round.sh TAG [steps...]   steps: tests smoke bench others launches full extra ops fused
set -u
TAG=${1:-r01}; shift
STEPS=${*:-"tests smoke bench others launches full"}
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,temperature.gpu --format=csv > $OUT/gpu.txt 2>&1
has() { [[ " $STEPS " == *" $1 "* ]]; }

if has tests; then
  timeout -s KILL 1500 python -m pytest tests -q -m gpu -x > $OUT/tests.log 2>&1; echo "tests rc=$?" | tee -a $OUT/status
  tail -3 $OUT/tests.log
fi
if has smoke; then
  timeout -s KILL 300 python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('smoke ok')" > $OUT/smoke.log 2>&1
  echo "smoke rc=$?" | tee -a $OUT/status
fi
if has bench; then
  timeout -s KILL 900 python bench.py --tables-out $OUT/tables_alexnet_tf32.npz --json-out $OUT/bench_alexnet_tf32.json \
    > $OUT/bench_alexnet_tf32.log 2>&1; echo "bench rc=$?" | tee -a $OUT/status
  tail -c 600 $OUT/bench_alexnet_tf32.log
fi
if has others; then
  for cfg in "resnet50 bf16" "resnet18 bf16" "alexnet bf16"; do
    set -- $cfg
    timeout -s KILL 900 python bench.py --config $1 --math $2 --no-cpu-baseline --tables-out $OUT/tables_$1_$2.npz \
      --json-out $OUT/bench_$1_$2.json > $OUT/bench_$1_$2.log 2>&1; echo "bench $1 $2 rc=$?" | tee -a $OUT/status
  done
  timeout -s KILL 900 python bench.py --wd-mib 120 --steps 5 --no-cpu-baseline --json-out $OUT/bench_alexnet_tf32_wd120.json \
    > $OUT/bench_wd.log 2>&1; echo "bench wd rc=$?" | tee -a $OUT/status
fi
TAB=$OUT/tables_alexnet_tf32.npz
if has launches; then
  MUCU_PROFILE=1 timeout -s KILL 900 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off \
    --csv --log-file $OUT/launches_alexnet_tf32.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline \
    --tables-in $TAB > $OUT/launches.log 2>&1; echo "launches rc=$?" | tee -a $OUT/status
fi
if has full; then
  CMD=$(python - $OUT/bench_alexnet_tf32.json <<'PY'
import json, sys, re
d = json.load(open(sys.argv[1]))
k = d["roofline"]["kernel"]
layer, typ = k.split()[0], k.split()[1]
algo, b = re.findall(r"\('(\w+)', (\d+)\)", k)[0]
t = {"FWD": "FWD", "BWD_DATA": "DGRAD", "BWD_FILTER": "WGRAD", "DGRAD": "DGRAD", "WGRAD": "WGRAD"}[typ]
print(f"--layer {layer} --type {t} --algo {algo} --b {b}")
PY
)
  echo "dominant: $CMD" | tee -a $OUT/status
  # one launch of the GEMM kernel only (a full-set report of every micro-batch is tens of MB)
  timeout -s KILL 900 ncu --set full --clock-control none --import-source on --profile-from-start off \
    -k regex:tc_conv_gemm -c 1 -o $OUT/dominant_full -f python tools/profile_one.py --config alexnet --math tf32 $CMD \
    > $OUT/full.log 2>&1
  echo "full rc=$?" | tee -a $OUT/status
  # DRAM bytes of every launch of one call of the dominant op (bench.py roofline.traffic)
  timeout -s KILL 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
    --clock-control none --profile-from-start off --csv --log-file $OUT/dominant_traffic.csv \
    python tools/profile_one.py --config alexnet --math tf32 $CMD > $OUT/traffic.log 2>&1
  python - $OUT/dominant_traffic.csv $OUT/bench_alexnet_tf32.json $OUT/traffic.json <<'PY'
import csv, io, json, sys
txt = open(sys.argv[1]).read()
rows = list(csv.DictReader(io.StringIO(txt[txt.find('"ID"'):])))
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
tot = sum(float(r["Metric Value"].replace(",", "")) * scale.get(r["Metric Unit"], 1)
          for r in rows if r["Metric Name"] in ("dram__bytes_read.sum", "dram__bytes_write.sum"))
d = json.load(open(sys.argv[2]))
k = d["roofline"]["kernel"].split()
key = f"alexnet/tf32/{k[0]}/{k[1]}"
json.dump({key: int(tot), "_note": "DRAM read+write bytes of one call of the op (all its launches), "
           "ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum, tools/gpu_round.sh"}, open(sys.argv[3], "w"), indent=1)
print("traffic", key, int(tot))
PY
fi
if has extra; then
  # BASELINE configs 1 / 2-F32 / 3 / 4 (WD) and the non-deterministic reduction mode
  timeout -s KILL 900 python bench.py --math f32 --layers conv2 --types fwd --batch 8 --ws-mib 8 --policy all \
    --json-out $OUT/bench_cfg1_alexnet_conv2_f32.json > $OUT/bench_cfg1.log 2>&1; echo "cfg1 rc=$?" | tee -a $OUT/status
  timeout -s KILL 900 python bench.py --math f32 --steps 5 --no-cpu-baseline --json-out $OUT/bench_alexnet_f32.json \
    > $OUT/bench_alexnet_f32.log 2>&1; echo "f32 rc=$?" | tee -a $OUT/status
  timeout -s KILL 900 python bench.py --config resnet18 --math bf16 --wd-mib 480 --no-cpu-baseline \
    --json-out $OUT/bench_resnet18_bf16_wd480.json > /dev/null 2>&1; echo "wd r18 rc=$?" | tee -a $OUT/status
  timeout -s KILL 900 python bench.py --config resnet50 --math bf16 --wd-mib 10176 --no-cpu-baseline \
    --json-out $OUT/bench_resnet50_bf16_wd10176.json > /dev/null 2>&1; echo "wd r50 rc=$?" | tee -a $OUT/status
  timeout -s KILL 900 python bench.py --config resnet50 --math bf16 --wd-mib 5088 --no-cpu-baseline \
    --json-out $OUT/bench_resnet50_bf16_wd5088.json > /dev/null 2>&1; echo "wd r50 half rc=$?" | tee -a $OUT/status
  timeout -s KILL 900 python bench.py --ws-mib 8 --policy undivided --no-cpu-baseline \
    --json-out $OUT/bench_alexnet_tf32_wr8_undivided.json > /dev/null 2>&1; echo "wr8 und rc=$?" | tee -a $OUT/status
  for cfg in "alexnet tf32" "resnet50 bf16"; do
    set -- $cfg
    timeout -s KILL 900 python bench.py --config $1 --math $2 --nondeterministic --no-cpu-baseline \
      --json-out $OUT/bench_$1_$2_nondet.json > /dev/null 2>&1; echo "nondet $1 rc=$?" | tee -a $OUT/status
  done
fi
if has ops; then
  # per-op ncu --set full summaries (tools/prof_ops.sh): the F32 dominant op, Winograd
  # (transforms + batched GEMM), the TF32 WGRAD/DGRAD IG GEMMs, ResNet-50 layer1 3x3 BF16
  bash tools/prof_ops.sh $OUT/ops alexnet:f32:conv2:WGRAD:IG:256 alexnet:f32:conv2:FWD:IG:256 \
    alexnet:f32:conv3:FWD:WG:32 alexnet:f32:conv5:WGRAD:WG:32 alexnet:tf32:conv2:WGRAD:IG:256 \
    alexnet:tf32:conv2:DGRAD:IG:256 alexnet:tf32:conv1:FWD:I2C:64 resnet50:bf16:layer1.0.conv2:FWD:IG:256 \
    resnet50:bf16:layer1.0.conv2:DGRAD:IG:256 resnet50:bf16:layer1.0.conv2:WGRAD:IG:256 2>&1 | tee -a $OUT/status
fi
if has fused; then
  # NEXT-3: the dW sum fused into BackwardFilter (P2P target at one GPU; multicast where the box allows)
  timeout -s KILL 600 python -m pytest tests/test_nvls_gpu.py -q -rs > $OUT/nvls_tests.log 2>&1; echo "nvls tests rc=$?" | tee -a $OUT/status
  timeout -s KILL 900 python bench.py --grad-reduce p2p --no-cpu-baseline --json-out $OUT/bench_alexnet_tf32_p2p.json \
    > $OUT/bench_p2p.log 2>&1; echo "bench p2p rc=$?" | tee -a $OUT/status
fi
