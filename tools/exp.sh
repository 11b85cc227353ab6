timeout 600 python -m pytest tests/test_conv_gpu.py -q -x -k "c3 or c2_k32" 2>&1 | tail -3
for cfg in "alexnet tf32 conv1" "alexnet bf16 conv1" "resnet50 bf16 conv1"; do set -- $cfg
  echo "== $cfg"
  for ud in 1 2; do MUCU_S2D_UD=$ud timeout 120 python tools/time_one.py --config $1 --math $2 --specs $3:DGRAD:I2C:256 $3:DGRAD:I2C:64; done
  for u in 2 4; do MUCU_S2D_U=$u timeout 120 python tools/time_one.py --config $1 --math $2 --specs $3:FWD:I2C:256 $3:FWD:I2C:64; done
done
