export MUCU_HALO=0
timeout 900 python -m pytest tests/test_conv_gpu.py -q -x 2>&1 | tail -2
for m4 in 0 1; do echo "== MT4=$m4"
MUCU_MT4=$m4 timeout 120 python tools/time_one.py --config alexnet --math tf32 --specs conv2:DGRAD:IG:256 conv2:FWD:IG:256
MUCU_MT4=$m4 timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs layer1.0.conv2:FWD:IG:256 layer1.0.conv2:DGRAD:IG:256 layer1.1.conv1:FWD:I2C:256 layer1.1.conv1:FWD:IG:256 layer1.0.conv3:DGRAD:I2C:256 layer1.0.conv3:DGRAD:IG:256
done
