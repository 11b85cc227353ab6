timeout 900 python -m pytest tests -q -x -m gpu 2>&1 | tail -2
timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs layer1.0.conv3:FWD:IG:256 layer1.0.conv3:FWD:I2C:256 layer1.1.conv1:DGRAD:I2C:256 layer2.0.downsample:DGRAD:IG:256 layer1.0.conv2:FWD:IG:256 layer3.1.conv2:FWD:IG:256 conv1:FWD:I2C:128
timeout 120 python tools/time_one.py --config alexnet --math tf32 --specs conv2:FWD:IG:256 conv3:DGRAD:IG:256 conv1:DGRAD:I2C:256
