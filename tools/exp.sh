for w in 0 1; do echo "== WIDE=$w"
MUCU_MT2_WIDE=$w timeout 120 python tools/time_one.py --config alexnet --math tf32 --specs conv2:FWD:IG:256 conv3:FWD:IG:256 conv3:DGRAD:IG:256 conv4:FWD:IG:256 conv4:DGRAD:IG:256 conv5:FWD:IG:256 conv5:DGRAD:IG:256 conv1:FWD:I2C:64
MUCU_MT2_WIDE=$w timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs layer3.1.conv2:FWD:IG:256 layer3.1.conv2:DGRAD:IG:256 layer4.1.conv2:FWD:IG:256 layer4.1.conv2:DGRAD:IG:256 layer2.1.conv2:FWD:IG:256 layer3.0.conv2:DGRAD:IG:256 conv1:FWD:I2C:128
done
