#!/bin/bash
set -u
timeout 900 python -m pytest tests/test_conv_gpu.py -q -x 2>&1 | tail -4
timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs layer1.0.conv2:WGRAD:WG:256 layer1.0.conv2:WGRAD:IG:256 layer2.1.conv2:WGRAD:WG:256 layer2.1.conv2:WGRAD:IG:256 layer3.1.conv2:WGRAD:WG:256 layer3.1.conv2:WGRAD:IG:256 layer4.1.conv2:WGRAD:WG:256 layer4.1.conv2:WGRAD:IG:256 layer4.1.conv2:WGRAD:WG:64
timeout 120 python tools/time_one.py --config alexnet --math tf32 --specs conv3:WGRAD:WG:256 conv3:WGRAD:IG:256 conv4:WGRAD:WG:256 conv4:WGRAD:IG:256 conv5:WGRAD:WG:256
