timeout 900 python -m pytest tests -q -x -m gpu 2>&1 | tail -2
timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs layer2.0.conv2:DGRAD:IG:256 layer3.0.conv2:DGRAD:IG:256 layer4.0.conv2:DGRAD:IG:256
MUCU_MERGE_PHASES=0 timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs layer2.0.conv2:DGRAD:IG:256 layer3.0.conv2:DGRAD:IG:256 layer4.0.conv2:DGRAD:IG:256
