timeout 900 python -m pytest tests/test_conv_gpu.py -q -x -k "c3 or c2_k32" 2>&1 | tail -1
timeout 120 python tools/time_one.py --config resnet50 --math bf16 --specs conv1:WGRAD:I2C:256 conv1:WGRAD:I2C:128
timeout 120 python tools/time_one.py --config alexnet --math bf16 --specs conv1:WGRAD:I2C:256
timeout 120 python tools/time_one.py --config alexnet --math tf32 --specs conv1:WGRAD:I2C:256
