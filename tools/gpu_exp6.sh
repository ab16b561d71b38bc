#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_linear.py -m gpu -q -p no:cacheprovider -x -k "decode" > gpurun_out/e6_pytest.log 2>&1
tail -2 gpurun_out/e6_pytest.log
SQ_GEMV_PATH=tc timeout 600 python tools/gemv_rot.py --graph --shapes 5120x5120,20480x5120,5120x20480,9216x9216,36864x9216,9216x36864 --bits 3,4,8 --ms 1,32 > gpurun_out/e6_rot16.log 2>&1
python tools/build_variant.py -DSQ_TC_DQG=8 > /dev/null 2>&1
SQ_GEMV_PATH=tc timeout 600 python tools/gemv_rot.py --graph --shapes 20480x5120,9216x9216,36864x9216 --bits 3,4,8 --ms 32 > gpurun_out/e6_rot8.log 2>&1
cat gpurun_out/e6_rot16.log gpurun_out/e6_rot8.log
