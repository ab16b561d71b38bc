#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_linear.py -m gpu -q -p no:cacheprovider -x -k "decode or adversarial" > gpurun_out/e9_pytest.log 2>&1
tail -1 gpurun_out/e9_pytest.log
echo "R1"; (cd r1_ref && SQ_GEMV_PATH=tc timeout 600 python tools/gemv_rot.py --graph --shapes 9216x36864,9216x9216,36864x9216,20480x5120 --bits 3,4,8 --ms 1,32)
echo "R2"; SQ_GEMV_PATH=tc timeout 600 python tools/gemv_rot.py --graph --shapes 9216x36864,9216x9216,36864x9216,20480x5120 --bits 3,4,8 --ms 1,32
