#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_linear.py -m gpu -q -p no:cacheprovider -x -k "decode or adversarial" > gpurun_out/e10_pytest.log 2>&1
tail -3 gpurun_out/e10_pytest.log
echo "CORR1"; SQ_GEMV_PATH=tc timeout 600 python tools/gemv_rot.py --graph --shapes 9216x36864,9216x9216,36864x9216,20480x5120,5120x20480 --bits 3,4,8 --ms 1,32
python tools/build_variant.py -DSQ_TC_CORR=0 > /dev/null 2>&1
echo "CORR0"; SQ_GEMV_PATH=tc timeout 600 python tools/gemv_rot.py --graph --shapes 9216x36864,9216x9216,36864x9216,20480x5120,5120x20480 --bits 3,4,8 --ms 1,32
