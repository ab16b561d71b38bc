#!/bin/bash
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_linear.py tests/test_gpu_stage.py -q -x -p no:cacheprovider > gpurun_out/k2s3_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/k2s3_pytest.log
tail -3 gpurun_out/k2s3_pytest.log
timeout 600 python tools/gemv_rot.py --graph --shapes 5120x5120,20480x5120,5120x20480,36864x9216,9216x9216 --bits 4,8,3 --ms 1,2,4,8 > gpurun_out/k2s3_rot.log 2>&1
cat gpurun_out/k2s3_rot.log
