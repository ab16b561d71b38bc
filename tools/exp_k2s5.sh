#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_linear.py -q -x -p no:cacheprovider -k "decode" > gpurun_out/k2s5_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/k2s5_pytest.log
tail -3 gpurun_out/k2s5_pytest.log
for K in 1 0; do
echo "== SQ_K2S=$K" >> gpurun_out/k2s5_rot.log
SQ_K2S=$K SQ_GEMV_PATH=mma timeout 600 python tools/gemv_rot.py --graph --shapes 5120x5120,20480x5120,5120x20480,36864x9216,9216x9216,768x768,3072x768 --bits 4,8,3 --ms 1,8 >> gpurun_out/k2s5_rot.log 2>&1
done
cat gpurun_out/k2s5_rot.log
