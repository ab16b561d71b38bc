#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_linear.py -q -x -p no:cacheprovider -k "decode" > gpurun_out/k2s16_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/k2s16_pytest.log
tail -3 gpurun_out/k2s16_pytest.log
for K in 0 1; do
echo "== SQ_K2S16=$K" >> gpurun_out/k2s16_rot.log
SQ_K2S16=$K timeout 600 python tools/gemv_rot.py --graph --shapes 5120x5120,20480x5120,5120x20480,36864x9216,9216x36864,27648x9216,9216x9216 --bits 4,8,3 --ms 12,16 >> gpurun_out/k2s16_rot.log 2>&1
done
cat gpurun_out/k2s16_rot.log
