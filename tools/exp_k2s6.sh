#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_linear.py -q -x -p no:cacheprovider -k "forced_path" > gpurun_out/k2s6_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/k2s6_pytest.log
tail -3 gpurun_out/k2s6_pytest.log
for Z in 1 2 4 8; do
echo "== Z=$Z" >> gpurun_out/k2s6_rot.log
SQ_K2S_Z=$Z SQ_K2S=1 SQ_GEMV_PATH=mma timeout 300 python tools/gemv_rot.py --graph --shapes 5120x5120,20480x5120,5120x20480,36864x9216 --bits 4 --ms 1 >> gpurun_out/k2s6_rot.log 2>&1
done
cat gpurun_out/k2s6_rot.log
