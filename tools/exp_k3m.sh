#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_linear.py tests/test_gpu_stage.py -q -x -p no:cacheprovider > gpurun_out/k3m_pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/k3m_pytest.log
tail -3 gpurun_out/k3m_pytest.log
timeout 600 python tools/gemv_rot.py --graph --shapes 5120x5120,20480x5120,5120x20480,36864x9216,9216x36864,768x3072 --bits 3 --ms 1,8,16 > gpurun_out/k3m_rot.log 2>&1
cat gpurun_out/k3m_rot.log
