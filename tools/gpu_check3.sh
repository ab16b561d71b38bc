#!/bin/bash
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_stage.py tests/test_gpu_linear.py tests/test_gpu_attention.py -m gpu -q -p no:cacheprovider -x > gpurun_out/pytest_c3.log 2>&1
tail -2 gpurun_out/pytest_c3.log
SQ_GEMV_PATH=tc timeout 600 python tools/gemv_rot.py --graph --shapes 9216x36864,5120x20480,9216x9216 --bits 3,4,8 --ms 32 > gpurun_out/c3_rot.log 2>&1
cat gpurun_out/c3_rot.log
timeout 1500 python bench.py --steps 3 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err
echo "bench rc=$?" >> gpurun_out/bench.err; tail -2 gpurun_out/bench.err
