#!/bin/bash
mkdir -p gpurun_out
for dqw in 8 16 24; do
  SQ_NVCC_EXTRA="-DSQ_TC_DEBUG=1 -DSQ_TC_DQW=$dqw" python tools/build_variant.py -DSQ_TC_DEBUG=1 -DSQ_TC_DQW=$dqw > gpurun_out/e5_build_$dqw.log 2>&1
  SQ_GEMV_PATH=tc timeout 300 python tools/gemv_rot.py --graph --shapes 20480x5120,36864x9216,9216x9216 --bits 3,4,8 --ms 32 > gpurun_out/e5_rot_$dqw.log 2>&1
  timeout 300 python tools/trace_tc.py 36864 9216 4 32 > gpurun_out/e5_trace_$dqw.log 2>&1
done
cat gpurun_out/e5_rot_*.log
