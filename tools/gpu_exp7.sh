#!/bin/bash
mkdir -p gpurun_out
for sm in 0 1 2; do
  echo "SPLIT $sm"
  SQ_TC_SPLIT=$sm SQ_GEMV_PATH=tc timeout 600 python tools/gemv_rot.py --graph --shapes 9216x36864,5120x20480,9216x9216,27648x9216,36864x9216 --bits 3,4,8 --ms 1,32
done > gpurun_out/e7.log 2>&1
cat gpurun_out/e7.log
