#!/bin/bash
mkdir -p gpurun_out
echo "R1"; (cd r1_ref && SQ_GEMV_PATH=tc timeout 600 python tools/gemv_rot.py --graph --shapes 9216x36864,9216x9216,36864x9216 --bits 3,4,8 --ms 1,32)
echo "R2"; SQ_GEMV_PATH=tc timeout 600 python tools/gemv_rot.py --graph --shapes 9216x36864,9216x9216,36864x9216 --bits 3,4,8 --ms 1,32
bash tools/profile_r02.sh > gpurun_out/prof.log 2>&1
