#!/bin/bash
# K2c: dequantize the first PRE batches before the A-slot wait (SQ_TC_PRE) vs the default
mkdir -p gpurun_out
for L in libsq.so libsq_pre1.so libsq_pre2.so; do
  echo "== $L" >> gpurun_out/pre.log
  SQ_LIB_PATH=$PWD/paper_conf_cluster_zhaowplw25_b200/$L timeout 600 python tools/gemv_rot.py --graph --shapes 27648x9216,9216x9216,36864x9216,9216x36864,20480x5120 --bits 4,3,8 --ms 32 >> gpurun_out/pre.log 2>&1
done
for L in libsq_pre1.so libsq_pre2.so; do
SQ_LIB_PATH=$PWD/paper_conf_cluster_zhaowplw25_b200/$L SQ_GEMV_PATH=tc timeout 600 python tests/_decode_path_check.py >> gpurun_out/pre.log 2>&1
done
cat gpurun_out/pre.log
