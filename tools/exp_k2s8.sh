#!/bin/bash
mkdir -p gpurun_out
for L in libsq.so libsq_s3a.so libsq_s3b.so libsq_s2b.so; do
  echo "== $L" >> gpurun_out/k2s8.log
  SQ_LIB_PATH=$PWD/paper_conf_cluster_zhaowplw25_b200/$L SQ_GEMV_PATH=mma SQ_K2S=1 timeout 600 python tools/gemv_rot.py --graph --shapes 5120x5120,20480x5120,5120x20480,36864x9216 --bits 4,8,3 --ms 1,8 >> gpurun_out/k2s8.log 2>&1
done
cat gpurun_out/k2s8.log
