#!/bin/bash
mkdir -p gpurun_out
for L in libsq.so libsq_ss2.so libsq_snofix2.so; do
  echo "== $L" >> gpurun_out/k2s4.log
  SQ_LIB_PATH=$PWD/paper_conf_cluster_zhaowplw25_b200/$L SQ_GEMV_PATH=mma SQ_K2S=1 timeout 600 python tools/gemv_rot.py --graph --shapes 5120x5120,20480x5120,5120x20480,36864x9216 --bits 4,8 --ms 1 >> gpurun_out/k2s4.log 2>&1
done
cat gpurun_out/k2s4.log
