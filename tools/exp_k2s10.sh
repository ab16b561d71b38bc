#!/bin/bash
mkdir -p gpurun_out
for L in libsq.so libsq_ilv.so; do
  echo "== $L" >> gpurun_out/k2s10.log
  SQ_LIB_PATH=$PWD/paper_conf_cluster_zhaowplw25_b200/$L timeout 600 python tools/gemv_rot.py --graph --shapes 5120x5120,20480x5120,5120x20480,36864x9216,9216x36864 --bits 4,8,3 --ms 1,8 >> gpurun_out/k2s10.log 2>&1
done
SQ_LIB_PATH=$PWD/paper_conf_cluster_zhaowplw25_b200/libsq_ilv.so SQ_GEMV_PATH=mma SQ_K2S=1 timeout 600 python tests/_decode_path_check.py >> gpurun_out/k2s10.log 2>&1
cat gpurun_out/k2s10.log
