#!/bin/bash
mkdir -p gpurun_out
for L in libsq.so libsq_udesc.so libsq.so libsq_udesc.so; do
  echo "== $L" >> gpurun_out/udesc.log
  SQ_LIB_PATH=$PWD/paper_conf_cluster_zhaowplw25_b200/$L timeout 600 python tools/gemv_rot.py --graph --shapes 27648x9216,9216x9216,36864x9216,9216x36864 --bits 4,3,8,16 --ms 32 >> gpurun_out/udesc.log 2>&1
done
SQ_LIB_PATH=$PWD/paper_conf_cluster_zhaowplw25_b200/libsq_udesc.so SQ_GEMV_PATH=tc timeout 600 python tests/_decode_path_check.py >> gpurun_out/udesc.log 2>&1
cat gpurun_out/udesc.log
