#!/bin/bash
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 --expt-relaxed-constexpr -I paper_conf_cluster_zhaowplw25_b200/csrc -I include tools/mb_ingest.cu -o tools/mb_ingest -lcuda > gpurun_out/mb_ingest_build.log 2>&1
timeout 300 ./tools/mb_ingest > gpurun_out/mb_ingest.log 2>&1
( time timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider ) > gpurun_out/pytest_gpu.log 2>&1
SQ_GEMV_PATH=tc timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_run.py tc > gpurun_out/san_racecheck_tc.log 2>&1; echo "rc=$?" >> gpurun_out/san_racecheck_tc.log
tail -3 gpurun_out/pytest_gpu.log
