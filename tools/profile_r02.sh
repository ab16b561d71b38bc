#!/bin/bash
# Round-2 profiles: launch lists of one bench step (prefill window, decode window; serialised, cold
# cache) and ncu --set full captures of the hot kernels.  Output under gpurun_out/ (scratch).
mkdir -p gpurun_out
K='regex:k_gemm|k_gemv|k_layernorm|k_copy|k_xsum|k_attn|k_kv'
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-gemv-sweep --no-gemm-sweep --no-configs0 --no-attention --no-bloom"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "$K" -c 2100 --csv --log-file gpurun_out/r02_launches_prefill.csv $B > gpurun_out/r02_launch_pre.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "$K" -s 2100 -c 3000 --csv --log-file gpurun_out/r02_launches_decode.csv $B > gpurun_out/r02_launch_dec.log 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemv_tc -s 3 -c 1 -o gpurun_out/r02_gemv_b4_36864x9216_m32 python tools/gemv_one.py 36864 9216 4 32 > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemv_tc -s 3 -c 1 -o gpurun_out/r02_gemv_b3_36864x9216_m32 python tools/gemv_one.py 36864 9216 3 32 > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemm -s 2 -c 1 -o gpurun_out/r02_gemm_b4_7168x28672_m4096 python tools/gemm_one.py 7168 28672 4 4096 > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemm -s 2 -c 1 -o gpurun_out/r02_gemm_b8_7168x28672_m4096 python tools/gemm_one.py 7168 28672 8 4096 > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_attn_decode -s 2 -c 1 -o gpurun_out/r02_attn_decode python tools/attn_one.py > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_attn_prefill -s 2 -c 1 -o gpurun_out/r02_attn_prefill python tools/attn_one.py > /dev/null 2>&1
ls -la gpurun_out/r02_*
