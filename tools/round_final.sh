#!/bin/bash
# End-of-round GPU pass: GPU tests, bench line, reference line, smoke, launch lists of one bench step,
# ncu --set full captures of the decode / prefill kernels (reports stay in /tmp; summaries to gpurun_out).
# (compute-sanitizer is closed on this pool: tests/test_gpu_linear.py::test_decode_mma_writes_in_bounds
# is the sentinel substitute for the decode kernels added after round 2's sanitizer pass.)
mkdir -p gpurun_out /tmp/ncu
( time timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider ) > gpurun_out/final_pytest.log 2>&1
timeout 1500 python bench.py --steps 3 --warmup 3 > gpurun_out/final_bench.json 2> gpurun_out/final_bench.err; echo "bench rc=$?" >> gpurun_out/final_bench.err
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/final_bench_ref.json 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/final_smoke.log
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemv_tc -s 3 -c 1 -o /tmp/ncu/final_gemv_tc_b4_36864x9216_m32 python tools/gemv_one.py 36864 9216 4 32 > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemv_tc -s 3 -c 1 -o /tmp/ncu/final_gemv_tc_b3_36864x9216_m32 python tools/gemv_one.py 36864 9216 3 32 > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemv_s -s 3 -c 1 -o /tmp/ncu/final_gemv_s_b4_36864x9216_m1 python tools/gemv_one.py 36864 9216 4 1 > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemv_s -s 3 -c 1 -o /tmp/ncu/final_gemv_s_b4_20480x5120_m1 python tools/gemv_one.py 20480 5120 4 1 > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemm -s 3 -c 1 -o /tmp/ncu/final_gemm_b4_36864x9216_m4096 python tools/gemm_one.py 36864 9216 4 4096 > /dev/null 2>&1
python tools/ncu_summary.py gpurun_out/final_ncu.json /tmp/ncu/final_*.ncu-rep > /dev/null 2>&1
# launch lists of one bench step (prefill window, decode window; serialised, cold cache)
K='regex:k_gemm|k_gemv|k_layernorm|k_copy|k_xsum|k_attn|k_kv'
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-gemv-sweep --no-gemm-sweep --no-configs0 --no-attention --no-bloom --no-tp"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "$K" -c 2100 --csv --log-file gpurun_out/final_launches_prefill.csv $B > gpurun_out/final_launch_pre.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "$K" -s 2100 -c 3000 --csv --log-file gpurun_out/final_launches_decode.csv $B > gpurun_out/final_launch_dec.log 2>&1
tail -2 gpurun_out/final_pytest.log
