#!/bin/bash
# End-of-round GPU pass: GPU tests, compute-sanitizer, bench line, smoke, ncu captures of the final kernels.
mkdir -p gpurun_out
( time timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider ) > gpurun_out/final_pytest.log 2>&1
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_run.py all > gpurun_out/final_san_${tool}.log 2>&1; echo "rc=$?" >> gpurun_out/final_san_${tool}.log
done
SQ_GEMV_PATH=tc SQ_TC_CLUSTER=0 timeout 900 compute-sanitizer --tool memcheck --print-limit 20 python tools/sanitize_run.py tc > gpurun_out/final_san_memcheck_tc_nocluster.log 2>&1; echo "rc=$?" >> gpurun_out/final_san_memcheck_tc_nocluster.log
SQ_GEMV_PATH=mma timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_run.py mma > gpurun_out/final_san_racecheck_mma.log 2>&1; echo "rc=$?" >> gpurun_out/final_san_racecheck_mma.log
timeout 1500 python bench.py --steps 3 --warmup 3 > gpurun_out/final_bench.json 2> gpurun_out/final_bench.err; echo "bench rc=$?" >> gpurun_out/final_bench.err
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/final_bench_ref.json 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/final_smoke.log
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemv_tc -s 3 -c 1 -o gpurun_out/final_gemv_b4_36864x9216_m32 python tools/gemv_one.py 36864 9216 4 32 > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemv_tc -s 3 -c 1 -o gpurun_out/final_gemv_b3_36864x9216_m32 python tools/gemv_one.py 36864 9216 3 32 > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemm_i8 -s 2 -c 1 -o gpurun_out/final_w8a8_prefill python -c "
import sys; sys.path.insert(0, '.')
import torch, synth, paper_conf_cluster_zhaowplw25_b200 as sq
n, k, m = 7168, 28672, 4096
w = torch.empty((n, k), dtype=torch.float16, device='cuda'); synth.device_weight_f16(w.data_ptr(), 1, n, k)
g = sq.W8Linear.from_fp16(w); x = torch.randn(m, k, device='cuda').half(); y = torch.empty(m, n, dtype=torch.float16, device='cuda')
for _ in range(4):
    xq, sx = sq.sq_quantize_act8(x); sq.sq_linear_w8a8(g, xq, sx, y, 0)
torch.cuda.synchronize()" > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemm -s 3 -c 1 -o gpurun_out/final_gemm_b4_36864x9216_m4096 python tools/gemm_one.py 36864 9216 4 4096 > /dev/null 2>&1
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemm -s 3 -c 1 -o gpurun_out/final_gemm_b16_27648x9216_m4096 python tools/gemm_one.py 27648 9216 16 4096 > /dev/null 2>&1
# launch lists of one bench step (prefill window, decode window; serialised, cold cache)
K='regex:k_gemm|k_gemv|k_layernorm|k_copy|k_xsum|k_attn|k_kv'
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-gemv-sweep --no-gemm-sweep --no-configs0 --no-attention --no-bloom --no-tp"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "$K" -c 2100 --csv --log-file gpurun_out/final_launches_prefill.csv $B > gpurun_out/final_launch_pre.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "$K" -s 2100 -c 3000 --csv --log-file gpurun_out/final_launches_decode.csv $B > gpurun_out/final_launch_dec.log 2>&1
tail -2 gpurun_out/final_pytest.log
