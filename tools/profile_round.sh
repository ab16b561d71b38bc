# Round profiles: launch list of one bench step (serialised, cold-cache) + ncu --set full of the
# top kernels.  Output under gpurun_out/; summaries are copied to profiles/ by the caller.
set -x
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_gemm|k_gemv|k_layernorm|k_copy|k_xsum" -c 4000 --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --no-gemv-sweep > gpurun_out/launch_bench.log 2>&1
for spec in "36864 9216 4 32" "36864 9216 8 32" "36864 9216 4 1" "36864 9216 3 32"; do
  set -- $spec
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemv -s 3 -c 1 -o gpurun_out/full_gemv_b$3_$1x$2_m$4 python tools/gemv_one.py $1 $2 $3 $4 > /dev/null 2>&1
done
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemm -s 2 -c 1 -o gpurun_out/full_gemm_b4_9216x9216_m4096 python tools/gemm_one.py 9216 9216 4 4096 > /dev/null 2>&1
ls -la gpurun_out
