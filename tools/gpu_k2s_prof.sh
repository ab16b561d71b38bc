#!/bin/bash
# K2s evidence: compute-sanitizer (memcheck / racecheck / synccheck) over the decode kernels with K2s
# forced and K2 forced, and ncu --set full captures of K2s at the configs[1] / OPT-66B fc1 shapes.
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  SQ_K2S=1 SQ_GEMV_PATH=mma timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_run.py mma > gpurun_out/san_k2s_${tool}.log 2>&1; echo "rc=$?" >> gpurun_out/san_k2s_${tool}.log
done
SQ_K2S=0 SQ_GEMV_PATH=mma timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_run.py mma > gpurun_out/san_k2_racecheck.log 2>&1; echo "rc=$?" >> gpurun_out/san_k2_racecheck.log
for f in gpurun_out/san_*.log; do echo "== $f"; tail -15 $f; done
mkdir -p /tmp/ncu
for shp in "20480 5120 4 1" "36864 9216 4 1" "36864 9216 4 8" "20480 5120 8 1" "36864 9216 3 1"; do
  tag=$(echo $shp | tr ' ' '_')
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_gemv_s -s 3 -c 1 -o /tmp/ncu/k2s_$tag python tools/gemv_one.py $shp > /dev/null 2>&1
done
python tools/ncu_summary.py gpurun_out/k2s_ncu.json /tmp/ncu/k2s_*.ncu-rep > /dev/null 2>&1
cp /tmp/ncu/k2s_20480_5120_4_1.ncu-rep gpurun_out/ 2>/dev/null
ls -la gpurun_out
