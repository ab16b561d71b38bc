#!/bin/bash
# One gpurun call: GPU tests, compute-sanitizer over every hot-path kernel, a short bench line.
# Outputs under gpurun_out/ (scratch); summaries are copied to profiles/ by hand.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt 2>&1
( time timeout 1800 python -m pytest tests -m gpu -x -q -p no:cacheprovider ) > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
# (compute-sanitizer is closed on this pool since round 2: SANITIZE=1 to try it where it runs)
if [ "${SANITIZE:-0}" = "1" ]; then
  for tool in memcheck racecheck synccheck; do
    timeout 900 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_run.py all > gpurun_out/san_${tool}.log 2>&1
    echo "rc=$?" >> gpurun_out/san_${tool}.log
  done
  SQ_GEMV_PATH=mma timeout 900 compute-sanitizer --tool memcheck --print-limit 50 python tools/sanitize_run.py mma > gpurun_out/san_memcheck_mma.log 2>&1; echo "rc=$?" >> gpurun_out/san_memcheck_mma.log
  SQ_GEMV_PATH=tc SQ_TC_CLUSTER=0 timeout 900 compute-sanitizer --tool memcheck --print-limit 50 python tools/sanitize_run.py tc > gpurun_out/san_memcheck_tc_nocluster.log 2>&1; echo "rc=$?" >> gpurun_out/san_memcheck_tc_nocluster.log
  SQ_GEMV_PATH=tc timeout 900 compute-sanitizer --tool racecheck --print-limit 50 python tools/sanitize_run.py tc > gpurun_out/san_racecheck_tc.log 2>&1; echo "rc=$?" >> gpurun_out/san_racecheck_tc.log
fi
if [ "${BENCH:-1}" = "1" ]; then
  timeout 1200 python bench.py --steps 3 --warmup 3 > gpurun_out/bench.json 2> gpurun_out/bench.err
  echo "bench rc=$?" >> gpurun_out/bench.err
fi
tail -3 gpurun_out/pytest_gpu.log
