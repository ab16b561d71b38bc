for cl in 1 0; do
echo "== CL $cl"
SQ_TC_CLUSTER=$cl SQ_GEMV_PATH=tc timeout 200 python -m pytest tests/test_gpu_linear.py -q -x -k "decode" 2>&1 | tail -2
SQ_TC_CLUSTER=$cl SQ_GEMV_PATH=tc timeout 300 python tools/gemv_rot.py --graph --shapes 5120x5120,20480x5120,5120x20480,9216x9216,27648x9216,36864x9216,9216x36864 --ms 32 --bits 3,4,8,16 2>&1 | grep GBps
done
