for v in 1 0; do
python tools/build_variant.py -DSQ_TC_XLDG=$v > /dev/null 2>&1
echo "== xldg$v"
SQ_GEMV_PATH=tc timeout 200 python -m pytest tests/test_gpu_linear.py -q -x -k "decode" 2>&1 | tail -1
SQ_GEMV_PATH=tc timeout 300 python tools/gemv_rot.py --graph --shapes 5120x5120,20480x5120,36864x9216,9216x36864 --ms 32 --bits 3,4,8,16 2>&1 | grep GBps
done
