python tools/build_variant.py -DSQ_TC_DEBUG=1 > /dev/null 2>&1
for s in "9216 9216 4 32" "36864 9216 4 32"; do echo "== trace $s"; SQ_PDL=0 timeout 60 python tools/trace_cta.py $s; done
python tools/build_variant.py > /dev/null 2>&1
SQ_GEMV_PATH=tc timeout 200 python -m pytest tests/test_gpu_linear.py -q -x -k "decode" 2>&1 | tail -1
SQ_GEMV_PATH=tc timeout 300 python tools/gemv_rot.py --graph --shapes 5120x5120,20480x5120,36864x9216,9216x36864 --ms 32 --bits 3,4,8,16 2>&1 | grep GBps
