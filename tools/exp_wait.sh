for w in 0 1 2; do
python tools/build_variant.py -DSQ_TC_WAIT=$w > /dev/null 2>&1
echo "== wait$w"
SQ_GEMV_PATH=tc timeout 300 python tools/gemv_rot.py --graph --shapes 5120x5120,20480x5120,36864x9216 --ms 32 --bits 3,4,8,16 2>&1 | grep GBps
done
