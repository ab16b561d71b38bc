# decode kernel choice after UG = 3: mma.sync K2 vs tcgen05 K2c at small m
for path in mma tc; do
echo "== PATH $path"
SQ_GEMV_PATH=$path timeout 300 python tools/gemv_rot.py --graph --shapes 27648x9216,36864x9216,9216x36864 --ms 1,4,8 --bits 3,4 2>&1 | grep GBps
SQ_GEMV_PATH=$path timeout 300 python tools/gemv_rot.py --graph --shapes 20480x5120,5120x20480 --ms 1,4 --bits 4 2>&1 | grep GBps
done
