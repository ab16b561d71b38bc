# UG = 3 experiment (three 128-k groups per K2c unit, INT3/INT4 when 3 | k/128): parity of the
# forced tcgen05 path, then OPT-66B-shape GEMV rates with and without it.
for u in 1 0; do  # SQ_TC_UG3=0 disables (default on)
echo "== UG3 $u"
SQ_TC_UG3=$u SQ_GEMV_PATH=tc timeout 300 python tests/_decode_path_check.py 2>&1 | tail -2
SQ_TC_UG3=$u SQ_GEMV_PATH=tc timeout 300 python tools/gemv_rot.py --graph --shapes 9216x9216,27648x9216,36864x9216,9216x36864 --ms 1,32 --bits 3,4 2>&1 | grep GBps
done
