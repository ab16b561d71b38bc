run() { echo "== $1 PZ=$2"; SQ_TC_PZ=$2 timeout 200 python tools/gemv_rot.py --graph --shapes $3 --ms 32 --bits 4,8 2>&1 | grep GBps; }
for v in 0 1; do
python tools/build_variant.py -DSQ_TC_DEEP_A=$v > /dev/null 2>&1
for pz in "" "2,1" "4,2" "4,1" "1,2"; do run deep$v "$pz" 36864x9216; done
for pz in "" "1,2" "1,3"; do run deep$v "$pz" 9216x36864; done
for pz in "" "1,1" "2,1" "1,2"; do run deep$v "$pz" 20480x5120; done
done
