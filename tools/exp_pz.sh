for pz in "" "2,1" "3,2" "1,2" "4,3"; do
echo "== PZ $pz"
SQ_TC_PZ=$pz SQ_GEMV_PATH=tc timeout 300 python tools/gemv_rot.py --graph --shapes 27648x9216,9216x9216,9216x36864 --ms 32 --bits 4,8 2>&1 | grep GBps
done
