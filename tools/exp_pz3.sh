# (P, Z) alternatives to tc_plan's choice under UG = 3, m = 32 (SQ_TC_PZ forces them)
for spec in "9216x9216 3,6" "9216x9216 4,8" "9216x9216 2,4" "9216x9216 1,2" "27648x9216 3,2" "27648x9216 2,1" "27648x9216 1,1" "36864x9216 4,2" "36864x9216 2,1" "36864x9216 1,1" "9216x36864 4,8" "9216x36864 2,4" "9216x36864 1,2"; do
set -- $spec
echo "== $1 PZ $2"
SQ_TC_PZ=$2 SQ_GEMV_PATH=tc timeout 120 python tools/gemv_rot.py --graph --shapes $1 --ms 32 --bits 4 2>&1 | grep GBps
done
