# PDL on/off x DEEP_A 0/1: back-to-back decode linears from one CUDA graph
for v in 0 1; do
python tools/build_variant.py -DSQ_TC_DEEP_A=$v > /dev/null 2>&1
for pdl in 1 0; do
echo "== deep$v pdl$pdl"
SQ_PDL=$pdl timeout 300 python tools/gemv_rot.py --graph --shapes 5120x5120,20480x5120,36864x9216 --ms 1,32 --bits 4,8,16 2>&1 | grep GBps
done
done
