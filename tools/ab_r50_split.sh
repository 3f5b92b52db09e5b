# ResNet-50 FP16 TA layers: the planner's (cs, Z) vs the alternatives that change the CTA count
for L in r50_c512_7_f16 r50_c128_28_f16 r50_c64_56_f16; do
  python tools/time_layer.py $L 50
  for cfg in "1 1" "2 1" "3 1" "4 1" "1 2" "2 2" "3 2" "4 2" "4 4" "8 2" "3 7" "2 7" "5 14" "4 14" "8 7" "6 7"; do
    set -- $cfg
    WINRS_FORCE_TA=1 WINRS_FORCE_CSPLIT=$1 WINRS_FORCE_Z=$2 timeout 60 python tools/time_layer.py $L 50
  done
done
