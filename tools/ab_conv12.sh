# VGG conv1_2 plan A/B (TA 64x2fh): the planner's pick vs forced cluster split / segment counts
L=vgg_64_64_224_f16
python tools/time_layer.py $L 20
for cfg in "4 16" "4 14" "2 28" "2 32" "1 56" "1 74" "4 18" "8 8" "3 21" "5 12"; do
  set -- $cfg
  WINRS_FORCE_TILE=64x64 WINRS_FORCE_TA=1 WINRS_FORCE_CSPLIT=$1 WINRS_FORCE_Z=$2 timeout 60 python tools/time_layer.py $L 20
done
