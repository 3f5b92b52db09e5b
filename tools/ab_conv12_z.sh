# VGG conv1_2 (TA 64x2fh): wave count vs segment count Z (bands x 112 columns, Alg. 2 granularity)
L=vgg_64_64_224_f16
python tools/time_layer.py $L 20
for cfg in "1 336" "1 560" "1 784" "1 448" "2 336" "2 224" "3 224" "4 112" "5 112" "2 112"; do
  set -- $cfg
  WINRS_FORCE_TA=1 WINRS_FORCE_CSPLIT=$1 WINRS_FORCE_Z=$2 timeout 60 python tools/time_layer.py $L 20
done
