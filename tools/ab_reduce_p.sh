# Bucket reduction with P z-parts per element (WINRS_REDUCE_P, default 8) vs one thread per element (1)
for L in vgg_64_64_224_f16 vgg_64_128_112_f16 vgg_128_128_112_f16 r50_c64_56_f16 r50_c128_28_f16; do
  for v in 1 8 1 8; do WINRS_REDUCE_P=$v timeout 60 python tools/time_layer.py $L 50; done
done
