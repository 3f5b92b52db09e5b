# Bucket reduction as a programmatic dependent launch (WINRS_PDL=1, default) vs a plain launch
for L in r50_c64_56_f16 r50_c128_28_f16 vgg_64_64_224_f16 vgg_64_128_112_f16 vgg_128_128_112_f16 vgg_128_256_56_f16 vgg_256_256_56_f16; do
  for v in 0 1 0 1; do WINRS_PDL=$v timeout 60 python tools/time_layer.py $L 50; done
done
