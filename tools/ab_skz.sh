# stream-K pairs over Z segments (forced) for the mid VGG layers
for L in vgg_128_128_112_f16 vgg_128_256_56_f16 vgg_256_256_56_f16; do
  python tools/time_layer.py $L 10 | tail -1
  for Z in 2 4 7 8 14 16 28 56; do WINRS_FORCE_TA=3 WINRS_FORCE_Z=$Z timeout 60 python tools/time_layer.py $L 10 2>&1 | tail -1; done
done
