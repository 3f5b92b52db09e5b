# stream-K xi-split pairs (forced) vs the planner's pick and the TA default (forced TA=1) per layer
for L in ${LAYERS:-r50_c64_56_f16 r50_c128_28_f16 r50_c256_14_f16 r50_c512_7_f16 vgg_64_64_224_f16 vgg_64_128_112_f16 vgg_128_128_112_f16 vgg_128_256_56_f16 vgg_256_256_56_f16 vgg_256_512_28_f16 vgg_512_512_28_f16 vgg_512_512_14_f16}; do
  WINRS_FORCE_TA=3 timeout 60 python tools/time_layer.py $L 10 2>&1 | tail -1
  timeout 60 python tools/time_layer.py $L 10 2>&1 | tail -1
done
