# xi-split pair (forced) vs the default plan on the large-K layers: linearity build vs FT-store build
# build first: python tools/build.py --variant xsft --define WINRS_TC2X_LIN=0   (FT stores on the e = 0 half)
for V in base xsft; do
  [ "$V" = base ] && V=""
  for L in ${LAYERS:-vgg_512_512_28_f16 vgg_256_256_56_f16 vgg_128_128_112_f16 vgg_256_512_28_f16 r50_c512_7_f16 r50_c256_14_f16}; do
    for cs in 1 2 3 4; do WINRS_LIB=libwinrs${V:+_$V}.so WINRS_FORCE_TA=2 WINRS_FORCE_CSPLIT=$cs timeout 60 python tools/time_layer.py $L 10 2>&1 | tail -1; done
    [ -z "$V" ] && python tools/time_layer.py $L 10 | tail -1
  done
done
