# balanced xi split (default build) vs the {0,1}/{2,3} split (libwinrs_nobal.so): forced xi-split / stream-K plans
for V in base nobal; do
  [ "$V" = base ] && V=""
  for L in vgg_128_128_112_f16 vgg_256_256_56_f16 vgg_512_512_28_f16 vgg_512_512_14_f16 vgg_256_512_28_f16 r50_c512_7_f16 r50_c256_14_f16; do
    WINRS_LIB=libwinrs${V:+_$V}.so WINRS_FORCE_TA=3 timeout 60 python tools/time_layer.py $L 10 2>&1 | tail -1
    WINRS_LIB=libwinrs${V:+_$V}.so WINRS_FORCE_TA=2 timeout 60 python tools/time_layer.py $L 10 2>&1 | tail -1
  done
done
