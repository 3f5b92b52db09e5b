# TA F = 2: deeper ring (17 KB stages) for the CTAs whose second fh slot is dead (WINRS_TC2_TA_DEAD_S)
for lib in libwinrs.so libwinrs_dr12.so libwinrs_dr10.so libwinrs.so libwinrs_dr12.so; do
  for L in vgg_64_64_224_f16 r50_c64_56_f16; do
    WINRS_LIB=$lib timeout 60 python tools/time_layer.py $L 30 | sed "s/^/$lib /"
  done
done
