# TA ring depth A/B: 8 slots (default) vs 6 (libwinrs_s6.so)
# build first: python tools/build.py --variant s6 --define WINRS_TC2_TA_S=6
for V in base s6; do [ "$V" = base ] && V=""; for L in vgg_64_64_224_f16 r50_c64_56_f16 r50_c256_14_f16 r50_c512_7_f16; do WINRS_LIB=libwinrs${V:+_$V}.so python tools/time_layer.py $L 20 | sed "s/^/${V:-s8} /"; done; done
