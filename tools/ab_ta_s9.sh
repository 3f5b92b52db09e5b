# TA ring depth 9 (libwinrs_s9.so) vs 8 (default build)
# build first: python tools/build.py --variant s9 --define WINRS_TC2_TA_S=9   (the default build is 8)
for V in s9 base; do [ "$V" = base ] && V=""; for L in vgg_64_64_224_f16 r50_c64_56_f16 r50_c128_28_f16 r50_c256_14_f16 r50_c512_7_f16; do WINRS_LIB=libwinrs${V:+_$V}.so python tools/time_layer.py $L 20 | sed "s/^/${V:-s8} /"; done; done
