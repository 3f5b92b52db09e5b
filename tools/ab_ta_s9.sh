# TA ring depth 9 (default build) vs 8 (libwinrs_s8.so)
for V in base s8; do [ "$V" = base ] && V=""; for L in vgg_64_64_224_f16 r50_c64_56_f16 r50_c128_28_f16 r50_c256_14_f16 r50_c512_7_f16; do WINRS_LIB=libwinrs${V:+_$V}.so python tools/time_layer.py $L 20 | sed "s/^/${V:-s9} /"; done; done
