# bucket-reduce load-batch A/B; build first: python tools/build.py --variant zb16 --define WINRS_REDUCE_ZB=16 (and zb32)
for V in base zb16 zb32; do [ "$V" = base ] && V=""; for L in vgg_64_64_224_f16 r50_c64_56_f16 vgg_64_128_112_f16; do WINRS_LIB=libwinrs${V:+_$V}.so python tools/time_layer.py $L 20 | sed "s/^/${V:-zb8} /"; done; done
