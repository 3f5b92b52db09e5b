# balanced xi split with 10-deep rings (build: python tools/build.py --variant bal --define WINRS_TC2X_BAL=1) vs default
WINRS_LIB=libwinrs_bal.so timeout 300 python -m pytest tests/test_gpu_r2.py -q -x -k "xs or exact" 2>&1 | tail -1
for V in base bal; do [ "$V" = base ] && V=""; for L in vgg_64_128_112_f16 vgg_128_128_112_f16 vgg_256_256_56_f16 vgg_256_512_28_f16 vgg_512_512_28_f16 vgg_512_512_14_f16; do WINRS_LIB=libwinrs${V:+_$V}.so python tools/time_layer.py $L 20 | sed "s/^/${V:-default} /"; done; done
