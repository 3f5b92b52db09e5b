# A/B of TA builds (cold-L2 layer times): usage ab_ablate.sh variant...  ("" = libwinrs.so)
mkdir -p gpurun_out
for V in "$@"; do
  [ "$V" = base ] && V=""
  echo "== variant ${V:-base}"
  WINRS_LIB=libwinrs${V:+_$V}.so timeout 300 python tools/sweep_tc2.py ${LAYERS:-r50_c512_7_f16,r50_c256_14_f16,vgg_64_64_224_f16,vgg_512_512_28_f16} --quick 2>&1 | grep '"auto"' | cut -c1-100,150-230
done
