# A/B of TA builds (cold-L2 layer times): usage ab_ablate.sh variant...  ("" = libwinrs.so)
# build the variants first, e.g. python tools/build.py --variant nosttm --define WINRS_TC2_NO_STTM
#   (nomma: WINRS_TC2_NO_MMA, notma: WINRS_TC2_NO_TMA, pf16: WINRS_TC2_PF=16, stx1: WINRS_TC2_STX4=0)
mkdir -p gpurun_out
for V in "$@"; do
  [ "$V" = base ] && V=""
  echo "== variant ${V:-base}"
  WINRS_LIB=libwinrs${V:+_$V}.so timeout 300 python tools/sweep_tc2.py ${LAYERS:-r50_c512_7_f16,r50_c256_14_f16,vgg_64_64_224_f16,vgg_512_512_28_f16} --quick 2>&1 | grep '"auto"' | cut -c1-100,150-230
done
