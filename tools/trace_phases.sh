mkdir -p gpurun_out
for L in r50_c64_56_f16 r50_c128_28_f16 r50_c256_14_f16 r50_c512_7_f16 vgg_64_64_224_f16 vgg_256_256_56_f16; do
  for C in 0 37; do
    echo "== $L cta $C"
    WINRS_LIB=libwinrs_tc2trace.so timeout 120 python tools/trace_tc2.py $L $C 2>&1 | grep -v "^ *[0-9]* " | head -8
  done
done > gpurun_out/trace_phases.txt 2>&1
