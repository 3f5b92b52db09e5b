for L in r50_c512_7_f16 r50_c128_28_f16; do
  for C in 0 41 100 146; do
    WINRS_LIB=libwinrs_tc2trace.so WINRS_FORCE_TA=3 timeout 60 python tools/trace_sk.py $L $C 2>&1 | tail -4
  done
done
