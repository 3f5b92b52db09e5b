# A/B timelines of one CTA: TA (NK = 64) vs the xi-split pair (NK = 128) on ResNet-50 L4
mkdir -p gpurun_out
run() { C=$1; shift; echo "== cta $C $*"; env "$@" WINRS_LIB=libwinrs_tc2trace.so timeout 120 python tools/trace_tc2.py $L $C 2>&1 | head -22; }
L=r50_c512_7_f16
run 0 X=1
run 0 WINRS_FORCE_TA=2 WINRS_FORCE_TILE=128x128 WINRS_FORCE_CSPLIT=1
run 1 WINRS_FORCE_TA=2 WINRS_FORCE_TILE=128x128 WINRS_FORCE_CSPLIT=1
