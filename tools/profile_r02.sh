#!/bin/bash
# Round-2 profile pass (run on the GPU box through gpurun): one ncu --set full
# capture of the default kernel of each profiled layer, and the launch list of a
# short default bench run.  Outputs under gpurun_out/ (summarised locally by
# tools/ncu_summary.py into profiles/r02/).
set -u
mkdir -p gpurun_out
for L in vgg_64_64_224_f16 r50_c256_14_f16 r50_c64_56_f16 r50_c256_14_f32 vgg_256_256_56_f16; do
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:"bfc_tc[23]" -c 1 \
      -o gpurun_out/prof_$L python tools/run_layer.py $L 2 > gpurun_out/prof_$L.log 2>&1
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_bench.csv python bench.py --steps 2 --warmup 3 > gpurun_out/bench_under_ncu.log 2>&1
ls -la gpurun_out/*.ncu-rep
