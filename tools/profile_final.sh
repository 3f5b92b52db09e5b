#!/bin/bash
# Final round-2 evidence on the GPU box (gpurun, repo root): the default bench line,
# the ncu launch list of the default bench command, one ncu --set full capture of the
# default kernel per profiled layer, and the 2-rank plumbing line.  Summarise here with
#   python tools/ncu_summary.py gpurun_out/prof_<layer>.ncu-rep; python tools/traffic.py --final
set -u
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
echo "bench rc=$?"
for L in vgg_64_64_224_f16 vgg_64_128_112_f16 vgg_128_128_112_f16 vgg_256_256_56_f16 vgg_512_512_28_f16 r50_c64_56_f16 r50_c256_14_f16 r50_c512_7_f16 r50_c256_14_f32; do
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:"bfc_tc[23]" -c 1 \
      -o gpurun_out/prof_$L python tools/run_layer.py $L 2 > gpurun_out/prof_$L.log 2>&1
  echo "ncu $L rc=$?"
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_bench.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/bench_under_ncu.log 2>&1
echo "launch list rc=$?"
timeout 600 python bench.py --gpus 2 --workload r50l3 --steps 5 --warmup 3 > gpurun_out/bench_2rank.json 2> gpurun_out/bench_2rank.err
echo "2-rank rc=$?"
ls -la gpurun_out/*.ncu-rep
