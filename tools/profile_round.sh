#!/bin/bash
# Round-end evidence on the GPU box (run under gpurun from the repo root):
# bench lines (FP16 / BF16 / FP32 ResNet-50, FP16 VGG-16, FP32 wide), the ncu launch list of the
# default bench command, and one ncu --set full capture per ResNet-50 layer
# for the FP16 and FP32 fused kernels.  Summarise here with
#   python tools/ncu_summary.py gpurun_out/prof_f16.ncu-rep; python tools/traffic.py
mkdir -p gpurun_out
timeout 600 python bench.py > gpurun_out/bench_f16.json 2> gpurun_out/bench_f16.err
timeout 600 python bench.py --dtype f32 --no-cpu-baseline > gpurun_out/bench_f32.json 2> gpurun_out/bench_f32.err
timeout 600 python bench.py --workload vgg --no-cpu-baseline > gpurun_out/bench_vgg.json 2> gpurun_out/bench_vgg.err
timeout 600 python bench.py --dtype bf16 --no-cpu-baseline > gpurun_out/bench_bf16.json 2> gpurun_out/bench_bf16.err
timeout 600 python bench.py --dtype f32 --workload wide --no-cpu-baseline > gpurun_out/bench_wide.json 2> gpurun_out/bench_wide.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_fp16_r50.csv \
   python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bfc_f16 -s 4 -c 4 \
   -o gpurun_out/prof_f16 python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_f16.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bfc_f32 -s 4 -c 4 \
   -o gpurun_out/prof_f32 python bench.py --dtype f32 --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_f32.log 2>&1
tail -n 2 gpurun_out/*.log
