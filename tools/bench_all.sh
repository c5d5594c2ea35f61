#!/bin/bash
# Run the bench for every config and ncu captures of k_main (run under gpurun).
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt
for c in 1 2 3 4; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 > gpurun_out/bench_c$c.json 2> gpurun_out/bench_c$c.err
  timeout 600 python bench.py --config $c --impl reference --steps 3 --warmup 1 > gpurun_out/ref_c$c.json 2>> gpurun_out/bench_c$c.err
done
timeout 900 python bench.py --config 5 --steps 5 --warmup 2 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
timeout 600 python bench.py --config 5 --impl reference --steps 3 --warmup 1 > gpurun_out/ref_c5.json 2>> gpurun_out/bench_c5.err
for c in 3 4; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_main -s 1 -c 1 -o gpurun_out/prof_c$c python tools/profile_run.py $c 2 > gpurun_out/ncu_c$c.log 2>&1
done
