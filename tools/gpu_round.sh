#!/bin/bash
# Round measurement: smoke, GPU tests, bench for every config (+ reference arm
# on C2), C2 launch list, one ncu --set full capture of k_main on C2, variants.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1
for c in 2 3 4 1; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 > gpurun_out/bench_c$c.json 2> gpurun_out/bench_c$c.err
done
timeout 900 python bench.py --config 5 --steps 5 --warmup 3 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/ref_c2.json 2> gpurun_out/ref_c2.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/c2_launches.csv python bench.py --config 2 --steps 2 --warmup 3 > gpurun_out/c2_ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_main -s 1 -c 1 -o gpurun_out/prof_c2 python tools/profile_run.py 2 2 > gpurun_out/ncu_c2.log 2>&1
for lib in base; do
  RCM_LIB=build/librcm_$lib.so timeout 300 python tools/sweep.py 2 '[{}]' 9 > gpurun_out/sw13_${lib}_c2.jsonl 2> gpurun_out/sw13_${lib}_c2.err
done
