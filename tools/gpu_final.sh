#!/bin/bash
# Round measurement after a default change: smoke, GPU tests, C1-C5 bench lines,
# reference arm, C2 launch list, ncu --set full of k_main on C2 and C3.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 1200 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1
for c in 2 3 4 1; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 > gpurun_out/bench_c$c.json 2> gpurun_out/bench_c$c.err
done
timeout 900 python bench.py --config 5 --steps 5 --warmup 3 > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/ref_c2.json 2> gpurun_out/ref_c2.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/c2_launches.csv python bench.py --config 2 --steps 2 --warmup 3 > gpurun_out/c2_ncu_bench.log 2>&1
for c in 2 3; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_main -s 1 -c 1 -o gpurun_out/prof_c$c python tools/profile_run.py $c 2 > gpurun_out/ncu_c$c.log 2>&1
done
