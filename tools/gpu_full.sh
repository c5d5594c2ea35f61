#!/bin/bash
# Round checkpoint: smoke, all GPU tests, default bench (C5 + secondary C4/C2), reference arm,
# C1/C3 lines, bench launch list under ncu, ncu --set full of k_solo (C5) and k_main (C2, C4).
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
timeout 600 python bench.py --impl reference > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
for c in 1 3; do timeout 600 python bench.py --config $c --steps 10 --warmup 3 > gpurun_out/bench_c$c.json 2> gpurun_out/bench_c$c.err; done
timeout 1500 python -m pytest tests -q -m gpu --timeout 300 --durations=20 > gpurun_out/pytest_gpu.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/c5_launches.csv python bench.py --steps 2 --warmup 1 --no-secondary > gpurun_out/c5_ncu_bench.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_solo$ -s 1 -c 1 -o gpurun_out/prof_c5_full python tools/profile_c5.py 8192 2 > gpurun_out/ncu_c5_full.log 2>&1
for c in 2 4 3; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_main -s 2 -c 1 -o gpurun_out/prof_c$c python tools/profile_run.py $c 3 > gpurun_out/ncu_c$c.log 2>&1
done
