#!/bin/bash
# round-2 measurement (r02e): smoke, GPU tests, default bench (C5 + C4/C3/C2 with leveled),
# reference arm, C1 line, C5 launch list, ncu --set full of k_solo (C5) and k_main (C2 chain / leveled)
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,driver_version,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu --timeout 300 > gpurun_out/pytest_gpu.log 2>&1
timeout 1200 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
timeout 900 python bench.py --impl reference > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
timeout 600 python bench.py --config 1 --steps 10 --warmup 3 > gpurun_out/bench_c1.json 2> gpurun_out/bench_c1.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/c5_launches.csv python bench.py --steps 2 --warmup 3 --no-secondary > gpurun_out/c5_ncu_bench.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_solo$ -s 1 -c 1 -o gpurun_out/prof_c5 python tools/profile_c5.py 8192 2 > gpurun_out/ncu_c5.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_main -s 1 -c 1 -o gpurun_out/prof_c2 python tools/profile_run.py 2 2 > gpurun_out/ncu_c2.log 2>&1
RCM_PLAN='{"flags": 32}' timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_main -s 1 -c 1 -o gpurun_out/prof_c2lv python tools/profile_run.py 2 2 > gpurun_out/ncu_c2lv.log 2>&1
