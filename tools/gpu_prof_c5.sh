#!/bin/bash
# ncu of the C5 batched launch: launch list of the bench command + one --set full capture of k_solo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/c5_launches.csv python bench.py --steps 2 --warmup 1 --no-secondary > gpurun_out/c5_ncu_bench.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_solo$ -s 1 -c 1 -o gpurun_out/prof_c5 python tools/profile_c5.py ${NMATS:-4096} 2 > gpurun_out/ncu_c5.log 2>&1
