#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for c in 2 3 4; do timeout 300 python tools/trace_leveled.py $c > gpurun_out/trlv_c$c.txt 2>&1; done
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_solo$ -s 1 -c 1 -o gpurun_out/prof_c5 python tools/profile_c5.py 2048 2 > gpurun_out/ncu_c5.log 2>&1
