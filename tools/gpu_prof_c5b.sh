#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_solo$ -s 1 -c 1 -o gpurun_out/prof_c5b python tools/profile_c5.py ${NMATS:-4096} 2 > gpurun_out/ncu_c5b.log 2>&1
