#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
: > gpurun_out/sweep_l2.jsonl
for g in 0 32 64 128; do
  if [ $g = 0 ]; then timeout 300 python tools/sweep_c5.py 5 >> gpurun_out/sweep_l2.jsonl 2>&1;
  else RCM_L2_FETCH=$g timeout 300 python tools/sweep_c5.py 5 >> gpurun_out/sweep_l2.jsonl 2>&1; fi
done
RCM_L2_FETCH=32 timeout 600 ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct -k regex:k_solo$ -s 1 -c 1 python tools/profile_c5.py 4096 2 > gpurun_out/ncu_l2_32.log 2>&1
timeout 600 ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct -k regex:k_solo$ -s 1 -c 1 python tools/profile_c5.py 4096 2 > gpurun_out/ncu_l2_def.log 2>&1
