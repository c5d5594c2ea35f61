#!/bin/bash
# which round-2 change moved k_main<2,0> spills onto the chain's hot path: C2-C4 time and
# ncu local-memory sectors of k_main on C2 for the current build (v0) and variants
# v1 = old GL finder + new barrier, v2 = new GL + old barrier, v3 = old GL + old barrier
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for lib in ${LIBS:-v0 v1 v2 v3}; do
  if [ $lib = v0 ]; then L=""; else L=build/librcm_$lib.so; fi
  for c in 2 3 4; do
    RCM_LIB=$L timeout 300 python tools/sweep.py $c '[{}]' 5 > gpurun_out/sp_${lib}_c$c.jsonl 2> gpurun_out/sp_${lib}_c$c.err
  done
  RCM_LIB=$L timeout 600 ncu --metrics gpu__time_duration.sum,l1tex__t_sectors_pipe_lsu_mem_local_op_ld.sum,l1tex__t_sectors_pipe_lsu_mem_local_op_st.sum,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum --clock-control none -k regex:k_main -c 2 --csv python tools/profile_run.py 2 2 > gpurun_out/sp_${lib}_ncu.csv 2> gpurun_out/sp_${lib}_ncu.err
done
