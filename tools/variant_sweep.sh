#!/bin/bash
# Parity of the default build, then compare build variants on C2-C4, then a C2 timeline.
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1
for lib in f1 f4 f8; do
  for c in 2 3 4; do
    RCM_LIB=build/librcm_$lib.so timeout 300 python tools/sweep.py $c '[{}]' 7 > gpurun_out/sw3_${lib}_c$c.jsonl 2> gpurun_out/sw3_${lib}_c$c.err
  done
done
RCM_LIB=build/librcm_f4_trace.so timeout 300 python tools/trace_timeline.py 2 '{}' 25 > gpurun_out/timeline_f4_c2.txt 2>&1
RCM_LIB=build/librcm_f4_trace.so timeout 300 python tools/trace_chain.py 2 > gpurun_out/trace_f4_c2.txt 2>&1
