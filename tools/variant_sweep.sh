#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1
for c in 2 3 4; do
  timeout 300 python tools/sweep.py $c '[{}, {"flags": 64}]' 9 > gpurun_out/sw12_c$c.jsonl 2> gpurun_out/sw12_c$c.err
done
RCM_LIB=build/librcm_trace.so timeout 300 python tools/trace_timeline.py 2 "{}" 25 > gpurun_out/timeline12_c2.txt 2>&1
