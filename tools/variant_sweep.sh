#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1
for c in 2 3 4; do
  timeout 300 python tools/sweep.py $c '[{}]' 9 > gpurun_out/sw11_c$c.jsonl 2> gpurun_out/sw11_c$c.err
done
RCM_LIB=build/librcm_trace.so timeout 300 python tools/trace_chain.py 2 "{}" gpurun_out/trace11_c2.npy > gpurun_out/trace11_c2.txt 2>&1
