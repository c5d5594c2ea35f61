#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -x -q -m gpu -k "tiny or full or stress" > gpurun_out/pytest_gpu_w1.log 2>&1
for i in 1 2; do
for lib in base w1; do
  for c in 2 3 4; do
    RCM_LIB=build/librcm_$lib.so timeout 300 python tools/sweep.py $c '[{}]' 7 > gpurun_out/sw19_${lib}_c${c}_$i.jsonl 2> gpurun_out/sw19_${lib}_c$c.err
  done
done
done
