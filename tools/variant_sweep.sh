#!/bin/bash
mkdir -p gpurun_out
for lib in base npf; do
  for c in 2 3 4 1; do
    RCM_LIB=build/librcm_$lib.so timeout 300 python tools/sweep.py $c '[{}]' 9 > gpurun_out/sw15_${lib}_c$c.jsonl 2> gpurun_out/sw15_${lib}_c$c.err
  done
done
