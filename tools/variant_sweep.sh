#!/bin/bash
mkdir -p gpurun_out
for lib in base mba mbb; do
  for c in 1 2; do
    RCM_LIB=build/librcm_$lib.so timeout 300 python tools/sweep.py $c '[{}]' 7 > gpurun_out/sw17_${lib}_c$c.jsonl 2> gpurun_out/sw17_${lib}_c$c.err
  done
done
