#!/bin/bash
# A/B of build variants (build/var/*.so) on the chain configs
mkdir -p gpurun_out
: > gpurun_out/ab_lib.jsonl
for c in ${AB_CFGS:-2 3 4}; do
  timeout 600 python tools/sweep.py $c '[{}]' 7 | sed 's/^/{"lib":"default",/;s/^{"lib":"default",{/{"lib":"default",/' >> gpurun_out/ab_lib.jsonl 2>> gpurun_out/ab_lib.err
  for lib in build/var/*.so; do
    RCM_LIB=$lib timeout 600 python tools/sweep.py $c '[{}]' 7 | sed "s#^{#{\"lib\":\"$lib\",#" >> gpurun_out/ab_lib.jsonl 2>> gpurun_out/ab_lib.err
  done
done
