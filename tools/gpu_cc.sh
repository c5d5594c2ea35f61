#!/bin/bash
# components phase out of line (LIB) vs the current build: C2-C4 chain
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for i in 1 2; do
  for lib in default $LIB; do
    if [ $lib = default ]; then L=""; else L=build/librcm_$lib.so; fi
    for c in 2 3 4; do RCM_LIB=$L timeout 300 python tools/sweep.py $c '[{}]' 5 >> gpurun_out/cc_${lib}.jsonl 2>> gpurun_out/cc.err; done
  done
done
