#!/bin/bash
# C5 timing of several variant libraries (LIBS) against the current build, interleaved
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for i in 1 2; do
  timeout 300 python tools/sweep_c5.py 7 >> gpurun_out/c5libs.jsonl 2>> gpurun_out/c5libs.err
  for lib in $LIBS; do
    RCM_LIB=build/librcm_${lib}.so timeout 300 python tools/sweep_c5.py 7 >> gpurun_out/c5libs.jsonl 2>> gpurun_out/c5libs.err
  done
done
