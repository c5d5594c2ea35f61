#!/bin/bash
# C5 timing, current build vs a variant library (LIB), alternating, plus parity sample
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for i in 1 2; do
  timeout 300 python tools/sweep_c5.py 7 >> gpurun_out/c5lib_default.jsonl 2>> gpurun_out/c5lib.err
  RCM_LIB=build/librcm_${LIB}.so timeout 300 python tools/sweep_c5.py 7 >> gpurun_out/c5lib_${LIB}.jsonl 2>> gpurun_out/c5lib.err
done
