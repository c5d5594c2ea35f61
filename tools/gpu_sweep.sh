#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
: > gpurun_out/sweep_c5.jsonl
for lib in build/var/librcm_*.so; do
  RCM_LIB=$lib timeout 300 python tools/sweep_c5.py 5 >> gpurun_out/sweep_c5.jsonl 2>> gpurun_out/sweep_c5.err
done
timeout 300 python tools/sweep_c5.py 5 >> gpurun_out/sweep_c5.jsonl 2>> gpurun_out/sweep_c5.err
