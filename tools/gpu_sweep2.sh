#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
: > gpurun_out/sweep2.jsonl
timeout 300 python tools/sweep_c5.py 5 >> gpurun_out/sweep2.jsonl 2>> gpurun_out/sweep2.err
for lib in build/var/librcm_*.so; do RCM_LIB=$lib timeout 300 python tools/sweep_c5.py 5 >> gpurun_out/sweep2.jsonl 2>> gpurun_out/sweep2.err; done
timeout 900 python -m pytest tests -q -m gpu --timeout 240 -k "${PYTEST_K:-batched or c5 or solo or tiny or edge or smoke}" > gpurun_out/pytest_q.log 2>&1
