#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
: > gpurun_out/ab_ovh.jsonl
for c in 2 3 4; do timeout 600 python tools/sweep.py $c '[{}, {"flags":1}]' 7 >> gpurun_out/ab_ovh.jsonl 2>> gpurun_out/ab_ovh.err; done
timeout 1500 python -m pytest tests -q -m gpu --timeout 300 > gpurun_out/pytest_gpu.log 2>&1
