#!/bin/bash
# C5 timing of the current build + batched parity tests
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 300 python tools/sweep_c5.py 7 > gpurun_out/c5ab.jsonl 2> gpurun_out/c5ab.err
timeout 900 python -m pytest tests -q -m gpu -x -k "batched or c5 or solo or tiny" --timeout 600 > gpurun_out/pt_c5.log 2>&1
timeout 300 python tools/sweep_c5.py 7 >> gpurun_out/c5ab.jsonl 2>> gpurun_out/c5ab.err
