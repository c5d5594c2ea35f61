#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 300 python tools/sweep_c5.py 5 > gpurun_out/sweep_now.jsonl 2> gpurun_out/sweep_now.err
timeout 900 python -m pytest tests -q -m gpu --timeout 240 -k "${PYTEST_K:-batched or c5 or solo or tiny or edge or smoke}" > gpurun_out/pytest_q.log 2>&1
