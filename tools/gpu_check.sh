#!/bin/bash
# build, smoke, C5 timing (sweep_c5), all GPU tests, optional sanitizer
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 300 python tools/sweep_c5.py 5 > gpurun_out/sweep_now.jsonl 2> gpurun_out/sweep_now.err
timeout 1500 python -m pytest tests -q -m gpu --timeout 300 --durations=15 ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1
if [ -n "$SANITIZE" ]; then bash tools/gpu_sanitize.sh; fi
