#!/bin/bash
# build, smoke, all GPU tests (per-test timeout), C5 bench without secondary lines
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 600 python bench.py --steps 5 --warmup 2 --no-secondary > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
timeout 1500 python -m pytest tests -q -m gpu --timeout 240 --durations=25 ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1
