#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 600 python -m pytest tests/test_gpu_edge.py -q -m gpu -k "host_pipeline" --timeout 300 > gpurun_out/pytest_q.log 2>&1
for c in 8 16 4; do RCM_E2E_CHUNKS=$c timeout 600 python bench.py --steps 3 --warmup 2 --no-secondary > gpurun_out/bench_e2e_$c.json 2> gpurun_out/bench_e2e_$c.err; done
