#!/bin/bash
# full GPU test suite, sanitizer on tiny cases, default bench, leveled traces
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu --timeout 300 > gpurun_out/pytest_gpu.log 2>&1
timeout 600 compute-sanitizer --tool memcheck --print-limit 20 python tools/sanitize_cases.py > gpurun_out/sanitize_memcheck.log 2>&1; echo "exit $?" >> gpurun_out/sanitize_memcheck.log
for c in 4; do timeout 300 python tools/trace_leveled.py $c > gpurun_out/trlv_c$c.txt 2>&1; done
timeout 1200 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
