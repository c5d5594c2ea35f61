#!/bin/bash
# full GPU tests, leveled traces with the barrier split, chain vs leveled on C2-C4, C5 timing
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu --timeout 300 > gpurun_out/pytest_gpu.log 2>&1
for c in 2 3; do timeout 300 python tools/trace_leveled.py $c > gpurun_out/trlv_c$c.txt 2>&1; done
for c in 2 3 4; do
  timeout 300 python tools/sweep.py $c '[{}, {"flags": 32}]' 5 > gpurun_out/lv_c$c.jsonl 2> gpurun_out/lv_c$c.err
done
timeout 300 python tools/sweep_c5.py 7 > gpurun_out/c5ab.jsonl 2> gpurun_out/c5ab.err
