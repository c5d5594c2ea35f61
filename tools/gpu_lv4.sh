#!/bin/bash
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 900 python -m pytest tests -q -m gpu -x -k "leveled" --timeout 300 > gpurun_out/pt_lv.log 2>&1
for c in 2 3 4; do timeout 300 python tools/trace_leveled.py $c > gpurun_out/trlv_c$c.txt 2>&1; done
for c in 2 3 4; do
  timeout 300 python tools/sweep.py $c '[{"flags": 32}]' 5 > gpurun_out/lv_c$c.jsonl 2> gpurun_out/lv_c$c.err
done
