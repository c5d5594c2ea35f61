#!/bin/bash
# multi-rank harness check on one GPU: two ranks sharing the device over gloo
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
RCM_BENCH_BACKEND=gloo RCM_BENCH_SHARE_DEVICE=1 timeout 1200 python bench.py --gpus 2 --steps 3 --warmup 3 > gpurun_out/bench_mr2.json 2> gpurun_out/bench_mr2.err
