#!/bin/bash
# C2 chain-path sweep: batch limits, blocks per SM, discovery width
mkdir -p gpurun_out
: > gpurun_out/sweep_chain.jsonl
timeout 600 python tools/sweep.py 2 '[{}, {"batch_nodes":64}, {"batch_nodes":96}, {"batch_nodes":128}, {"blocks_per_sm":1}, {"blocks_per_sm":1,"batch_nodes":96}, {"batch_nodes":96,"temp_elems":3072}]' 5 >> gpurun_out/sweep_chain.jsonl 2>> gpurun_out/sweep_chain.err
RCM_LIB=build/var/librcm_du8.so timeout 300 python tools/sweep.py 2 '[{"blocks_per_sm":1}, {"blocks_per_sm":1,"batch_nodes":128}, {"blocks_per_sm":1,"batch_nodes":256}]' 5 >> gpurun_out/sweep_chain.jsonl 2>> gpurun_out/sweep_chain.err
