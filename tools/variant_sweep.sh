#!/bin/bash
mkdir -p gpurun_out
RCM_LIB=build/librcm_trace.so timeout 300 python tools/trace_timeline.py 2 '{}' 25 > gpurun_out/timeline_c2.txt 2>&1
timeout 600 python tools/sweep.py 2 '[{}, {"batch_nodes": 96, "temp_elems": 6144}, {"batch_nodes": 128, "temp_elems": 6144}, {"batch_nodes": 256, "temp_elems": 6144}, {"batch_nodes": 256, "temp_elems": 8192}, {"batch_nodes": 160, "temp_elems": 4608}]' 7 > gpurun_out/sw4_c2.jsonl 2> gpurun_out/sw4_c2.err
timeout 600 python tools/sweep.py 3 '[{}, {"batch_nodes": 128}, {"batch_nodes": 512}, {"batch_nodes": 256, "temp_elems": 6144}]' 7 > gpurun_out/sw4_c3.jsonl 2> gpurun_out/sw4_c3.err
timeout 600 python tools/sweep.py 4 '[{}, {"batch_nodes": 128}, {"batch_nodes": 512}]' 7 > gpurun_out/sw4_c4.jsonl 2> gpurun_out/sw4_c4.err
