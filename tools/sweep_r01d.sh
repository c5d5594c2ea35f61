#!/bin/bash
# r01d plan-option sweep (B_s, T, blocks per SM) on C2-C4; parity checked per point.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/sw_build.log 2>&1
G2='[{},{"batch_nodes":96,"temp_elems":4096},{"batch_nodes":128,"temp_elems":4096},{"batch_nodes":128,"temp_elems":6144},{"batch_nodes":192,"temp_elems":6144},{"batch_nodes":160,"temp_elems":6144,"blocks_per_sm":1},{"batch_nodes":160,"temp_elems":6144,"blocks_per_sm":3},{"batch_nodes":128,"temp_elems":4096,"blocks_per_sm":3},{"batch_nodes":96,"temp_elems":3072,"blocks_per_sm":4},{"batch_nodes":64,"temp_elems":2048,"blocks_per_sm":4}]'
GS='[{},{"batch_nodes":128},{"batch_nodes":192},{"batch_nodes":384},{"blocks_per_sm":1},{"blocks_per_sm":3},{"batch_nodes":128,"blocks_per_sm":3},{"batch_nodes":128,"blocks_per_sm":4}]'
timeout 600 python tools/sweep.py 2 "$G2" 7 > gpurun_out/sw_c2.jsonl 2> gpurun_out/sw_c2.err
timeout 600 python tools/sweep.py 3 "$GS" 5 > gpurun_out/sw_c3.jsonl 2> gpurun_out/sw_c3.err
timeout 600 python tools/sweep.py 4 "$GS" 5 > gpurun_out/sw_c4.jsonl 2> gpurun_out/sw_c4.err
