#!/bin/bash
# r01d second sweep: temp budget T (shared memory vs L1) on C3/C4, B_s on C2, C5 T.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/sw_build.log 2>&1
G2='[{},{"batch_nodes":176,"temp_elems":6144},{"batch_nodes":192,"temp_elems":6144},{"batch_nodes":224,"temp_elems":6144},{"batch_nodes":256,"temp_elems":6144},{"batch_nodes":192,"temp_elems":8192},{"batch_nodes":192,"temp_elems":5120}]'
GS='[{},{"temp_elems":4608},{"temp_elems":5632},{"temp_elems":6656},{"temp_elems":7680},{"temp_elems":8704},{"batch_nodes":384,"temp_elems":6656},{"batch_nodes":384,"temp_elems":8704},{"batch_nodes":320,"temp_elems":7680}]'
timeout 600 python tools/sweep.py 2 "$G2" 7 > gpurun_out/sw2_c2.jsonl 2> gpurun_out/sw2_c2.err
timeout 600 python tools/sweep.py 3 "$GS" 5 > gpurun_out/sw2_c3.jsonl 2> gpurun_out/sw2_c3.err
timeout 600 python tools/sweep.py 4 "$GS" 5 > gpurun_out/sw2_c4.jsonl 2> gpurun_out/sw2_c4.err
for p in '{}' '{"temp_elems":6656}' '{"temp_elems":4608}'; do
  RCM_PLAN="$p" timeout 600 python bench.py --config 5 --steps 3 --warmup 3 >> gpurun_out/sw2_c5.jsonl 2>> gpurun_out/sw2_c5.err
done
