#!/bin/bash
# A/B of discovery unroll (RCM_DISC_U 4 / 8 / 12) on C2-C4, chain and leveled
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for c in 2 3 4; do
  for lib in default du8 du12; do
    if [ $lib = default ]; then L=""; else L=build/librcm_$lib.so; fi
    RCM_LIB=$L timeout 300 python tools/sweep.py $c '[{}, {"flags": 32}]' 5 > gpurun_out/du_${lib}_c$c.jsonl 2> gpurun_out/du_${lib}_c$c.err
  done
done
