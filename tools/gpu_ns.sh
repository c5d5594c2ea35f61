#!/bin/bash
# grid-barrier polling without __nanosleep (ns0) vs the current build: chain and leveled on C2-C4, GL via bench secondary
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for lib in v0 ns0; do
  if [ $lib = v0 ]; then L=""; else L=build/librcm_$lib.so; fi
  for c in 2 3 4; do
    RCM_LIB=$L timeout 300 python tools/sweep.py $c '[{}, {"flags": 32}]' 5 > gpurun_out/ns_${lib}_c$c.jsonl 2> gpurun_out/ns_${lib}_c$c.err
  done
  RCM_LIB=$L timeout 300 python tools/trace_leveled.py 2 > gpurun_out/ns_${lib}_trlv2.txt 2>&1
done
