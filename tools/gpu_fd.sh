#!/bin/bash
# capped first batch of each generator (RCM_FIRST_DIV 4 / 8) vs default: C2-C4 chain timing + parity tests
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for i in 1 2; do
  for lib in default fd4 fd8; do
    if [ $lib = default ]; then L=""; else L=build/librcm_$lib.so; fi
    for c in 2 3 4; do RCM_LIB=$L timeout 300 python tools/sweep.py $c '[{}]' 5 >> gpurun_out/fd_${lib}.jsonl 2>> gpurun_out/fd.err; done
  done
done
for lib in fd4 fd8; do
  RCM_LIB=build/librcm_$lib.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "chain or full_config or stress or tiny or components" --timeout 600 > gpurun_out/pt_$lib.log 2>&1
done
