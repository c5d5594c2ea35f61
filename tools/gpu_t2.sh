mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_edge.py tests/test_gpu_c5_full.py -q -m gpu --durations=15 > gpurun_out/pytest_edge.log 2>&1
