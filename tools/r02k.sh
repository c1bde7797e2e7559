python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 2400 python -m pytest tests/test_gpu_parity.py tests/test_dist_gpu.py -q --durations=12 2>&1 | tail -25
timeout 900 python bench.py --config c5 --steps 3 --warmup 3 > gpurun_out/r02k_c5.json 2> gpurun_out/r02k_c5.err
