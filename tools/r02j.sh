python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 2400 python -m pytest tests/test_gpu_parity.py -q -x --durations=15 2>&1 | tail -30
timeout 600 python bench.py --config c5 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02j_c5.json 2>&1
timeout 600 python bench.py --config c2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02j_c2.json 2>&1
