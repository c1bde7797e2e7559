python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "long or bitmap" 2>&1 | tail -3
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "every_path" -s 2>&1 | grep -E "never|passed|failed"
timeout 600 python bench.py --config c3 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02n_c3.json 2>&1
timeout 600 python bench.py --config c4 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02n_c4.json 2>&1
