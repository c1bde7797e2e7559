python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "long or bitmap or every_path or det or chunk or transpose or path_forcing" 2>&1 | tail -4
timeout 600 python bench.py --config c3 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02l_c3.json 2>&1
timeout 600 python bench.py --config c4 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02l_c4.json 2>&1
timeout 2400 python tools/ablation.py --configs c2,c4,c3,c5 --steps 3 --lb-sweep > gpurun_out/r02l_ablation.json 2> gpurun_out/r02l_ablation.err
