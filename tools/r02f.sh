python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "not full_size" 2>&1 | tail -4
for e in 0 1 2; do
  timeout 600 python bench.py --config c5 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --opt bucket_sort=$e > gpurun_out/r02f_c5_esc$e.json 2>&1
done
timeout 600 python bench.py --config c2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02f_c2.json 2>&1
timeout 600 python bench.py --config c3 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02f_c3.json 2>&1
