python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "not full_size and not c4_full" 2>&1 | tail -3
for U in 1 2; do
  SPECK_NVCC_EXTRA=-DSPECK_WARP_U=$U python -m paper_conf_ppopp_pargerwms20_b200.build --force | tail -1
  timeout 600 python bench.py --config c5 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02i_c5_U$U.json 2>&1
  timeout 600 python bench.py --config c2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02i_c2_U$U.json 2>&1
done
