for L in 1 2 4; do
  SPECK_NVCC_EXTRA=-DSPECK_ESC_LAMBDA=$L python -m paper_conf_ppopp_pargerwms20_b200.build --force | tail -1
  for e in 1 2; do
    timeout 600 python bench.py --config c5 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --opt bucket_sort=$e > gpurun_out/r02h_c5_L${L}_esc$e.json 2>&1
  done
  timeout 600 python bench.py --config c2 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --opt bucket_sort=2 > gpurun_out/r02h_c2_L${L}_esc2.json 2>&1
done
