for P in 1 0; do
  SPECK_NVCC_EXTRA=-DSPECK_PERSIST=$P python -m paper_conf_ppopp_pargerwms20_b200.build --force | tail -1
  for c in c5 c3 c2; do
    timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02q_${c}_P$P.json 2>&1
  done
done
python -m paper_conf_ppopp_pargerwms20_b200.build --force | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "not full_size" 2>&1 | tail -2
