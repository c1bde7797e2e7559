# round-1 re-entry: parity suite + bench lines for every config at the current commit
mkdir -p gpurun_out
nproc > gpurun_out/s_nproc.txt
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/s_pytest.txt
timeout 300 python bench.py > gpurun_out/s_bench_c2.json 2> gpurun_out/s_bench_c2.err
for c in c1 c3 c4 c5; do
  timeout 400 python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/s_bench_$c.json 2> gpurun_out/s_bench_$c.err
done
tail -3 gpurun_out/s_pytest.txt; for c in c1 c2 c3 c4 c5; do head -c 400 gpurun_out/s_bench_$c.json; echo; done
