python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "not full_size" 2>&1 | tail -2
for c in c2 c5; do
  timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02s_$c.json 2>&1
done
timeout 900 python tools/ablation.py --configs "" --steps 3 --lb-sweep > gpurun_out/r02s_lbsweep.jsonl 2> gpurun_out/r02s_lbsweep.err
