set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -15
for e in 0 1 2; do
  timeout 600 python bench.py --config c5 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --opt bucket_sort=$e 2>&1 | tail -1 | cut -c1-900
done
