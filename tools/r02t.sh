#!/bin/bash
# Session re-entry check at HEAD: GPU suite + C5/C2/C3 bench lines (no e2e) for the perf baseline.
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
( time timeout 1500 python -m pytest tests -m gpu -q -x --durations=10 ) > gpurun_out/r02t_pytest_gpu.txt 2>&1
for c in c5 c2 c3; do
  timeout 600 python bench.py --config $c --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02t_$c.json 2> gpurun_out/r02t_$c.err
done
echo done
