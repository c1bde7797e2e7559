#!/bin/bash
# Quick GPU check of the working tree: selected parity tests + one bench line per config.
#   TAG=… TESTK="pytest -k expr" CFGS="c5 …" bash tools/gpu_check.sh
python paper_conf_ppopp_pargerwms20_b200/build.py 2>&1 | tail -1
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "${TESTK:-not full_size}" > gpurun_out/${TAG}_pytest.txt 2>&1
tail -3 gpurun_out/${TAG}_pytest.txt
for c in ${CFGS:-c5}; do
  timeout 600 python bench.py --config $c --steps ${STEPS:-5} --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.json 2>/tmp/b.err
  C=$c python - >> gpurun_out/${TAG}_bench.txt <<'PY'
import json, os
d = json.loads(open('/tmp/b.json').read().strip().splitlines()[-1])
print(f"== {os.environ['C']}: {d['ms_per_step']} ms  stages {d['config']['stage_ms']}")
for k in d['roofline']['kernels']: print('   ', k['kernel'], k['problem'], k['bin'], k['ms'])
PY
done
cat gpurun_out/${TAG}_bench.txt
