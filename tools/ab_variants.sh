#!/bin/bash
# A/B of compile-time variants on one box: VARIANTS="name=flags;name=flags", CFGS, TAG.
# Each variant: forced rebuild, one bench line per config (no e2e/cpu) -> gpurun_out/${TAG}_ab.txt
# TESTS=1 first runs the fast GPU parity suite on the default build.
set -u
out=gpurun_out/${TAG}_ab.txt
if [ "${TESTS:-0}" = 1 ]; then
  python paper_conf_ppopp_pargerwms20_b200/build.py --force 2>&1 | tail -1
  timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "${TESTK:-not full_size}" > gpurun_out/${TAG}_pytest.txt 2>&1
  tail -3 gpurun_out/${TAG}_pytest.txt
fi
IFS=";" read -ra VS <<< "${VARIANTS}"
for v in "${VS[@]}"; do
  name=${v%%=*}; flags=${v#*=}
  SPECK_NVCC_EXTRA="$flags" python paper_conf_ppopp_pargerwms20_b200/build.py --force 2>&1 | tail -1
  for c in ${CFGS:-c5}; do
    timeout 600 python bench.py --config $c --steps ${STEPS:-3} --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.json 2>/tmp/b.err
    NAME=$name CFG=$c python - >> $out <<'PY'
import json, os
try:
    d = json.loads(open('/tmp/b.json').read().strip().splitlines()[-1])
    print(f"== {os.environ['NAME']} {os.environ['CFG']}: {d['ms_per_step']} ms  stages {d['config']['stage_ms']}")
    for k in d['roofline']['kernels']: print('   ', k['kernel'], k['problem'], k['bin'], k['ms'])
except Exception as ex:
    print(f"== {os.environ['NAME']} {os.environ['CFG']}: FAILED {ex}"); print(open('/tmp/b.err').read()[-2000:])
PY
  done
done
python paper_conf_ppopp_pargerwms20_b200/build.py --force 2>&1 | tail -1
echo done
