#!/bin/bash
# ESC knob sweep on C5 (compile-time macros): per-kernel times per variant.
for v in "" "-DSPECK_ESC_RATIO_PCT=110" "-DSPECK_ESC_RATIO_PCT=102" "-DSPECK_ESC_LAMBDA=1" "-DSPECK_ESC_LAMBDA=4"; do
  SPECK_NVCC_EXTRA="$v" python paper_conf_ppopp_pargerwms20_b200/build.py --force 2>&1 | tail -1
  echo "== variant '$v'" >> gpurun_out/r02v_sweep.txt
  timeout 600 python bench.py --config ${CFG:-c5} --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.json 2>/tmp/b.err
  python - >> gpurun_out/r02v_sweep.txt <<'PY'
import json
d=json.loads(open('/tmp/b.json').read().strip().splitlines()[-1])
print(d['ms_per_step'], d['config']['stage_ms'])
for k in d['roofline']['kernels']: print('   ', k['kernel'], k['bin'], k['ms'])
PY
done
echo done
