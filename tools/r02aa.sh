python paper_conf_ppopp_pargerwms20_b200/build.py 2>&1 | tail -1
timeout 120 python tools/repro_small.py c3 2>&1 | grep "^ok\|^failed" > gpurun_out/r02aa_repro.txt
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "not full_size" > gpurun_out/r02aa_pytest.txt 2>&1
tail -3 gpurun_out/r02aa_pytest.txt
for o in "" "--opt bucket_sort=2"; do
  timeout 600 python bench.py --config c5 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline $o > /tmp/b.json 2>/tmp/b.err
  O="$o" python - >> gpurun_out/r02aa_ab.txt <<'PY'
import json, os
d = json.loads(open('/tmp/b.json').read().strip().splitlines()[-1])
print(f"== staged {os.environ['O']}: {d['ms_per_step']} ms  stages {d['config']['stage_ms']}")
for k in d['roofline']['kernels']: print('   ', k['kernel'], k['problem'], k['bin'], k['ms'])
PY
done
