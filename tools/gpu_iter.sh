# one build->measure iteration: GPU parity suite, then bench lines for c2 (default), c3, c5
mkdir -p gpurun_out
T=${TAG:-it}
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -6 > gpurun_out/${T}_pytest.txt
timeout 300 python bench.py --steps 10 --no-cpu-baseline --no-e2e > gpurun_out/${T}_c2.json 2> gpurun_out/${T}_c2.err
for c in ${CFGS:-c3 c5}; do
  timeout 400 python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${T}_$c.json 2> gpurun_out/${T}_$c.err
done
cat gpurun_out/${T}_pytest.txt
for f in gpurun_out/${T}_c*.json; do python -c "
import json,sys; d=json.load(open('$f')); c=d['config']; print('$f', d['value'], d['ms_per_step'], json.dumps(c.get('stage_ms')), d['roofline']['frac'])" 2>/dev/null || tail -3 ${f%.json}.err; done
