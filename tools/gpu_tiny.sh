# A/B of the numeric tiny-row geometry (variants/libspeck_tN.so: N CTAs/SM with 2 KB regions)
mkdir -p gpurun_out
T=${TAG:-ty}
L=paper_conf_ppopp_pargerwms20_b200/libspeck.so
cp $L /tmp/libspeck_orig.so
for v in ${VARIANTS:-base t5 t6}; do
  cp variants/libspeck_$v.so $L
  for c in c2 c5; do
    st=3; [ $c = c2 ] && st=10
    timeout 400 python bench.py --config $c --steps $st --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${T}_${c}_$v.json 2> gpurun_out/${T}_${c}_$v.err
  done
  timeout 300 python -m pytest tests -m gpu -x -q 2>&1 | tail -2 > gpurun_out/${T}_pytest_$v.txt
done
cp /tmp/libspeck_orig.so $L
for f in gpurun_out/${T}_c*.json; do python -c "
import json; d=json.load(open('$f')); c=d['config']; print('$f', d['value'], d['ms_per_step'], json.dumps(c.get('stage_ms')))" 2>/dev/null || tail -3 ${f%.json}.err; done
cat gpurun_out/${T}_pytest_*.txt
