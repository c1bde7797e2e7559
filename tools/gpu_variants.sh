# A/B of library variants (variants/libspeck_<v>.so) on C2, same box, back to back
mkdir -p gpurun_out
T=${TAG:-va}
L=paper_conf_ppopp_pargerwms20_b200/libspeck.so
cp $L /tmp/libspeck_orig.so
for c in ${CFGS:-c2}; do for r in 1 2; do
for v in ${VARIANTS}; do
  cp variants/libspeck_$v.so $L
  st=20; [ $c != c2 ] && st=3
  timeout 300 python bench.py --config $c --steps $st --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/${T}_${c}_${v}_$r.json 2> gpurun_out/${T}_${c}_${v}_$r.err
done
done
done
cp /tmp/libspeck_orig.so $L
for f in gpurun_out/${T}_c*.json; do python -c "
import json; d=json.load(open('$f')); c=d['config']; print('$f', d['value'], d['ms_per_step'], json.dumps(c.get('stage_ms')))" 2>/dev/null || tail -3 ${f%.json}.err; done
