# per-kernel launch list (ncu, serialised, cold L2) for the configs in $CFGS; only libspeck kernels
mkdir -p gpurun_out /tmp/rep
B="--steps 1 --warmup 3 --no-e2e --no-cpu-baseline"
for c in ${CFGS:-c3 c5}; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:^k_" --csv --log-file /tmp/rep/l_$c.csv python bench.py --config $c $B > /dev/null 2>&1
  python tools/ncu_launches.py /tmp/rep/l_$c.csv 40 > gpurun_out/${TAG:-l}_launch_$c.txt 2>&1
  cp /tmp/rep/l_$c.csv gpurun_out/${TAG:-l}_launch_$c.csv
done
