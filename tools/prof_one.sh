# full ncu capture of one kernel (regex K, config CFG) + launch list of CFG; TAG names outputs
rm -rf /tmp/rep; mkdir -p gpurun_out /tmp/rep
B="--steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
if [ -n "$LAUNCHES" ]; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:^k_" --csv --log-file /tmp/rep/l.csv python bench.py --config $CFG $B > /dev/null 2>&1
  python tools/ncu_launches.py /tmp/rep/l.csv 40 > gpurun_out/${TAG}_launch.txt 2>&1
fi
i=0
IFS=";" read -ra KS <<< "$K"
for k in "${KS[@]}"; do
  timeout 900 ncu --set full --clock-control none --import-source on -k "regex:$k" --kernel-name-base demangled -c 1 -o /tmp/rep/k$i python bench.py --config $CFG $B > gpurun_out/${TAG}_k$i.log 2>&1
  python tools/ncu_summary.py /tmp/rep/k$i.ncu-rep 0 > gpurun_out/${TAG}_k$i.txt 2>&1
  cp /tmp/rep/k$i.ncu-rep gpurun_out/${TAG}_k$i.ncu-rep
  i=$((i+1))
done
