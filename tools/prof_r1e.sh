mkdir -p gpurun_out /tmp/rep
B="--steps 1 --warmup 3 --no-e2e --no-cpu-baseline"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file /tmp/rep/l5.csv python bench.py --config c5 $B > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file /tmp/rep/l3.csv python bench.py --config c3 $B > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file /tmp/rep/l2.csv python bench.py --config c2 $B > /dev/null 2>&1
for c in 5 3 2; do python tools/ncu_launches.py /tmp/rep/l$c.csv > gpurun_out/p3_launch_c$c.txt 2>&1; done
N="timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled"
$N -k "regex:k_warp_rows" -s 2 -c 2 -o /tmp/rep/wr5 python bench.py --config c5 $B > /dev/null 2>&1
python tools/ncu_summary.py /tmp/rep/wr5.ncu-rep 0 > gpurun_out/p3_c5_wr0.txt 2>&1
python tools/ncu_summary.py /tmp/rep/wr5.ncu-rep 1 > gpurun_out/p3_c5_wr1.txt 2>&1
