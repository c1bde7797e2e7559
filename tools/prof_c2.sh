mkdir -p gpurun_out /tmp/rep
N="timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled"
B="--steps 1 --warmup 3 --no-e2e --no-cpu-baseline"
$N -k "regex:k_warp_rows" -s 4 -c 2 -o /tmp/rep/c2w python bench.py --config c2 $B > /dev/null 2>&1
python tools/ncu_summary.py /tmp/rep/c2w.ncu-rep 0 > gpurun_out/p4_c2_w0.txt 2>&1
python tools/ncu_summary.py /tmp/rep/c2w.ncu-rep 1 > gpurun_out/p4_c2_w1.txt 2>&1
