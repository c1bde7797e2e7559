# profiling pass 2: C5 symbolic/numeric cfg0 + C2 symbolic (A*P) after the ballot-window epilogue
mkdir -p gpurun_out /tmp/rep
N="timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled"
B="--steps 1 --warmup 3 --no-e2e --no-cpu-baseline"
$N -k "regex:k_spgemm<.int.0, .int.[01]" -s 2 -c 2 -o /tmp/rep/c5 python bench.py --config c5 $B > /dev/null 2>&1
$N -k "regex:k_spgemm<.int.1, .int.0" -s 2 -c 1 -o /tmp/rep/c2s python bench.py --config c2 $B > /dev/null 2>&1
python tools/ncu_summary.py /tmp/rep/c5.ncu-rep 0 > gpurun_out/p2_c5_0.txt 2>&1
python tools/ncu_summary.py /tmp/rep/c5.ncu-rep 1 > gpurun_out/p2_c5_1.txt 2>&1
python tools/ncu_summary.py /tmp/rep/c2s.ncu-rep 0 > gpurun_out/p2_c2_sym.txt 2>&1
