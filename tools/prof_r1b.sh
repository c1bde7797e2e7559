# round-1 profiling, second pass: long-row jobs (C3), C5 numeric cfg0, C2 symbolic/numeric
N="ncu --set full --clock-control none --import-source on --kernel-name-base demangled"
$N -k "regex:k_segments" -s 2 -c 1 -o gpurun_out/q_c3_seg python bench.py --config c3 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
$N -k "regex:k_spgemm<.int.0, .int.1" -s 2 -c 1 -o gpurun_out/q_c5_num0 python bench.py --config c5 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
$N -k "regex:k_spgemm<.int.1, .int.[01]" -s 4 -c 2 -o gpurun_out/q_c2 python bench.py --config c2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
for f in q_c3_seg q_c5_num0; do python tools/ncu_summary.py gpurun_out/$f.ncu-rep > gpurun_out/$f.txt 2>&1; done
python tools/ncu_summary.py gpurun_out/q_c2.ncu-rep 0 > gpurun_out/q_c2_sym.txt 2>&1
python tools/ncu_summary.py gpurun_out/q_c2.ncu-rep 1 > gpurun_out/q_c2_num.txt 2>&1
