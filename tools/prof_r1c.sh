# round-1 re-entry profiling of the current code: dominant kernel per config.
# Reports stay in /tmp on the box (gpurun_out is capped at 64 MiB); only text summaries return.
mkdir -p gpurun_out /tmp/rep
N="timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled"
B="--steps 1 --warmup 3 --no-e2e --no-cpu-baseline"
$N -k "regex:k_segments" -s 1 -c 1 -o /tmp/rep/r_c3_seg python bench.py --config c3 $B > /dev/null 2>&1
$N -k "regex:k_spgemm<.int.1, .int.[01]" -s 4 -c 2 -o /tmp/rep/r_c2 python bench.py --config c2 $B > /dev/null 2>&1
$N -k "regex:k_spgemm<.int.0, .int.1|k_analysis" -s 2 -c 2 -o /tmp/rep/r_c5_num0 python bench.py --config c5 $B > /dev/null 2>&1
python tools/ncu_summary.py /tmp/rep/r_c3_seg.ncu-rep > gpurun_out/r_c3_seg.txt 2>&1
python tools/ncu_summary.py /tmp/rep/r_c2.ncu-rep 0 > gpurun_out/r_c2_sym.txt 2>&1
python tools/ncu_summary.py /tmp/rep/r_c2.ncu-rep 1 > gpurun_out/r_c2_num.txt 2>&1
python tools/ncu_summary.py /tmp/rep/r_c5_num0.ncu-rep 0 > gpurun_out/r_c5_a.txt 2>&1
python tools/ncu_summary.py /tmp/rep/r_c5_num0.ncu-rep 1 > gpurun_out/r_c5_b.txt 2>&1
ls -la /tmp/rep gpurun_out
