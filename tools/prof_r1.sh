# round-1 profiling: top kernels per workload (ncu --set full, one launch each)
set -x
N="ncu --set full --clock-control none --import-source on --kernel-name-base demangled"
$N -k "regex:k_spgemm<.int.0, .int.1" -s 2 -c 1 -o gpurun_out/p_c5_num0 python bench.py --config c5 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
$N -k "regex:k_spgemm<.int.4, .int.0" -s 2 -c 1 -o gpurun_out/p_c3_sym4 python bench.py --config c3 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
$N -k "regex:k_spgemm<.int.1, .int.1" -s 4 -c 1 -o gpurun_out/p_c2_num1 python bench.py --config c2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ls -la gpurun_out
