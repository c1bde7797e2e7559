set -x
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:k_spgemm<0, 1" -s 2 -c 1 -o gpurun_out/p_c5_num0 python bench.py --config c5 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:k_segments" -s 2 -c 1 -o gpurun_out/p_c3_seg python bench.py --config c3 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:k_spgemm<4, 0" -s 2 -c 1 -o gpurun_out/p_c3_sym4 python bench.py --config c3 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:k_spgemm<1, 1" -s 4 -c 1 -o gpurun_out/p_c2_num1 python bench.py --config c2 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ls -la gpurun_out
