# round evidence: default bench line (full contract), launch list of the same command, full
# capture of the dominant C2 kernel (numeric tiny-row warp kernel of A*P)
rm -rf /tmp/rep; mkdir -p gpurun_out /tmp/rep
T=${TAG:-fin}
timeout 600 python bench.py > gpurun_out/${T}_bench_c2.json 2> gpurun_out/${T}_bench_c2.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${T}_launches_c2.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
python tools/ncu_launches.py gpurun_out/${T}_launches_c2.csv 40 > gpurun_out/${T}_launches_c2.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k "regex:k_warp_rows<.int.1, double, .int.1" --kernel-name-base demangled -c 1 -o /tmp/rep/w python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
python tools/ncu_summary.py /tmp/rep/w.ncu-rep 0 > gpurun_out/${T}_ncu_c2_numeric.txt 2>&1
cp /tmp/rep/w.ncu-rep gpurun_out/${T}_ncu_c2_numeric.ncu-rep
