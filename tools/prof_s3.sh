# full ncu captures of the top C5 kernels (one launch each)
mkdir -p gpurun_out /tmp/rep
B="--steps 1 --warmup 0 --no-e2e --no-cpu-baseline"
N="timeout 900 ncu --set full --clock-control none --import-source on"
for k in "k_spgemm<.int.1, .int.1, float" "k_warp_rows<.int.1, float" "k_spgemm<.int.1, .int.0, float" "k_spgemm<.int.3, .int.1, float"; do
  t=$(echo "$k" | tr -dc 'a-z0-9_')
  $N -k "regex:$k" --kernel-name-base demangled -c 1 -o /tmp/rep/$t python bench.py --config c5 $B > gpurun_out/${TAG}_$t.log 2>&1
  python tools/ncu_summary.py /tmp/rep/$t.ncu-rep 0 > gpurun_out/${TAG}_$t.txt 2>&1
done
ls -la /tmp/rep
