#!/bin/bash
# GPU-side profiling job (run under gpurun from the repo root).
#   CFG=c5 TAG=r02a K="k_spgemm<1, 1,;k_warp_rows<1, float, 2>" LAUNCHES=1 BENCH=1 bash tools/gpu_profile.sh
# BENCH=1: one bench line (no e2e/cpu) -> gpurun_out/${TAG}_bench_${CFG}.json
# LAUNCHES=1: ncu launch list of one step -> gpurun_out/${TAG}_launch_${CFG}.txt
# K: ';'-separated kernel regexes, one `ncu --set full` capture each -> gpurun_out/${TAG}_${CFG}_kN.{txt,ncu-rep}
set -u
mkdir -p gpurun_out /tmp/rep
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { cat gpurun_out/${TAG}_build.log; exit 1; }
B="--config $CFG --no-e2e --no-cpu-baseline"
if [ "${BINSTATS:-0}" = 1 ]; then
  timeout 600 python tools/binstats.py $CFG > gpurun_out/${TAG}_binstats_${CFG}.txt 2>&1
fi
if [ "${BENCH:-0}" = 1 ]; then
  timeout 900 python bench.py $B --steps ${STEPS:-5} --warmup 3 ${BENCH_OPTS:-} > gpurun_out/${TAG}_bench_${CFG}.json 2> gpurun_out/${TAG}_bench_${CFG}.err
fi
if [ "${LAUNCHES:-0}" = 1 ]; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:^k_" --csv --log-file /tmp/rep/l.csv \
    python bench.py $B --steps 1 --warmup 3 > /dev/null 2>&1
  python tools/ncu_launches.py /tmp/rep/l.csv 40 > gpurun_out/${TAG}_launch_${CFG}.txt 2>&1
fi
i=0
IFS=";" read -ra KS <<< "${K:-}"
for k in "${KS[@]}"; do
  rm -f /tmp/rep/k$i.ncu-rep
  timeout 900 ncu -f --set full --clock-control none --import-source on -k "regex:$k" --kernel-name-base demangled -c 1 \
    -o /tmp/rep/k$i python bench.py $B --steps 1 --warmup 3 > gpurun_out/${TAG}_${CFG}_k$i.log 2>&1
  python tools/ncu_summary.py /tmp/rep/k$i.ncu-rep 0 > gpurun_out/${TAG}_${CFG}_k$i.txt 2>&1
  python tools/ncu_sass.py /tmp/rep/k$i.ncu-rep 0 > gpurun_out/${TAG}_${CFG}_k${i}_sass.txt 2>&1
  python tools/traffic_from_ncu.py --dry $CFG $TAG /tmp/rep/k$i.ncu-rep >> gpurun_out/${TAG}_${CFG}_traffic.txt 2>&1
  # reports are ~10-40 MB each: only brought back on request (gpurun_out is capped at 64 MiB)
  if [ "${KEEP_REP:-0}" = 1 ]; then cp /tmp/rep/k$i.ncu-rep gpurun_out/${TAG}_${CFG}_k$i.ncu-rep; fi
  i=$((i+1))
done
echo done
