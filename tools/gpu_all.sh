# all bench lines (c1..c5) + the default full-contract line + reference arm + launch list + dominant-kernel capture
mkdir -p gpurun_out
T=${TAG:-all}
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -3 > gpurun_out/${T}_pytest.txt
for c in c1 c3 c4 c5; do
  timeout 600 python bench.py --config $c --steps 5 --warmup 3 > gpurun_out/${T}_bench_$c.json 2> gpurun_out/${T}_bench_$c.err
done
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${T}_ref_c2.json 2> gpurun_out/${T}_ref_c2.err
TAG=$T bash tools/prof_final.sh
cat gpurun_out/${T}_pytest.txt
