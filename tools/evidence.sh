#!/bin/bash
# Evidence job (GPU box): tests, bench lines, reference arm, launch lists, ncu captures,
# sanitizers, 2-rank path.  Outputs under gpurun_out/${TAG}_*.
TAG=${TAG:-r02e}
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
if [ "${TESTS:-1}" = 1 ]; then
  ( time timeout 1500 python -m pytest tests -m gpu -q --durations=25 ) > gpurun_out/${TAG}_pytest_gpu.txt 2>&1
fi
if [ "${BENCH:-1}" = 1 ]; then
  for c in ${CFGS:-c5 c2 c3 c4 c1}; do
    timeout 900 python bench.py --config $c --steps ${STEPS:-5} --warmup 3 > gpurun_out/${TAG}_bench_$c.json 2> gpurun_out/${TAG}_bench_$c.err
  done
  timeout 900 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${TAG}_reference_c5.json 2>&1
fi
if [ "${DIST:-1}" = 1 ]; then
  timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
    bench.py --gpus 2 --steps 3 --warmup 3 --config c4 --dist-backend gloo --no-cpu-baseline > gpurun_out/${TAG}_dist2_gloo_c4.json 2> gpurun_out/${TAG}_dist2_gloo_c4.err
fi
if [ "${SAN:-0}" = 1 ]; then   # compute-sanitizer is closed on the GPU pool (round 2)
  for tool in memcheck racecheck synccheck initcheck; do
    timeout 1200 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize_cases.py > gpurun_out/${TAG}_sanitizer_$tool.txt 2>&1
    echo "exit $?" >> gpurun_out/${TAG}_sanitizer_$tool.txt
  done
fi
if [ "${NCU:-1}" = 1 ]; then
  CFG=c5 TAG=${TAG} LAUNCHES=1 K="k_spgemm<.int.1, .int.1, float>;k_spgemm<.int.1, .int.0, float>;k_spgemm<.int.2, .int.1, float>;k_spgemm<.int.3, .int.1, float>;k_spgemm<.int.4, .int.1, float>;k_warp_rows<.int.1, float, .int.2>;k_warp_rows<.int.0, float, .int.0>" bash tools/gpu_profile.sh
  CFG=c3 TAG=${TAG} LAUNCHES=1 K="k_long_bitmap<float>;k_spgemm<.int.4, .int.0, float>" bash tools/gpu_profile.sh
  CFG=c2 TAG=${TAG} LAUNCHES=1 K="k_warp_rows<.int.1, double, .int.1>;k_warp_rows<.int.0, double, .int.0>" bash tools/gpu_profile.sh
fi
echo evidence-done
