python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 600 python bench.py --config c5 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r02d_bench_c5.json 2>&1
CFG=c5 TAG=r02d K="k_spgemm<.int.1, .int.1, float>;k_warp_rows<.int.1, float, .int.2>;k_spgemm<.int.2, .int.1, float>" bash tools/gpu_profile.sh
