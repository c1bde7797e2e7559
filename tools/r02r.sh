python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
CFG=c2 TAG=r02r K="k_warp_rows<.int.1, double, .int.1>;k_warp_rows<.int.0, double, .int.0>" bash tools/gpu_profile.sh
timeout 1500 python tools/ablation.py --configs c3 --steps 3 --lb-sweep > gpurun_out/r02r_ablation.jsonl 2> gpurun_out/r02r_ablation.err
