python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "every_path" -s 2>&1 | grep -E "path counts|passed|failed|Error" | cut -c1-2000
CFG=c5 TAG=r02g K="k_spgemm<.int.1, .int.1, float>;k_spgemm<.int.1, .int.0, float>;k_warp_rows<.int.0, float, .int.0>" bash tools/gpu_profile.sh
