set -x
mkdir -p gpurun_out
python -m pytest tests -m gpu -x -q 2>&1 | tail -5 > gpurun_out/b19_pytest.txt
python bench.py > gpurun_out/b19_bench.json 2> gpurun_out/b19_bench.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --dist-backend gloo --no-cpu-baseline > gpurun_out/b19_dist_c2.json 2> gpurun_out/b19_dist_c2.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29534 bench.py --gpus 2 --steps 5 --warmup 3 --dist-backend gloo --no-cpu-baseline --config c4 > gpurun_out/b19_dist_c4.json 2> gpurun_out/b19_dist_c4.err
tail -3 gpurun_out/b19_pytest.txt; cat gpurun_out/b19_bench.json | head -c 600; echo; cat gpurun_out/b19_dist_c2.json | head -c 800; tail -5 gpurun_out/b19_dist_c2.err; cat gpurun_out/b19_dist_c4.json | head -c 500; tail -5 gpurun_out/b19_dist_c4.err
