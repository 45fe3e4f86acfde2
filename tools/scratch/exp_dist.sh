timeout 600 python -m pytest tests/test_dist.py -x -q 2>&1 | tail -3
timeout 600 python bench.py --dist --steps 3 --warmup 3 --no-cpu-baseline 2>gpurun_out/bench_dist.err | tee gpurun_out/bench_dist.json
tail -3 gpurun_out/bench_dist.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 1 --dist --steps 2 --warmup 3 --no-cpu-baseline 2>&1 | tail -2
