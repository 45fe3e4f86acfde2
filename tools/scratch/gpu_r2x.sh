#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 300 python tools/sweep.py C2 1000 0x512 > gpurun_out/sweep_c2_x.log 2>&1; grep -v "^phase" gpurun_out/sweep_c2_x.log
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "levels or solve_kernel_order or sticky or edge or full_size_C2 or literal or torch_alloc" > gpurun_out/x_tests.log 2>&1; echo rc=$? >> gpurun_out/x_tests.log; tail -3 gpurun_out/x_tests.log
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/bench_C2_x.json 2> gpurun_out/bench_C2_x.err; cut -c1-300 gpurun_out/bench_C2_x.json
