#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 600 python tools/sptrsv_time.py C4spd 2 > gpurun_out/sptrsv_time.log 2>&1; cat gpurun_out/sptrsv_time.log
ONLY=10 timeout 600 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -c 1 -o gpurun_out/prof_sweep \
   python tools/sptrsv_time.py C4spd 1 > gpurun_out/ncu_sweep.log 2>&1; tail -2 gpurun_out/ncu_sweep.log
timeout 300 python tools/sweep.py C1 1000 0x512,16x256,8x256 > gpurun_out/sweep_c1.log 2>&1; grep -v "^phase" gpurun_out/sweep_c1.log
timeout 900 python -m pytest tests/test_dist.py -q -m gpu -x > gpurun_out/dist_tests.log 2>&1; echo rc=$? >> gpurun_out/dist_tests.log; tail -3 gpurun_out/dist_tests.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "solve_kernel_order or edge or single_reduction or sticky" > gpurun_out/cl_tests.log 2>&1; echo rc=$? >> gpurun_out/cl_tests.log; tail -3 gpurun_out/cl_tests.log
