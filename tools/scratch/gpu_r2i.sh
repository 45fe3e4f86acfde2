#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
for m in 0 1 2; do echo "== C1 mode$m"; timeout 120 python tools/one_solve.py C1 1 $m 2>&1 | tail -1; done
echo "== C2 mode1"; timeout 120 python tools/one_solve.py C2 1 1 2>&1 | tail -1
timeout 300 python tools/sweep.py C2 1000 0x512 > gpurun_out/sweep_c2.log 2>&1; grep -v "^phase" gpurun_out/sweep_c2.log
timeout 600 python tools/sptrsv_time.py C4spd 2 > gpurun_out/sptrsv_time.log 2>&1; cat gpurun_out/sptrsv_time.log
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "sptrsv or rb_ or ilu0 or preconditioned or solve_kernel_order or edge" > gpurun_out/pre_tests.log 2>&1; echo rc=$? >> gpurun_out/pre_tests.log; tail -3 gpurun_out/pre_tests.log
timeout 600 python -m pytest tests/test_dist.py -q -m gpu -x > gpurun_out/dist_tests.log 2>&1; echo rc=$? >> gpurun_out/dist_tests.log; tail -3 gpurun_out/dist_tests.log
