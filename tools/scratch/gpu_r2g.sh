#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 300 compute-sanitizer --tool memcheck --print-limit 5 python tools/one_solve.py C1 1 0 > gpurun_out/sanitizer_c1.log 2>&1; tail -40 gpurun_out/sanitizer_c1.log
MF_CLUSTER=0 timeout 120 python tools/one_solve.py C1 1 0 > gpurun_out/c1_nocl.log 2>&1; tail -3 gpurun_out/c1_nocl.log
