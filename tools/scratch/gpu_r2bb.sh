#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
{ timeout 120 python tools/spmv_kern.py C2; timeout 120 python tools/spmv_kern.py C2 dyn; } 2>&1 | grep mf_spmv
timeout 300 python tools/sweep.py C2 1000 0x512 > gpurun_out/sweep_c2_bb.log 2>&1; grep -v "^phase" gpurun_out/sweep_c2_bb.log
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "spmv or solve_kernel_order or sticky or full_size_C2 or literal or levels" > gpurun_out/bb_tests.log 2>&1; echo rc=$? >> gpurun_out/bb_tests.log; tail -3 gpurun_out/bb_tests.log
