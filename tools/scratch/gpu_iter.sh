#!/bin/bash
# one iteration of the SpMV work: parity subset, C2 solve sweep with the SpMV breakdown
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "spmv_bit_exact or levels or dot_tree or solve_kernel_order or edge or precond or sticky or ilu" > gpurun_out/chk.log 2>&1; echo rc=$? >> gpurun_out/chk.log
tail -15 gpurun_out/chk.log
MF_PHASE_DUMP=1 timeout 300 python tools/sweep.py C2 1000 0x512 > gpurun_out/sweep_c2.log 2>&1; grep -v "^phase" gpurun_out/sweep_c2.log | tail -8
