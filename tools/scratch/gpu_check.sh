#!/bin/bash
# quick GPU check after a kernel change: SpMV / solve parity subset, C2 phase sweep
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "spmv_bit_exact or levels or dot_tree" > gpurun_out/chk_spmv.log 2>&1; echo rc=$? >> gpurun_out/chk_spmv.log
tail -15 gpurun_out/chk_spmv.log
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "solve_kernel_order or edge or precond or sticky or ilu" > gpurun_out/chk_solve.log 2>&1; echo rc=$? >> gpurun_out/chk_solve.log
tail -25 gpurun_out/chk_solve.log
MF_PHASE_DUMP=1 timeout 300 python tools/sweep.py C2 1000 0x512 > gpurun_out/sweep_c2.log 2>&1; tail -20 gpurun_out/sweep_c2.log
