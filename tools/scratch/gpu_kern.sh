#!/bin/bash
export PYTHONUNBUFFERED=1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "spmv_bit_exact or levels or dot_tree or solve_kernel_order or edge or precond or sticky or ilu or convert" > gpurun_out/chk.log 2>&1; echo rc=$? >> gpurun_out/chk.log
tail -3 gpurun_out/chk.log
timeout 120 python tools/spmv_kern.py C2 2>&1 | grep -E "mf_spmv"
timeout 120 python tools/spmv_kern.py C2 dyn 2>&1 | grep -E "mf_spmv"
timeout 300 python tools/sweep.py C2 1000 0x512 2>&1 | grep -v "^phase" | tail -3
