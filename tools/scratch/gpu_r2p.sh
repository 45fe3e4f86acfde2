#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
for wv in 8 4; do echo "warps=$wv: "; ONLY=10 MF_SWEEP_DBG=1 MF_SWEEP_WARPS=$wv timeout 300 python tools/sptrsv_time.py C4spd 1 2>&1 | tail -3; done
echo -n "plain: "; ONLY=10 timeout 300 python tools/sptrsv_time.py C4spd 2 2>&1 | tail -1
{ timeout 120 python tools/spmv_kern.py C2; timeout 120 python tools/spmv_kern.py C2 dyn; } 2>&1 | grep mf_spmv
timeout 300 python tools/sweep.py C2 1000 0x512 > gpurun_out/sweep_c2.log 2>&1; grep -v "^phase" gpurun_out/sweep_c2.log
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "sptrsv or rb_ or ilu0 or preconditioned or C4 or spmv or solve_kernel_order or sticky" > gpurun_out/pre_tests.log 2>&1; echo rc=$? >> gpurun_out/pre_tests.log; tail -3 gpurun_out/pre_tests.log
