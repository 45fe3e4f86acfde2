#!/bin/bash
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
MF_SPMV_REPS=2 MF_SPMV_DBG=${1:-9} timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 1 -c 1 -o gpurun_out/prof_spmv_d${1:-9} \
   python tools/spmv_kern.py C2 > gpurun_out/ncu_spmv.log 2>&1
tail -2 gpurun_out/ncu_spmv.log
