#!/bin/bash
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -c 1 -o gpurun_out/prof_spmv3 \
   python tools/spmv_time.py C2 > gpurun_out/ncu_spmv3.log 2>&1
tail -2 gpurun_out/ncu_spmv3.log
