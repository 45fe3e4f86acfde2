#!/bin/bash
# SpMV diagnostics: standalone mf_spmv timing (full / stream-only / ring depths) + one ncu capture
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
for d in 0 1; do for nst in 2 4 6; do MF_SPMV_DBG=$d MF_NST=$nst timeout 120 python tools/spmv_time.py C2 2>&1 | sed "s/^/nst=$nst /"; done; done > gpurun_out/spmv_time.log
cat gpurun_out/spmv_time.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -c 1 -o gpurun_out/prof_spmv \
   python tools/spmv_time.py C2 > gpurun_out/ncu_spmv.log 2>&1
tail -3 gpurun_out/ncu_spmv.log
