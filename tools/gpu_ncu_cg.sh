#!/bin/bash
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out
MODE=${1:-1}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cg_persistent -c 1 -o gpurun_out/prof_cg_m$MODE \
   python tools/one_solve.py C2 1 $MODE > gpurun_out/ncu_cg.log 2>&1
tail -3 gpurun_out/ncu_cg.log
