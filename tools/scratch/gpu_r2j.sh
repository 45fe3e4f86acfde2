#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
ONLY=10 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:sweep_kernel python tools/sptrsv_time.py C4spd 1 > gpurun_out/ncu_sweep_times.log 2>&1; grep -E "sweep_kernel|gpu__time" gpurun_out/ncu_sweep_times.log | head -12
ONLY=10 timeout 600 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 2 -c 2 -o gpurun_out/prof_sweep2 \
   python tools/sptrsv_time.py C4spd 1 > gpurun_out/ncu_sweep2.log 2>&1; tail -2 gpurun_out/ncu_sweep2.log
