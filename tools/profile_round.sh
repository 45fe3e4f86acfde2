#!/bin/bash
# GPU side: launch list of a short bench run + one full ncu capture of the dominant kernel
# (the persistent solve, dynamic mixed mode, C2).  Summaries are made here by tools/ncu_summary.py.
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cg_persistent -c 1 \
    -o gpurun_out/prof_cg_dyn python tools/one_solve.py C2 1 2 > gpurun_out/ncu_full.log 2>&1
ls -la gpurun_out
