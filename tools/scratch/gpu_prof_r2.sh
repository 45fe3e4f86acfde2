#!/bin/bash
# r02 diagnostics: standalone SpMV timing (static / dynamic levels), phase sweep, one ncu capture of the
# standalone SpMV and of the persistent CG, launch list of a short bench run (conversion kernels).
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
{ timeout 120 python tools/spmv_kern.py C2; timeout 120 python tools/spmv_kern.py C2 dyn; } > gpurun_out/spmv_kern.log 2>&1
grep mf_spmv gpurun_out/spmv_kern.log
timeout 300 python tools/sweep.py C2 1000 0x512 > gpurun_out/sweep_c2.log 2>&1; grep -v "^phase" gpurun_out/sweep_c2.log | tail -3
MF_SPMV_REPS=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -c 1 -o gpurun_out/prof_spmv \
   python tools/spmv_kern.py C2 dyn > gpurun_out/ncu_spmv.log 2>&1; tail -2 gpurun_out/ncu_spmv.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cg_persistent -c 1 \
    -o gpurun_out/prof_cg_dyn python tools/one_solve.py C2 1 2 > gpurun_out/ncu_full.log 2>&1; tail -2 gpurun_out/ncu_full.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1; tail -2 gpurun_out/ncu_bench.log
ls -la gpurun_out
