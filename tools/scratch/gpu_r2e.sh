#!/bin/bash
# SpTRSV schedules + dist local group + C4 bench lines + C2 SpMV ring variants
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 600 python tools/spmv_kern.py C2 > gpurun_out/spmv_kern.log 2>&1; timeout 600 python tools/spmv_kern.py C2 dyn >> gpurun_out/spmv_kern.log 2>&1; grep mf_spmv gpurun_out/spmv_kern.log
for kc in 32 64; do for nst in 3 6; do
  echo "KCAP=$kc NST=$nst" >> gpurun_out/sweep_c2.log
  MF_KCAP=$kc MF_NST=$nst timeout 300 python tools/sweep.py C2 1000 0x512 2>&1 | grep -v "^phase" >> gpurun_out/sweep_c2.log
done; done
cat gpurun_out/sweep_c2.log
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "rb_ or ilu0 or preconditioned or sptrsv or C4 or spmv or solve_kernel_order" > gpurun_out/pre_tests.log 2>&1; echo rc=$? >> gpurun_out/pre_tests.log
tail -3 gpurun_out/pre_tests.log
timeout 900 python -m pytest tests/test_dist.py -q -m gpu > gpurun_out/dist_tests.log 2>&1; echo rc=$? >> gpurun_out/dist_tests.log
tail -3 gpurun_out/dist_tests.log
for c in C4spd C4ind; do
  timeout 900 python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; cut -c1-400 gpurun_out/bench_$c.json; tail -2 gpurun_out/bench_$c.err
done
