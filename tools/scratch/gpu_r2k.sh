#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 600 python tools/sptrsv_time.py C4spd 2 > gpurun_out/sptrsv_time.log 2>&1; cat gpurun_out/sptrsv_time.log
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "sptrsv or rb_ or ilu0 or preconditioned or C4" > gpurun_out/pre_tests.log 2>&1; echo rc=$? >> gpurun_out/pre_tests.log; tail -3 gpurun_out/pre_tests.log
for c in C4spd C4ind; do
  timeout 900 python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; cut -c1-300 gpurun_out/bench_$c.json; tail -2 gpurun_out/bench_$c.err
done
