#!/bin/bash
# SpTRSV schedules (sweep / chunked, rb), dist local group, C4 bench lines
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "rb_ or ilu0 or preconditioned or sptrsv or C4" > gpurun_out/pre_tests.log 2>&1; echo rc=$? >> gpurun_out/pre_tests.log
tail -3 gpurun_out/pre_tests.log
timeout 900 python -m pytest tests/test_dist.py -q -m gpu > gpurun_out/dist_tests.log 2>&1; echo rc=$? >> gpurun_out/dist_tests.log
tail -3 gpurun_out/dist_tests.log
for c in C4spd C4ind; do
  timeout 900 python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; cut -c1-400 gpurun_out/bench_$c.json; tail -2 gpurun_out/bench_$c.err
done
