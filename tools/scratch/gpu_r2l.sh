#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
for wv in 8 4 2 1; do for sl in 0 20 100; do
  echo -n "warps=$wv sleep=$sl: "; ONLY=10 MF_SWEEP_WARPS=$wv MF_SWEEP_SLEEP=$sl timeout 300 python tools/sptrsv_time.py C4spd 2 2>&1 | tail -1
done; done > gpurun_out/sweep_knobs.log 2>&1; cat gpurun_out/sweep_knobs.log
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "sptrsv or rb_ or ilu0 or preconditioned or C4" > gpurun_out/pre_tests.log 2>&1; echo rc=$? >> gpurun_out/pre_tests.log; tail -3 gpurun_out/pre_tests.log
