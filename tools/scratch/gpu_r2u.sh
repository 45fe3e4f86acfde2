#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
ONLY=10 MF_SWEEP_DBG=1 timeout 300 python tools/sptrsv_time.py C4spd 1 2>&1 | tail -3
echo -n "plain: "; ONLY=10 timeout 300 python tools/sptrsv_time.py C4spd 2 2>&1 | tail -1
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "sptrsv or rb_ or ilu0 or preconditioned or C4" > gpurun_out/pre_tests.log 2>&1; echo rc=$? >> gpurun_out/pre_tests.log; tail -3 gpurun_out/pre_tests.log
for c in C4spd C4ind; do timeout 900 python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; cut -c1-250 gpurun_out/bench_$c.json; done
