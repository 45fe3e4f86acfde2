#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "literal_absolute or sptrsv or preconditioned or solve_kernel_order or edge" > gpurun_out/v_tests.log 2>&1; echo rc=$? >> gpurun_out/v_tests.log; tail -3 gpurun_out/v_tests.log
grep -E "Error|assert" gpurun_out/v_tests.log | head -5
for c in C4spd C4ind; do timeout 900 python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; cut -c1-250 gpurun_out/bench_$c.json; done
timeout 300 python tools/sweep.py C2 1000 0x512 > gpurun_out/sweep_c2_v.log 2>&1; grep -v "^phase" gpurun_out/sweep_c2_v.log
