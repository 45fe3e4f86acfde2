#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "solve_kernel_order or sticky or edge or full_size_C3 or literal or levels" > gpurun_out/y_tests.log 2>&1; echo rc=$? >> gpurun_out/y_tests.log; tail -3 gpurun_out/y_tests.log
timeout 900 python bench.py --config C3 --no-cpu-baseline > gpurun_out/bench_C3_y.json 2> gpurun_out/bench_C3_y.err; python -c "
import json; d=json.loads(open('gpurun_out/bench_C3_y.json').read().strip().splitlines()[-1]); print(d['value'], d['us_per_iter'], d['iterations'], d['roofline']['frac'], d['phase_us_per_iter'], d['modes'].get('sticky'))"
