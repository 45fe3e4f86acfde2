#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 1500 python -m pytest tests/test_gpu_parity.py -q -x -k "bicg or C3 or sticky or edge" > gpurun_out/aa_tests.log 2>&1; echo rc=$? >> gpurun_out/aa_tests.log; tail -3 gpurun_out/aa_tests.log
timeout 900 python bench.py --config C3 --no-cpu-baseline --no-modes > gpurun_out/bench_C3_aa.json 2> gpurun_out/bench_C3_aa.err; python -c "
import json; d=json.loads(open('gpurun_out/bench_C3_aa.json').read().strip().splitlines()[-1]); print(d['value'], d['us_per_iter'], d['iterations'], d['roofline']['frac'], d['phase_us_per_iter'])"
