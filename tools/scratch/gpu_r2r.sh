#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 300 python tools/sweep.py C2 1000 0x512 > gpurun_out/sweep_c2_lv.log 2>&1; grep -v "^phase" gpurun_out/sweep_c2_lv.log
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_boundary.py -q -x -k "levels or solve_kernel_order or sticky or edge or spmv or single_reduction or full_size_C2" > gpurun_out/lv_tests.log 2>&1; echo rc=$? >> gpurun_out/lv_tests.log; tail -3 gpurun_out/lv_tests.log
timeout 900 python bench.py --config C1 > gpurun_out/bench_C1_new.json 2> gpurun_out/bench_C1_new.err; python -c "
import json; d=json.loads(open('gpurun_out/bench_C1_new.json').read().strip().splitlines()[-1]); print(d['value'], d['modes'].get('sticky'), d['precision'])"; tail -2 gpurun_out/bench_C1_new.err
