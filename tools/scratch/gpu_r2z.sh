#!/bin/bash
# final verification at HEAD: smoke, full GPU suite, bench lines C2 (default, with CPU baseline) and C1
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$? >> gpurun_out/smoke.log; tail -2 gpurun_out/smoke.log
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_tests.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests.log
tail -3 gpurun_out/gpu_tests.log
timeout 900 python bench.py > gpurun_out/bench_C2.json 2> gpurun_out/bench_C2.err; cut -c1-300 gpurun_out/bench_C2.json
timeout 900 python bench.py --config C1 > gpurun_out/bench_C1.json 2> gpurun_out/bench_C1.err; cut -c1-200 gpurun_out/bench_C1.json
timeout 1500 python bench.py --config C5 > gpurun_out/bench_C5.json 2> gpurun_out/bench_C5.err; cut -c1-200 gpurun_out/bench_C5.json
