#!/bin/bash
# quick GPU check: parity tests (stop at first failure), C2 phase sweep, bench line
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests.log
tail -30 gpurun_out/gpu_tests.log
timeout 300 python tools/sweep.py C2 1000 0x512 > gpurun_out/sweep_c2.log 2>&1; cat gpurun_out/sweep_c2.log | tail -5
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; cat gpurun_out/bench.json; tail -3 gpurun_out/bench.err
