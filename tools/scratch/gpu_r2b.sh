#!/bin/bash
# full GPU suite, default bench, f3 crossover, per-config bench lines
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests.log
grep -E "passed|failed|FAILED|Error" gpurun_out/gpu_tests.log | tail -12
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; cat gpurun_out/bench.json; tail -3 gpurun_out/bench.err
timeout 900 python tools/f3_crossover.py > gpurun_out/f3.jsonl 2> gpurun_out/f3.err; cat gpurun_out/f3.jsonl; tail -3 gpurun_out/f3.err
for c in C1 C3 C4spd C4ind; do
  timeout 900 python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; cut -c1-600 gpurun_out/bench_$c.json; tail -2 gpurun_out/bench_$c.err
done
