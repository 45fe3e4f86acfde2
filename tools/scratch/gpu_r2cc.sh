#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 900 python bench.py --dist --steps 3 --warmup 3 > gpurun_out/bench_dist1.json 2> gpurun_out/bench_dist1.err; cut -c1-300 gpurun_out/bench_dist1.json; python -c "
import json; d=json.loads(open('gpurun_out/bench_dist1.json').read().strip().splitlines()[-1]); print(d['value'], d['config'].get('dist_mode'))"; tail -3 gpurun_out/bench_dist1.err
