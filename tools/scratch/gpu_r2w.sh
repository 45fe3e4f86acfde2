#!/bin/bash
# final verification at HEAD: smoke, full GPU suite, C2 bench, C3 traffic with the config's eps
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$? >> gpurun_out/smoke.log; tail -2 gpurun_out/smoke.log
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_tests.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests.log
tail -3 gpurun_out/gpu_tests.log
timeout 900 python bench.py > gpurun_out/bench_C2.json 2> gpurun_out/bench_C2.err; cut -c1-400 gpurun_out/bench_C2.json
timeout 1200 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:_persistent -c 1 \
    --log-file gpurun_out/traffic_C3.csv python tools/one_solve.py C3 1 2 > gpurun_out/ncu_traffic_C3.log 2>&1; tail -2 gpurun_out/ncu_traffic_C3.log
