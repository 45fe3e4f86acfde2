#!/bin/bash
# rb SpTRSV parity, C1 launch-shape sweep, SpMV/CG profiles, bench launch list
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "rb_ or ilu0 or preconditioned" > gpurun_out/rb_tests.log 2>&1; echo rc=$? >> gpurun_out/rb_tests.log
timeout 900 python -m pytest tests/test_dist.py -q -m gpu >> gpurun_out/rb_tests.log 2>&1; echo rc=$? >> gpurun_out/rb_tests.log
tail -3 gpurun_out/rb_tests.log
timeout 300 python tools/sweep.py C1 1000 1x1024,1x512,2x512,4x512,8x256,16x256,32x512 > gpurun_out/sweep_c1.log 2>&1; grep -v "^phase" gpurun_out/sweep_c1.log
bash tools/gpu_prof_r2.sh
