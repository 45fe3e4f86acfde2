#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
ONLY=10 MF_SWEEP_DBG=1 timeout 300 python tools/sptrsv_time.py C4spd 1 2>&1 | tail -3
