#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
for wv in 8 1; do echo "warps=$wv: "; ONLY=10 MF_SWEEP_DBG=1 MF_SWEEP_WARPS=$wv timeout 300 python tools/sptrsv_time.py C4spd 1 2>&1 | tail -5; done
