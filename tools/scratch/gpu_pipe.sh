#!/bin/bash
export PYTHONUNBUFFERED=1
for sh in 0x1024; do
  MF_PHASE_DUMP=1 timeout 120 python tools/sweep.py C2 100 $sh 2>&1 | grep -E "mode=|SpMV, warp|smem" | sed "s/^/$sh /" | tail -6
done
