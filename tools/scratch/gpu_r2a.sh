#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 900 python -m pytest tests -m gpu -q -k "dist_world1 or nonsymmetric or single_reduction or watchdog or multiwindow" > gpurun_out/t.log 2>&1; echo rc=$? >> gpurun_out/t.log
grep -E "passed|failed|FAILED|Error|invalid" gpurun_out/t.log | tail -12
for cfg in "0 0" "32 2" "32 3" "16 2"; do set -- $cfg
  echo "== KCAP=$1 MINRING=$2"; MF_KCAP=$1 MF_MU_MINRING=$2 MF_PHASE_DUMP=1 timeout 300 python tools/sweep.py C2 1000 0x512 2>&1 | grep -E "^C2|smem|ring" | tail -6
done
echo "== C2 cgsr"; CGV=1 timeout 300 python tools/sweep.py C2 1000 0x512 2>&1 | grep "^C2"
echo "== C1"; timeout 300 python tools/sweep.py C1 1000 0x128,0x256,0x512,1x1024,2x1024,4x512,8x256 2>&1 | grep "^C1"
echo "== C1 cgsr"; CGV=1 timeout 300 python tools/sweep.py C1 1000 0x256,1x1024,4x512 2>&1 | grep "^C1"
