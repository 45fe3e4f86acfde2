#!/bin/bash
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
echo "== r2e build (630e4c1)"; (cd tmp_bisect && timeout 120 python tools/one_solve.py C1 1 0 2>&1 | tail -2)
echo "== HEAD C1 mode0"; timeout 120 python tools/one_solve.py C1 1 0 2>&1 | tail -1
echo "== HEAD C1 mode2"; timeout 120 python tools/one_solve.py C1 1 2 2>&1 | tail -1
echo "== HEAD C2 mode0"; timeout 120 python tools/one_solve.py C2 1 0 2>&1 | tail -1
echo "== HEAD C2 mode1"; timeout 120 python tools/one_solve.py C2 1 1 2>&1 | tail -1
