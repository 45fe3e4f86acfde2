#!/bin/bash
# TMA streaming diagnostics of the standalone SpMV: full / stream both / blobs only / windows only / nothing
export PYTHONUNBUFFERED=1
for d in 0 1 2 3 4; do MF_SPMV_DBG=$d timeout 120 python tools/spmv_time.py C2 2>&1 | sed "s/^/dbg=$d /"; done
for nst in 1 2 3; do MF_SPMV_DBG=1 MF_NST=$nst timeout 120 python tools/spmv_time.py C2 2>&1 | sed "s/^/dbg=1 nst=$nst /"; done
