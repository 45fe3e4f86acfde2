timeout 120 python tools/spmv_time.py C2 512
timeout 300 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
timeout 300 python tools/sweep.py C2 1000 0x512
