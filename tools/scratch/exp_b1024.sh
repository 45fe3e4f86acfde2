timeout 300 python tools/sweep.py C2 1000 0x1024,0x512 2>&1 | grep -v Warn
timeout 300 python tools/sweep.py C1 1000 0x512,0x256,0x128 2>&1 | grep -v Warn
