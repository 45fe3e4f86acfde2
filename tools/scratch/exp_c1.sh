python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 300 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
timeout 300 python bench.py --config C1 --no-cpu-baseline 2>/dev/null | tee gpurun_out/bench_C1.json | python -c "import json,sys; b=json.loads(sys.stdin.read()); print('C1', b['value'], b['solve_iters_per_s'], b['config']['plan'])"
