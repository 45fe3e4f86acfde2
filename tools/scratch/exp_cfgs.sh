for c in C1 C3; do timeout 900 python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; tail -c 1500 gpurun_out/bench_$c.json; tail -2 gpurun_out/bench_$c.err; done
timeout 600 python tools/sweep.py C3 20000 0x512 2>&1 | grep -v Warn
timeout 1500 python bench.py --config C5 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_C5.json 2> gpurun_out/bench_C5.err; tail -c 1500 gpurun_out/bench_C5.json; tail -3 gpurun_out/bench_C5.err
free -g | head -2
