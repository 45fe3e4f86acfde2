#!/bin/bash
# Round-end GPU evidence: smoke, the whole -m gpu suite, bench lines (all single-GPU configs, the
# oracle arm), ncu launch list of the C2 bench, one full capture of the persistent CG solve, DRAM
# traffic of the other configs' solves.  Summaries: python tools/ncu_summary.py r02 (here).
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt 2>&1
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$? >> gpurun_out/smoke.log
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests.log 2>&1; echo rc=$? >> gpurun_out/gpu_tests.log
tail -3 gpurun_out/gpu_tests.log
timeout 900 python bench.py > gpurun_out/bench_C2.json 2> gpurun_out/bench_C2.err; cut -c1-300 gpurun_out/bench_C2.json
timeout 600 python bench.py --impl reference --steps 3 --warmup 0 > gpurun_out/bench_ref.json 2> gpurun_out/bench_ref.err
for c in C1 C3 C4spd C4ind C5; do
  timeout 1500 python bench.py --config $c > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; cut -c1-200 gpurun_out/bench_$c.json
done
timeout 300 python tools/sweep.py C2 1000 0x512 > gpurun_out/sweep_c2.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-modes > gpurun_out/ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cg_persistent -c 1 \
    -o gpurun_out/prof_cg_dyn python tools/one_solve.py C2 1 2 > gpurun_out/ncu_full.log 2>&1
for c in C1 C3 C5; do
  timeout 1200 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:_persistent -c 1 \
      --log-file gpurun_out/traffic_$c.csv python tools/one_solve.py $c 1 2 > gpurun_out/ncu_traffic_$c.log 2>&1
done
ls -la gpurun_out
