#!/bin/bash
# One GPU session: unit parity tests, variant sweep, bench, ncu.  Usage (via gpurun):
#   bash tools/gpu_check.sh [tests|sweep|bench|ncu|slow]...
set -u
mkdir -p gpurun_out
for what in "$@"; do
  case "$what" in
    tests) timeout -s KILL 420 python -m pytest tests -m "gpu and not slow" -q --timeout 180 --timeout-method=thread -x 2>&1 | tail -25 | tee gpurun_out/pytest_gpu.log ;;
    slow)  timeout -s KILL 1500 python -m pytest tests -m "gpu and slow" -q -s --timeout 900 --timeout-method=thread 2>&1 | tail -15 | tee gpurun_out/pytest_slow.log ;;
    smoke) timeout -s KILL 120 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3 ;;
    sweep) timeout -s KILL 300 python tools/sweep_variants.py --n 32768 --dtype f32 --orders ${SWEEP_ORDERS:-0} 2>&1 | tee gpurun_out/sweep.jsonl ;;
    bench) timeout -s KILL 900 python bench.py --steps 20 --warmup 5 2>&1 | tail -2 | tee gpurun_out/bench.json ;;
    launches) timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --no-extras > gpurun_out/launches_bench.log 2>&1; tail -3 gpurun_out/launches.csv ;;
    stats) timeout -s KILL 200 python tools/stats_ws.py --variants ${STATS_VARIANTS:-0,1,2} 2>&1 | tail -4 ;;
    ncu) timeout 1500 ncu --set full --clock-control none --import-source on -k regex:sat_ -s 3 -c 1 -o gpurun_out/prof -f python bench.py --steps 1 --warmup 3 --no-cpu --no-e2e --no-extras > gpurun_out/ncu_bench.log 2>&1; tail -3 gpurun_out/ncu_bench.log ;;
  esac
done
