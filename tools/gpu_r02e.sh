#!/bin/bash
# round-2: wide SATs (NEXT-3) parity, stress worker, GPU tests, quick wide timing
set -u
mkdir -p gpurun_out
timeout -s KILL 300 python -m pytest tests/test_gpu_wide.py -x -q --timeout 200 2>&1 | tail -8
SAT_LIB=$PWD/paper_conf_ipps_emotofthni18_b200/libsat_stress.so timeout -s KILL 400 python tests/stress_worker.py --reps 2 --verbose > gpurun_out/stress_worker.log 2>&1
echo "stress rc=$?"; grep -v '^libsat watchdog\|^case' gpurun_out/stress_worker.log | tail -3; grep '^case' gpurun_out/stress_worker.log | tail -1; grep -m2 '^libsat watchdog' gpurun_out/stress_worker.log
timeout -s KILL 600 python -m pytest tests -m "gpu and not slow" -q --timeout 300 -x 2>&1 | tail -3
timeout -s KILL 200 python tools/bench_wide.py 2>&1 | tail -6
