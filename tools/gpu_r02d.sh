#!/bin/bash
# round-2 session: stress worker (jitter + watchdog build), GPU tests, L2-prefetch size sweep
set -u
mkdir -p gpurun_out
SAT_LIB=$PWD/paper_conf_ipps_emotofthni18_b200/libsat_stress.so timeout -s KILL 400 python tests/stress_worker.py --reps 2 --verbose > gpurun_out/stress_worker.log 2>&1
echo "stress rc=$?"; grep -v '^libsat watchdog\|^case' gpurun_out/stress_worker.log | tail -3; grep '^case' gpurun_out/stress_worker.log | tail -1; grep -m2 '^libsat watchdog' gpurun_out/stress_worker.log
timeout -s KILL 600 python -m pytest tests -m "gpu and not slow" -q --timeout 300 -x 2>&1 | tail -3
for pf in 0 1; do
  SAT_L2_PREFETCH=$pf timeout -s KILL 200 python tools/graph_sweep.py --sizes 4096,8192 --variants 1,3 --dtype i32 2>&1 | grep '^{' | sed "s/^{/{\"l2_prefetch\": $pf, /" | tee -a gpurun_out/sweep_prefetch_sizes.jsonl
  SAT_L2_PREFETCH=$pf timeout -s KILL 200 python tools/sweep_variants.py --n 16384 --dtype i32 --variants 1,3 --orders 0 --reps 20 2>&1 | grep '^{' | sed "s/^{/{\"l2_prefetch\": $pf, /" | tee -a gpurun_out/sweep_prefetch_sizes.jsonl
  SAT_L2_PREFETCH=$pf timeout -s KILL 200 python tools/sweep_variants.py --n 65536 --dtype i32 --variants 3 --orders 512 --reps 5 2>&1 | grep '^{' | sed "s/^{/{\"l2_prefetch\": $pf, /" | tee -a gpurun_out/sweep_prefetch_sizes.jsonl
done
