#!/bin/bash
# look-back width sweep (round 2): experimental build with LB / DW variants, device time via CUDA graphs
set -u
mkdir -p gpurun_out
export SAT_LIB=paper_conf_ipps_emotofthni18_b200/libsat_exp_r02a.so
timeout -s KILL 400 python tools/graph_sweep.py --sizes 2048,4096,8192 --variants 1,18,19,20,21,24,3,22,23 --dtype i32 2>&1 | tee gpurun_out/sweep_lb_small.jsonl | tail -30
for v in 3 22 23 13; do
  timeout -s KILL 200 python tools/sweep_variants.py --n 16384 --dtype f32 --variants $v --orders 0,512 --reps 20 2>&1 | tee -a gpurun_out/sweep_lb_16k.jsonl
  timeout -s KILL 200 python tools/sweep_variants.py --n 32768 --dtype f32 --variants $v --orders 512 --reps 20 2>&1 | tee -a gpurun_out/sweep_lb_32k.jsonl
done
