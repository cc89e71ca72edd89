#!/bin/bash
set -u
mkdir -p gpurun_out
timeout -s KILL 600 python tools/graph_sweep.py --sizes 1024,2048,4096,8192 --variants 1,5,6,7,8,3,9 --dtype i32 2>&1 | grep '^{' | tee gpurun_out/sweep_medium.jsonl
timeout -s KILL 300 python tools/sweep_variants.py --n 16384 --dtype i32 --variants 1,5,6,7,3,9 --orders 0 --reps 20 2>&1 | grep '^{' | tee -a gpurun_out/sweep_medium.jsonl
timeout -s KILL 600 python -m pytest tests/test_gpu_chain.py -x -q --timeout 300 2>&1 | tail -3 | tee gpurun_out/pytest_chain.log
timeout -s KILL 900 python bench.py --steps 20 --warmup 5 --no-cpu --no-e2e 2>&1 | tail -1 > gpurun_out/bench_chain.json
