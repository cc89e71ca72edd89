#!/bin/bash
# per-tile timelines at medium sizes (instrumented build) + the bench line with the chain projection
set -u
mkdir -p gpurun_out
for n in 2048 4096 8192; do
  timeout -s KILL 120 python tools/trace_dump.py --n $n --variant 1 2>&1 | tail -1
done
timeout -s KILL 120 python tools/trace_dump.py --n 4096 --variant 0 2>&1 | tail -1
timeout -s KILL 120 python tools/trace_dump.py --n 8192 --variant 3 2>&1 | tail -1
timeout -s KILL 900 python bench.py --steps 20 --warmup 5 --no-cpu 2>&1 | tail -1 > gpurun_out/bench_chain.json
