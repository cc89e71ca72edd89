#!/bin/bash
# Round-end evidence: bench line, ncu launch list of the same command, one ncu --set full capture of
# the SAT kernel (32K x 32K fp32) and of the box filter (r = 8), smoke.  Outputs under gpurun_out/.
set -u
mkdir -p gpurun_out
timeout -s KILL 900 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; tail -1 gpurun_out/bench_full.json | cut -c1-400
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e > gpurun_out/launches_bench.log 2>&1; echo "launch list rows: $(wc -l < gpurun_out/launches.csv)"
timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:sat_ -s 3 -c 1 -o gpurun_out/prof_full -f python tools/ncu_one.py 32768 f32 -1 4 > gpurun_out/ncu_full.log 2>&1; tail -1 gpurun_out/ncu_full.log
timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:box -s 3 -c 1 -o gpurun_out/prof_box -f python tools/ncu_box_one.py 8 > gpurun_out/ncu_box.log 2>&1; tail -1 gpurun_out/ncu_box.log
