#!/bin/bash
# L2-prefetch modes 1 (plain) vs 2 (evict_last) across sizes and paths
set -u
for pf in 1 2; do
  echo "== pf $pf"
  SAT_L2_PREFETCH=$pf timeout -s KILL 200 python tools/graph_sweep.py --sizes 4096,8192 --variants -1 --dtype i32 2>&1 | grep "^{"
  SAT_L2_PREFETCH=$pf timeout -s KILL 200 python tools/sweep_variants.py --n 16384 --dtype i32 --variants 3 --orders 0 --reps 20 2>&1 | grep "^{"
  SAT_L2_PREFETCH=$pf timeout -s KILL 200 python tools/sweep_variants.py --n 65536 --dtype i32 --variants 3 --orders 512 --reps 5 2>&1 | grep "^{"
  SAT_L2_PREFETCH=$pf timeout -s KILL 200 python tools/u8_probe.py 32768 5 2>&1 | grep variant
  SAT_L2_PREFETCH=$pf SAT_LIB=$PWD/paper_conf_ipps_emotofthni18_b200/libsat.so timeout -s KILL 300 python tools/exp_candidates.py --chain 4 2>&1 | grep "^{"
done
