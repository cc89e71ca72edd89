#!/bin/bash
set -u
for cfg in 0 1 2; do for occ in 4 5; do echo "cfg $cfg occ $occ"; SAT_BOX_BAND_CFG=$cfg SAT_BOX_BAND_OCC=$occ timeout -s KILL 200 python tools/bench_box.py 2>&1 | sed -n 2,3p; done; done
