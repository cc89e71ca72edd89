#!/bin/bash
set -u
mkdir -p gpurun_out
timeout -s KILL 300 python -m pytest tests/test_gpu_parity.py -k box -x -q --timeout 200 2>&1 | tail -2
for occ in 8 0; do echo "occ_max $occ"; SAT_BOX_BAND_OCC=$occ timeout -s KILL 200 python tools/bench_box.py 2>&1 | tail -6; done
