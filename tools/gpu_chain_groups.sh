#!/bin/bash
set -u
timeout -s KILL 600 python -m pytest tests/test_gpu_chain.py -x -q --timeout 300 2>&1 | tail -3
for g in 0 8 4; do echo "group $g"; SAT_CHAIN_GROUP=$g timeout -s KILL 300 python tools/chain_proj.py 2>&1 | tail -4 | head -3; done
