#!/bin/bash
set -u
timeout -s KILL 300 python -m pytest tests/test_gpu_parity.py -k box -x -q --timeout 200 2>&1 | tail -2
timeout -s KILL 200 python tools/bench_box.py 2>&1 | tail -6
