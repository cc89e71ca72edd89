#!/bin/bash
# compute-sanitizer runs of the protocol-stress worker (every shipped kernel family, small ragged shapes,
# one shape per variant) with the product libsat.so; logs -> gpurun_out/sanitize_<tool>.log
set -u
mkdir -p gpurun_out
for tool in ${SANITIZE_TOOLS:-memcheck racecheck synccheck}; do
  timeout -s KILL ${SANITIZE_TIMEOUT:-600} compute-sanitizer --tool $tool --print-limit 20 --error-exitcode 9 \
    python tests/stress_worker.py --quick --reps 1 > gpurun_out/sanitize_$tool.log 2>&1
  echo "sanitize $tool rc=$?" | tee -a gpurun_out/sanitize_$tool.log
  tail -4 gpurun_out/sanitize_$tool.log
done
